"""One F2 row sweep for ncu (k_find of one band): python tools/band_prof.py c5_l20 16000000"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth  # noqa: E402

P = synth.make_pair(sys.argv[1])
band = int(sys.argv[2])
Q = gm.pack(torch.from_numpy(P.Q).cuda())
m, st = gm.find_mems_banded(torch.from_numpy(P.R).pin_memory().numpy(), Q, P.ls, P.L, band)
print(st)
