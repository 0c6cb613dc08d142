"""One warm pack -> index -> find step on a config (for ncu captures of single kernels).
Usage: python tools/one_step.py CONFIG [opt=val ...]"""
import sys
import torch
sys.path.insert(0, '.')
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth

P = synth.make_pair(sys.argv[1])
for kv in sys.argv[2:]:
    k, v = kv.split('='); gm.set_option(k, int(v))
R = torch.from_numpy(P.R).cuda(); Q = torch.from_numpy(P.Q).cuda()
for it in range(2):
    Rs = gm.pack(R); Qs = gm.pack(Q)
    idx = gm.index_build(Rs, P.ls, P.L)
    m = gm.find_mems(idx, Qs)
    print(len(m), flush=True)
    for h in (m, idx, Qs, Rs): h.free()
torch.cuda.synchronize()
