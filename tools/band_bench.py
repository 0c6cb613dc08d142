"""F2 row sweep experiment: the whole path with a band-local R window,
R kept in host memory, for several band lengths; time per run (wall, the call
synchronises per band), windows, MEMs carried across windows, and identity with the
whole-R result.
    python tools/band_bench.py c5_l20 0 64000000 16000000 4000000"""
import json
import os
import statistics
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth  # noqa: E402

cfg = sys.argv[1]
bands = [int(x) for x in sys.argv[2:]] or [0]
P = synth.make_pair(cfg)
Rh = torch.from_numpy(P.R).pin_memory().numpy()
Q = gm.pack(torch.from_numpy(P.Q).cuda())
out = {"config": cfg, "R_bp": len(P.R), "Q_bp": len(P.Q)}
ref = None
for b in bands:
    ts, st, m = [], None, None
    for i in range(4):
        torch.cuda.synchronize()
        t = time.perf_counter()
        m, st = gm.find_mems_banded(Rh, Q, P.ls, P.L, b)
        torch.cuda.synchronize()
        if i:
            ts.append(time.perf_counter() - t)
        if i < 3:
            m.free()
    got = m.view_u32().clone()
    same = ref is None or bool(torch.equal(got, ref))
    ref = got if ref is None else ref
    out[f"band_{b}"] = {"ms": round(1e3 * statistics.median(ts), 2), "identical": same, **st}
    m.free()
print(json.dumps(out))
