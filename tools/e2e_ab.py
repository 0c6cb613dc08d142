"""e2e (host inputs -> sorted triples in pinned host memory) per q_chunks setting:
    python tools/e2e_ab.py c4 1 4 8 16
Median wall time of 10 runs per setting (bench.py's e2e protocol), the H2D-only time of
the same bytes, and whether the results agree."""
import json
import os
import statistics
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth  # noqa: E402

cfg = sys.argv[1]
Ks = [int(x) for x in sys.argv[2:]] or [1, 16]
P = synth.make_pair(cfg)
Rh, Qh = torch.from_numpy(P.R).pin_memory(), torch.from_numpy(P.Q).pin_memory()
dev = torch.empty(len(P.R) + len(P.Q), dtype=torch.uint8, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
out = {"config": cfg}
ts = []
for _ in range(10):  # the copies alone
    torch.cuda.synchronize()
    t = time.perf_counter()
    dev[:len(P.R)].copy_(Rh, non_blocking=True)
    dev[len(P.R):].copy_(Qh, non_blocking=True)
    torch.cuda.synchronize()
    ts.append(time.perf_counter() - t)
out["h2d_only_ms"] = round(1e3 * statistics.median(ts), 3)
ref = None
for K in Ks:
    gm.set_option("q_chunks", K)
    pl = gm.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
    host = None
    ts = []
    for i in range(12):
        flush.zero_()
        torch.cuda.synchronize()
        t = time.perf_counter()
        pl.run_host(Rh, Qh)
        n = pl.result()
        if host is None:
            host = torch.empty((n * 5 // 4 + 1, 3), dtype=torch.uint32, pin_memory=True)
        host[:n].copy_(pl.view_u32(), non_blocking=True)
        torch.cuda.current_stream().synchronize()
        if i >= 2:
            ts.append(time.perf_counter() - t)
    got = host[:n].clone()
    same = ref is None or bool(torch.equal(got, ref))
    ref = got if ref is None else ref
    out[f"K{K}"] = {"ms_median": round(1e3 * statistics.median(ts), 3), "ms_min": round(1e3 * min(ts), 3),
                    "identical": same}
    pl.free()
gm.set_option("q_chunks", 8)
print(json.dumps(out))
