"""Time the K9 merge kernel (gpumem_merge_sorted) on the real shard runs of a config:
    python tools/merge_bench.py c5_l20 [G ...]
Prints per G the median of 20 timed merges (CUDA events) and whether the merged bytes
equal the single pipeline's result."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem, synth  # noqa: E402
from paper_conf_ipps_abu_dolehkac14_b200.dist import shard_range  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c5_l20"
Gs = [int(x) for x in sys.argv[2:]] or [2, 4, 8]
P = synth.make_pair(cfg)
Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
pl.run(Rt, Qt)
pl.result()
whole = pl.view_u32().clone()
pl.free()
out = {"config": cfg, "mems": int(whole.shape[0])}
for G in Gs:
    runs = []
    for g in range(G):
        pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L, shard_range(len(P.Q), g, G))
        pl.run(Rt, Qt)
        pl.result()
        runs.append(pl.view_u32().clone().view(torch.int32))
        pl.free()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    ts = []
    for i in range(25):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        m = gpumem.merge_sorted(runs)
        b.record()
        torch.cuda.synchronize()
        if i >= 5:
            ts.append(a.elapsed_time(b))
        same = bool(torch.equal(m.view_u32(), whole))
        m.free()
    nbytes = whole.numel() * 4 * 2
    med = statistics.median(ts)
    out[f"G{G}"] = {"ms_median": round(med, 4), "ms_min": round(min(ts), 4), "identical": same,
                    "GBps_read_write": round(nbytes / med / 1e6, 1)}
print(json.dumps(out))
