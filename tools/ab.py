"""A/B timing of library options on the pipeline bench.py times:
    python tools/ab.py c4 heavy_tail=0 heavy_tail=1 [--steps 20]
Each setting: a fresh pipeline (options read at capture), warm-up, then --steps steps
timed with CUDA events (L2 flushed between steps, as bench.py does); prints the mean ms
per step, the live find stage and whether the MEMs equal the first setting's."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth  # noqa: E402

args = [a for a in sys.argv[1:] if not a.startswith("--")]
steps = 20
if "--steps" in sys.argv:
    steps = int(sys.argv[sys.argv.index("--steps") + 1])
    args = [a for a in args if a != str(steps)]
cfg, settings = args[0], args[1:] or ["pdl=1"]
P = synth.make_pair(cfg)
R, Q = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
ref, out = None, {"config": cfg}
for st in settings:
    opts = dict(kv.split("=") for kv in st.split(",")) if st else {}
    for k, v in opts.items():
        gm.set_option(k, int(v))
    gm.set_option("pipe_events", 2)
    pl = gm.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
    for _ in range(3):
        pl.run(R, Q)
        pl.result()
    ts, fs = [], []
    for _ in range(steps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        pl.run(R, Q)
        b.record()
        pl.result()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
        fs.append(pl.profile().get("find", (0.0, 0))[0])
    got = pl.view_u32().clone()
    same = ref is None or bool(torch.equal(got, ref))
    ref = got if ref is None else ref
    out[st] = {"ms": round(statistics.mean(ts), 4), "ms_min": round(min(ts), 4), "find_ms": round(statistics.mean(fs), 4),
               "mems": int(got.shape[0]), "identical": same, "attempts": pl.stats()["attempts"]}
    pl.free()
    for k in opts:
        gm.set_option(k, {"heavy_tail": 1, "pdl": 1, "find_spill": 64, "sort_impl": 0, "radix_bits": 0,
                          "rank_sectors": -1, "rec8": -1, "find_grid": 0, "find_hints": -1}.get(k, 0))
    gm.set_option("pipe_events", 0)
print(json.dumps(out))
