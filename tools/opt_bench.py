"""Stage times of the pipeline under option settings (tuning experiments, not the bench).

    python tools/opt_bench.py c5_l20 radix_bits=8 sort_impl=1 ...
Each argument after the config is one option set, applied alone ('base' = defaults);
comma-separate several options in one set (radix_bits=8,find_grid=296)."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth  # noqa: E402

DEFAULTS = {"find_grid": 0, "find_spill": 64, "out_capacity": 0, "use_bitmap": 1, "static_lb": 0, "sort_impl": 0,
            "index_msd": 0, "small_sort": 0, "radix_bits": 0, "rank_sectors": -1, "rec8": -1, "index_fused": 0,
            "pdl": 1, "index_alg1": 0, "pipe_events": 1}  # stage times (event nodes cost ~50 us)
cfg = sys.argv[1]
P = synth.make_pair(cfg)
R = torch.from_numpy(P.R).cuda()
Q = torch.from_numpy(P.Q).cuda()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
ref = None
for spec in sys.argv[2:] or ["base"]:
    for k, v in DEFAULTS.items():
        gm.set_option(k, v)
    if spec != "base":
        for kv in spec.split(","):
            k, v = kv.split("=")
            gm.set_option(k, int(v))
    pl = gm.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
    tot, prof, steps = [], {}, 10
    for i in range(3 + steps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        pl.run(R, Q)
        b.record()
        n = pl.result()
        b.synchronize()
        if i >= 3:
            tot.append(a.elapsed_time(b))
            for k, (t, _) in pl.profile().items():
                prof[k] = prof.get(k, 0.0) + t / steps
    out = pl.numpy()
    if ref is None:
        ref = out
    same = (out.shape == ref.shape) and bool((out == ref).all())
    print(f"{cfg} {spec:28s} step {sum(tot) / steps:.4f} ms  n={n} same={same} | "
          + " ".join(f"{k}={v:.3f}" for k, v in prof.items()), flush=True)
    pl.free()
