"""Pack kernel alone: device time per call for R-sized and Q-sized inputs (tuning)."""
import sys
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth  # noqa: E402
P = synth.make_pair("c4")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for name, x in (("R", torch.from_numpy(P.R).cuda()), ("Q", torch.from_numpy(P.Q).cuda())):
    ts = []
    for i in range(12):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        s = gm.pack(x)
        b.record()
        b.synchronize()
        s.free()
        if i >= 2:
            ts.append(a.elapsed_time(b))
    t = sum(ts) / len(ts)
    print(f"{gm.LIB_PATH.split('/')[-2]} pack {name}: {t * 1e3:.1f} us  {1.25 * x.numel() / t / 1e6:.0f} GB/s", flush=True)
