"""Radix-sort robustness: random vs pre-sorted vs reversed vs constant-high-bits inputs."""
import sys, time
import torch
sys.path.insert(0, '.')
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm
n = int(sys.argv[1]) if len(sys.argv) > 1 else 13_000_000
if len(sys.argv) > 2: gm.set_option('radix_bits', int(sys.argv[2]))
only = sys.argv[3] if len(sys.argv) > 3 else None
g = torch.Generator(device='cuda').manual_seed(0)
base = torch.randint(0, 2**28, (n, 3), device='cuda', dtype=torch.int32, generator=g)
cases = {}
cases['random'] = base
srt = base[torch.argsort(base[:, 0].long() * 2**32 + base[:, 1].long())]
cases['sorted'] = srt.contiguous()
cases['reversed'] = srt.flip(0).contiguous()
c = base.clone(); c[:, 0] = 12345; cases['same_r'] = c
c2 = base.clone(); c2[:, 0] = torch.arange(n, device='cuda', dtype=torch.int32) // 64; cases['blocky_r'] = c2
import statistics
for name, t in cases.items():
    if only and name != only: continue
    ts = []
    for i in range(12):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        m = gm.merge_sorted([t])
        torch.cuda.synchronize(); ts.append(time.perf_counter() - t0)
        m.free()
    ts = sorted(ts[2:])
    print(f"{name:10s} n={n} min {ts[0]*1e3:7.3f} med {statistics.median(ts)*1e3:7.3f} max {ts[-1]*1e3:7.3f} ms", flush=True)
