"""Radix-sort robustness: random vs pre-sorted vs reversed vs constant-high-bits inputs."""
import sys, time
import torch
sys.path.insert(0, '.')
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm
n = int(sys.argv[1]) if len(sys.argv) > 1 else 13_000_000
g = torch.Generator(device='cuda').manual_seed(0)
base = torch.randint(0, 2**28, (n, 3), device='cuda', dtype=torch.int32, generator=g)
cases = {}
cases['random'] = base
srt = base[torch.argsort(base[:, 0].long() * 2**32 + base[:, 1].long())]
cases['sorted'] = srt.contiguous()
cases['reversed'] = srt.flip(0).contiguous()
c = base.clone(); c[:, 0] = 12345; cases['same_r'] = c
c2 = base.clone(); c2[:, 0] = torch.arange(n, device='cuda', dtype=torch.int32) // 64; cases['blocky_r'] = c2
for name, t in cases.items():
    for i in range(2):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        m = gm.merge_sorted([t])
        torch.cuda.synchronize(); dt = time.perf_counter() - t0
    print(f"{name:10s} n={n} {dt*1e3:8.3f} ms", flush=True)
