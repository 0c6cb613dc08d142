"""Micro-benchmark of the radix sort through gpumem_merge_sorted (random triples)."""
import sys, time
import torch
sys.path.insert(0, '.')
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm
n = int(sys.argv[1]) if len(sys.argv) > 1 else 13_000_000
g = torch.Generator(device='cuda').manual_seed(0)
t = torch.randint(0, 2**28, (n, 3), device='cuda', dtype=torch.int32, generator=g)
for i in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    m = gm.merge_sorted([t])
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    print(f"n={n} merge_sorted (8 passes) {dt*1e3:.3f} ms  -> {n*24*8/dt/1e9:.1f} GB/s eff", flush=True)
v = m.numpy()
k = v[:, 0].astype('u8') << 32 | v[:, 1]
assert (k[1:] >= k[:-1]).all()
print("sorted ok")
