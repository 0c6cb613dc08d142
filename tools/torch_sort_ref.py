"""Library reference point: torch.sort (CUB radix sort) on the same sizes as our sorts."""
import time, torch
g = torch.Generator(device='cuda').manual_seed(0)
for n, hi, name in ((13_000_000, 2**56, 'u64 56-bit 13M'), (13_000_000, 2**26, 'u32 26-bit 13M (int32)')):
    k = torch.randint(0, hi, (n,), device='cuda', dtype=torch.int64, generator=g)
    if hi <= 2**31: k = k.int()
    for i in range(3):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        v, idx = torch.sort(k, stable=True)
        torch.cuda.synchronize(); dt = time.perf_counter() - t0
    print(f"torch.sort {name}: {dt*1e3:.3f} ms", flush=True)
