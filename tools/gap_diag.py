"""Where does a step's time go between stages? Device events between the public API
calls (same stream) + the library's per-stage events; host time per call."""
import sys, time
import torch
sys.path.insert(0, '.')
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth
cfg = sys.argv[1] if len(sys.argv) > 1 else 'c4'
P = synth.make_pair(cfg)
R = torch.from_numpy(P.R).cuda(); Q = torch.from_numpy(P.Q).cuda()
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
gm.profile_enable(True)
for it in range(6):
    flush.zero_(); torch.cuda.synchronize(); gm.profile_read()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
    ht = []
    ev[0].record(); t0 = time.perf_counter()
    Rs = gm.pack(R); ht.append(time.perf_counter()); ev[1].record()
    Qs = gm.pack(Q); ht.append(time.perf_counter()); ev[2].record()
    idx = gm.index_build(Rs, P.ls, P.L); ht.append(time.perf_counter()); ev[3].record()
    m = gm.find_mems(idx, Qs); ht.append(time.perf_counter()); ev[4].record()
    torch.cuda.synchronize()
    prof = gm.profile_read()
    d = [ev[i].elapsed_time(ev[i + 1]) for i in range(4)]
    h = [1e3 * (ht[0] - t0)] + [1e3 * (ht[i] - ht[i - 1]) for i in range(1, 4)]
    st = {k: v[0] for k, v in prof.items()}
    print(f"it{it} dev: packR {d[0]:.3f} packQ {d[1]:.3f} index {d[2]:.3f} find+sort {d[3]:.3f} total {sum(d):.3f} | "
          f"host: {' '.join(f'{x:.3f}' for x in h)} | stages: " + " ".join(f"{k}={v:.3f}" for k, v in st.items()), flush=True)
    for x in (m, idx, Qs, Rs): x.free()
