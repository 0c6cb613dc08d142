"""Host-side breakdown of one bench step (wall clock with syncs) to find gaps."""
import sys, time
import torch
sys.path.insert(0, '.')
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth
cfg = sys.argv[1] if len(sys.argv) > 1 else 'c5_l20'
P = synth.make_pair(cfg)
R = torch.from_numpy(P.R).cuda(); Q = torch.from_numpy(P.Q).cuda()
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
def t(): torch.cuda.synchronize(); return time.perf_counter()
for it in range(8):
    flush.zero_()
    t0 = t(); Rs = gm.pack(R); t1 = t(); Qs = gm.pack(Q); t2 = t()
    idx = gm.index_build(Rs, P.ls, P.L); t3 = t()
    m = gm.find_mems(idx, Qs); t4 = t()
    for h in (m, idx, Qs, Rs): h.free()
    t5 = t()
    print(f"it{it} pack {1e3*(t1-t0):.2f} {1e3*(t2-t1):.2f} index {1e3*(t3-t2):.2f} find {1e3*(t4-t3):.2f} free {1e3*(t5-t4):.2f} total {1e3*(t5-t0):.2f}", flush=True)
