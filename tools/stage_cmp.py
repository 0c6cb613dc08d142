"""Per-stage device times (CUDA-event profile) of full steps under different option settings.
Usage: python tools/stage_cmp.py CONFIG opt=val[,opt=val] [opt=val ...]"""
import sys
import torch
sys.path.insert(0, '.')
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth

cfg = sys.argv[1]
settings = sys.argv[2:] or ["radix_bits=0"]
P = synth.make_pair(cfg)
R = torch.from_numpy(P.R).cuda(); Q = torch.from_numpy(P.Q).cuda()
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
gm.profile_enable(True)
for s in settings * 2:  # second round = warm
    for kv in s.split(','):
        k, v = kv.split('='); gm.set_option(k, int(v))
    acc = {}
    reps = 10
    for it in range(reps + 2):
        flush.zero_(); torch.cuda.synchronize()
        gm.profile_read()
        Rs = gm.pack(R); Qs = gm.pack(Q)
        idx = gm.index_build(Rs, P.ls, P.L)
        m = gm.find_mems(idx, Qs); n = len(m)
        torch.cuda.synchronize()
        prof = gm.profile_read()
        for h in (m, idx, Qs, Rs): h.free()
        if it >= 2:
            for k, (ms, nl) in prof.items():
                acc[k] = acc.get(k, 0.0) + ms / reps
    tot = sum(acc.values())
    print(f"{cfg} {s:28s} mems={n} total={tot:.3f} ms  " + " ".join(f"{k}={v:.3f}" for k, v in acc.items()), flush=True)
