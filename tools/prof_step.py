"""One pipeline step of a config for ncu's per-kernel DRAM table:
    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum \
        --clock-control none --csv --log-file out.csv python tools/prof_step.py c4
Profiles one graph launch (the step bench.py times) between cudaProfilerStart/Stop:
run ncu with --profile-from-start off. Prints the MEM count."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem, synth  # noqa: E402

P = synth.make_pair(sys.argv[1] if len(sys.argv) > 1 else "c4")
for kv in filter(None, os.environ.get("GM_OPTS", "").split(",")):  # e.g. GM_OPTS=index_tiled=1
    k, v = kv.split("=")
    gpumem.set_option(k, int(v))
R, Q = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
pl.run(R, Q)  # measuring run + capture + first launch: not profiled
pl.result()
torch.cuda.synchronize()
torch.cuda.profiler.start()  # ncu --profile-from-start off: only this graph launch
pl.run(R, Q)
n = pl.result()
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("mems", n)
pl.free()
