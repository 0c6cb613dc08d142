mkdir -p gpurun_out
for c in c4 c3 c5_l300 c5_l50; do
timeout 600 python tools/ab.py $c pdl=1 l2_persist=8,l2_window=1 l2_persist=16,l2_window=1 l2_persist=24,l2_window=1 l2_persist=32,l2_window=1 l2_persist=48,l2_window=1 pdl=1 > gpurun_out/l2_$c.json 2>gpurun_out/l2_$c.err; python -c "
import json,sys; d=json.load(open('gpurun_out/l2_$c.json')); print(d.pop('config'), {k:(v['ms'],v['find_ms'],v['identical']) for k,v in d.items()})"; tail -2 gpurun_out/l2_$c.err
done
