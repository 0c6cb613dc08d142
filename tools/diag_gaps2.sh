mkdir -p gpurun_out
nproc; uptime
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/t2.log 2>&1; tail -1 gpurun_out/t2.log
uptime; ps aux --sort=-%cpu | head -8
for i in 1 2; do
timeout 300 python bench.py --steps 30 > gpurun_out/b2_$i.json 2>&1; python -c "import json;d=json.loads(open('gpurun_out/b2_$i.json').read().strip().splitlines()[-1]);print('run$i',d['ms_per_step'],d['host_ms_per_step'],d['step_ms_minmax'],d['e2e']['ms_per_step'])"
done
