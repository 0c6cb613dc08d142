mkdir -p gpurun_out
timeout 300 python tools/gap_diag.py c4 > gpurun_out/gap_c4.log 2>&1; cat gpurun_out/gap_c4.log | tail -4
GM_BENCH_NOCLK=1 timeout 300 python bench.py --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/b_noclk.json 2>&1; python -c "import json;d=json.loads(open('gpurun_out/b_noclk.json').read().strip().splitlines()[-1]);print('noclk',d['ms_per_step'],d['stage_ms'])"
timeout 300 python bench.py --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/b_clk.json 2>&1; python -c "import json;d=json.loads(open('gpurun_out/b_clk.json').read().strip().splitlines()[-1]);print('clk',d['ms_per_step'],d['stage_ms'])"
