mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_pipeline.py -x -q > gpurun_out/tp.log 2>&1; tail -15 gpurun_out/tp.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 300 python bench.py --steps 30 --no-cpu-baseline > gpurun_out/bp.json 2> gpurun_out/bp.err; python tools/jq.py gpurun_out/bp.json; tail -5 gpurun_out/bp.err
timeout 300 python bench.py --config c5_l20 --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/bp5.json 2> gpurun_out/bp5.err; python tools/jq.py gpurun_out/bp5.json; tail -5 gpurun_out/bp5.err
