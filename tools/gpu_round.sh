#!/bin/bash
# Full evidence pass for one round: GPU tests, default bench (N=1, with cpu_baseline + e2e),
# C5 L=20 bench, launch lists + ncu --set full of k_find. Usage: tools/gpu_round.sh TAG
TAG=${1:-r1}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu_$TAG.txt
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_default_$TAG.json 2> gpurun_out/bench_default_$TAG.err; cat gpurun_out/bench_default_$TAG.json; tail -3 gpurun_out/bench_default_$TAG.err
timeout 300 python bench.py --config c5_l20 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_l20_$TAG.json 2>&1; tail -c 600 gpurun_out/bench_c5_l20_$TAG.json; echo
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2>&1; tail -c 600 gpurun_out/bench_ref_$TAG.json; echo
bash tools/profile_round.sh $TAG c4
bash tools/profile_round.sh $TAG c5_l20
