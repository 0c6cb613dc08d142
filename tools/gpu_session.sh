#!/bin/bash
# One GPU-box session: tests, bench, optional ncu. Usage: tools/gpu_session.sh [tag] [ncu]
TAG=${1:-run}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
timeout 600 python bench.py --steps 30 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c4_$TAG.json 2> gpurun_out/bench_c4_$TAG.err; cat gpurun_out/bench_c4_$TAG.json; tail -3 gpurun_out/bench_c4_$TAG.err
timeout 300 python bench.py --config c5_l20 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_l20_$TAG.json 2>&1; tail -c 1500 gpurun_out/bench_c5_l20_$TAG.json; echo
if [ "$2" = "ncu" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_find -s 1 -c 1 -o gpurun_out/prof_find_c4_$TAG python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_$TAG.log 2>&1; tail -2 gpurun_out/ncu_full_$TAG.log
fi
if [ "$3" = "full" ]; then
timeout 900 python -m pytest tests -m gpu -x -q -k full_size > gpurun_out/full_size_$TAG.log 2>&1; tail -3 gpurun_out/full_size_$TAG.log
fi
