#!/bin/bash
# Bench every config on one GPU (bench.py lines -> gpurun_out/bench_<cfg>_<tag>.json): bench_all.sh TAG
TAG=${1:-x}
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench_c4_$TAG.json 2> gpurun_out/bench_c4_$TAG.err; python tools/jq.py gpurun_out/bench_c4_$TAG.json
for c in c1 c2 c3 c5_l20 c5_l50 c5_l100 c5_l300; do
timeout 300 python bench.py --config $c --steps 20 --no-cpu-baseline > gpurun_out/bench_${c}_$TAG.json 2> gpurun_out/bench_${c}_$TAG.err; python tools/jq.py gpurun_out/bench_${c}_$TAG.json | head -2
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>&1; tail -c 400 gpurun_out/bench_ref_$TAG.json
