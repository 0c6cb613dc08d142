#!/bin/bash
# Round-2 evidence pass: GPU tests, bench lines of every config, ncu launch lists + k_find
# --set full (C4, C5 L=20), per-kernel DRAM tables (C2, C3, C4, C5 L=20), sanitizers,
# merge / e2e / band experiments, paper-experiment analogues. Usage: tools/gpu_r2_final.sh TAG
TAG=${1:-r2}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu_$TAG.txt
timeout 2000 python -m pytest tests -m gpu -q > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
bash tools/bench_all.sh $TAG > /dev/null 2>&1; echo bench done
for c in c4 c5_l20; do bash tools/profile_round.sh $TAG $c; done
for c in c2 c3 c4 c5_l20; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/ncu_tab_${c}_$TAG.csv python tools/prof_step.py $c > gpurun_out/ncu_tab_${c}_$TAG.log 2>&1; echo "ncu $c rc=$?"
done
for tool in memcheck racecheck synccheck initcheck; do
  arg=quick; [ $tool = memcheck ] && arg=full
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_cases.py $arg > gpurun_out/san_${tool}_$TAG.log 2>&1
  echo "$tool rc=$?"
done
timeout 600 python tools/merge_bench.py c5_l20 2 4 8 > gpurun_out/merge_c5_l20_$TAG.json 2>&1
timeout 600 python tools/merge_bench.py c4 2 4 8 > gpurun_out/merge_c4_$TAG.json 2>&1
timeout 600 python tools/e2e_ab.py c4 1 8 > gpurun_out/e2e_c4_$TAG.json 2>&1
timeout 900 python tools/band_bench.py c5_l20 0 64000000 16000000 4000000 > gpurun_out/band_c5_l20_$TAG.json 2>&1
timeout 900 python tools/band_bench.py c4 0 64000000 16000000 > gpurun_out/band_c4_$TAG.json 2>&1
timeout 1200 python tools/experiments.py --out gpurun_out/${TAG}_experiments > gpurun_out/experiments_$TAG.log 2>&1; echo "experiments rc=$?"
ls gpurun_out | wc -l
