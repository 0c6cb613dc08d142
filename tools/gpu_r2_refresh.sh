#!/bin/bash
# Round-2 evidence refresh after the tiled index (tag r2e): GPU tests, bench lines of every
# config, ncu launch lists + k_find --set full (C4, C5 L=20), per-kernel DRAM tables (C2,
# C3, C4, C5 L=20), the four sanitizers. Usage: tools/gpu_r2_refresh.sh TAG
TAG=${1:-r2e}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu_$TAG.txt
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
bash tools/bench_all.sh $TAG > /dev/null 2>&1; echo bench done
for c in c4 c5_l20; do bash tools/profile_round.sh $TAG $c; done
for c in c2 c3 c4 c5_l20; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/ncu_tab_${c}_$TAG.csv python tools/prof_step.py $c > gpurun_out/ncu_tab_${c}_$TAG.log 2>&1; echo "ncu $c rc=$?"
done
for tool in memcheck racecheck synccheck initcheck; do
  arg=quick; [ $tool = memcheck ] && arg=full
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_cases.py $arg > gpurun_out/san_${tool}_$TAG.log 2>&1
  echo "$tool rc=$?"
done
ls gpurun_out | wc -l
