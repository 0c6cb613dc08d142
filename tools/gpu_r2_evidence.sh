#!/bin/bash
# Round-2 evidence: sanitizers, per-kernel DRAM table, merge timing. Usage: tools/gpu_r2_evidence.sh TAG
TAG=${1:-r2}
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  arg=quick; [ $tool = memcheck ] && arg=full
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_cases.py $arg > gpurun_out/san_${tool}_$TAG.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/san_${tool}_$TAG.log
done
for c in c2 c3 c4 c5_l20; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/ncu_tab_${c}_$TAG.csv python tools/prof_step.py $c > gpurun_out/ncu_tab_${c}_$TAG.log 2>&1; echo "ncu $c rc=$?"
done
timeout 600 python tools/merge_bench.py c5_l20 2 4 8 > gpurun_out/merge_c5_l20_$TAG.json 2>&1; tail -2 gpurun_out/merge_c5_l20_$TAG.json
