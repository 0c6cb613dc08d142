#!/bin/bash
# ncu --set full of single kernels on one config (second, warm step). Usage: gpu_prof3.sh CFG TAG kernel:skip ...
CFG=$1; TAG=$2; shift 2
mkdir -p gpurun_out
for ks in "$@"; do
  k=${ks%%:*}; sk=${ks##*:}
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s $sk -c 1 -o gpurun_out/prof_${k}_${CFG}_$TAG python tools/one_step.py $CFG > gpurun_out/ncu_${k}_$TAG.log 2>&1; tail -1 gpurun_out/ncu_${k}_$TAG.log
done
