#!/bin/bash
# Profiles for profiles/: launch list of the bench command + one ncu --set full of k_find.
TAG=${1:-r1}; CFG=${2:-c4}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}_$TAG.csv python bench.py --config $CFG --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-d9 > gpurun_out/ncu_launch_${CFG}_$TAG.log 2>&1; tail -1 gpurun_out/ncu_launch_${CFG}_$TAG.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_find -s 1 -c 1 -o gpurun_out/prof_find_${CFG}_$TAG python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-d9 > gpurun_out/ncu_full_${CFG}_$TAG.log 2>&1; tail -1 gpurun_out/ncu_full_${CFG}_$TAG.log
