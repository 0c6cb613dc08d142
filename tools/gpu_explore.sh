#!/bin/bash
# Exploration session: launch list of the C4 bench + stage comparisons of sort impls.
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c4_x.csv python bench.py --config c4 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_c4_x.log 2>&1; tail -1 gpurun_out/ncu_launch_c4_x.log
timeout 300 python tools/stage_cmp.py c4 sort_impl=1 sort_impl=0 2>&1 | tail -2
timeout 300 python tools/stage_cmp.py c5_l20 sort_impl=1 sort_impl=0 2>&1 | tail -2
