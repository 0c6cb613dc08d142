python tools/bench_sort.py 13000000
ncu --set full --clock-control none -k regex:"k_onesweep|k_hist_all" -s 9 -c 2 -o gpurun_out/prof_sort python tools/bench_sort.py 13000000 > gpurun_out/ncu_sort.log 2>&1; tail -2 gpurun_out/ncu_sort.log
