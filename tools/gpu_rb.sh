timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/tests_all.log 2>&1; tail -3 gpurun_out/tests_all.log
timeout 300 python tools/stage_cmp.py c4 radix_bits=8 radix_bits=0 2>&1 | tail -2
timeout 300 python tools/stage_cmp.py c5_l20 radix_bits=8 radix_bits=0 2>&1 | tail -2
timeout 120 python tools/bench_sort2.py 13000000 0
