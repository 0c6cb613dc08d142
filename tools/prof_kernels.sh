# ncu --set full captures of single kernels (tuning): prof_kernels.sh TAG
TAG=${1:-x}
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scatter -s 3 -c 1 -o gpurun_out/prof_scatter_c5_$TAG python tools/opt_bench.py c5_l20 base > gpurun_out/ncu_sc_$TAG.log 2>&1; tail -2 gpurun_out/ncu_sc_$TAG.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_bs_local -s 1 -c 1 -o gpurun_out/prof_bslocal_c4_$TAG python tools/opt_bench.py c4 base > gpurun_out/ncu_bl_$TAG.log 2>&1; tail -2 gpurun_out/ncu_bl_$TAG.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ptrs_fill -s 1 -c 1 -o gpurun_out/prof_ptrs_c4_$TAG python tools/opt_bench.py c4 base > gpurun_out/ncu_pf_$TAG.log 2>&1; tail -2 gpurun_out/ncu_pf_$TAG.log
