mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_scatter -s 1 -c 1 -o gpurun_out/prof_scat32 python tools/prof_step.py c5_l20 > gpurun_out/p1.log 2>&1; tail -2 gpurun_out/p1.log
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_scatter -s 5 -c 1 -o gpurun_out/prof_scat64 python tools/prof_step.py c5_l20 > gpurun_out/p2.log 2>&1; tail -2 gpurun_out/p2.log
