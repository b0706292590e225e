set -x
B="python bench.py --config c4 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline --no-secondary --peak-seconds 0.2"
timeout 300 $B > gpurun_out/c4p_plain.json 2>gpurun_out/c4p_plain.err; echo rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/c4p_launches.csv $B > gpurun_out/c4p_ncu1.log 2>&1; echo rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:zdot_kernel -s 40 -c 1 -o gpurun_out/prof_dot_c4_r02 $B > gpurun_out/c4p_ncu2.log 2>&1; echo rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:zgemm -s 30 -c 1 -o gpurun_out/prof_gemm_c4_r02 $B > gpurun_out/c4p_ncu3.log 2>&1; echo rc=$?
