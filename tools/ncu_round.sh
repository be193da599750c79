#!/bin/bash
# ncu launch list of the bench command + one full capture of each hot kernel
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --campaign 0 > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_f64 -s 2 -c 1 -o gpurun_out/prof_gemm_f64 -f python tools/prof_gemm.py 4096 2 > gpurun_out/ncu_gemm.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"encode|check_kernel|topp" -s 4 -c 4 -o gpurun_out/prof_small -f python tools/prof_gemm.py 4096 2 > gpurun_out/ncu_small.log 2>&1
ls -la gpurun_out
