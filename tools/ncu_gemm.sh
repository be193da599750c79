#!/bin/bash
mkdir -p gpurun_out
timeout 900 ncu ${NCU_EXTRA} --set full --clock-control none --import-source on -k regex:${KERN:-gemm_f64} -s ${SKIP:-2} -c 1 -o gpurun_out/${OUT:-prof_gemm_f64} -f python tools/prof_gemm.py ${N:-4096} 2 ${DT:-f64} > gpurun_out/ncu_gemm.log 2>&1
