#!/bin/bash
mkdir -p gpurun_out
for v in build_variants/*/libaabft.so; do
  AABFT_LIB=$v timeout 300 python tools/time_gemm.py 4096 f64 >> gpurun_out/variants.jsonl 2>&1
  AABFT_LIB=$v timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "fault or fused or clean or gemm" 2>&1 | tail -1 >> gpurun_out/variants.jsonl
done
