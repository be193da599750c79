#!/bin/bash
mkdir -p gpurun_out
for v in build_variants/*/libaabft.so; do
  AABFT_LIB=$v timeout 300 python tools/time_gemm.py ${N:-4096} >> gpurun_out/variants.jsonl 2>&1
done
