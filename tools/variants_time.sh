#!/bin/bash
# time every build_variants/*/libaabft.so with tools/time_gemm.py (N, dtype from args)
mkdir -p gpurun_out
for v in build_variants/*/libaabft.so; do
  AABFT_LIB=$v timeout ${TO:-90} python tools/time_gemm.py ${1:-4096} ${2:-f64} >> gpurun_out/variants.jsonl 2>&1
done
