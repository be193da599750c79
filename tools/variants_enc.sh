#!/bin/bash
mkdir -p gpurun_out
for v in build_variants/*/libaabft.so; do
  AABFT_LIB=$v timeout 300 python tools/time_encode.py ${1:-4096} ${2:-f64} >> gpurun_out/variants_enc.jsonl 2>&1
done
