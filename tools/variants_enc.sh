#!/bin/bash
# encode variants: stage probe (c2 FP64 and c3 FP32) + encode parity, per build_variants/*
mkdir -p gpurun_out
for v in build_variants/*/libaabft.so; do
  echo "$v" >> gpurun_out/variants_enc.log
  AABFT_LIB=$v timeout 300 python tools/stage_probe.py 4096 f64 64 >> gpurun_out/variants_enc.log 2>&1
  AABFT_LIB=$v timeout 300 python tools/stage_probe.py 8192 f32 64 >> gpurun_out/variants_enc.log 2>&1
  AABFT_LIB=$v timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "encode or full_size_c2" 2>&1 | tail -1 >> gpurun_out/variants_enc.log
done
