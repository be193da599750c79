#!/bin/bash
# build_variant.sh NAME "EXTRA NVCC FLAGS" -> build_variants/NAME/libaabft.so (tuning experiments)
set -e
mkdir -p build_variants/$1
AABFT_BUILD_OUT=build_variants/$1/libaabft.so AABFT_BUILD_OBJ=build_variants/$1/obj AABFT_EXTRA_FLAGS="$2" \
  python -m paper_conf_dsn_braunhw14_b200.build > build_variants/$1/build.log 2>&1
