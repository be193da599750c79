#!/bin/bash
# fast iteration: gemm parity tests + bench without the slow legs
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "${TESTK:-gemm or fault or clean}" > gpurun_out/quick_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/quick_pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu ${BENCH_ARGS} > gpurun_out/quick_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/quick_bench.log
