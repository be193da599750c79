#!/bin/bash
# Step-0 box facts: FP64/FP32 pipe throughput + cuBLAS DGEMM/SGEMM context ceiling.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/step0_clocks.csv &
SMI=$!
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fp64_pipes tools/microbench/fp64_pipes.cu
/tmp/fp64_pipes | tee gpurun_out/step0_pipes.jsonl
python - <<'PY' | tee gpurun_out/step0_cublas.jsonl
import torch, json, time
for dt, n in [(torch.float64, 4096), (torch.float64, 8192), (torch.float32, 8192)]:
    a = torch.rand(n, n, dtype=dt, device='cuda'); b = torch.rand(n, n, dtype=dt, device='cuda')
    for _ in range(3): torch.matmul(a, b)
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(10):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); torch.matmul(a, b); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    print(json.dumps({"kernel": f"cublas_{dt}", "n": n, "ms": best, "tflops": 2 * n**3 / best / 1e9}))
PY
kill $SMI
