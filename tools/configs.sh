#!/bin/bash
mkdir -p gpurun_out
for w in c1 c3 c4 c5; do
  timeout 900 python bench.py --workload $w --steps ${STEPS:-3} --warmup 3 --no-e2e --no-cpu >> gpurun_out/configs.jsonl 2> gpurun_out/configs_$w.err
done
