#!/bin/bash
# every config on 1 GPU (bench lines, no CPU baseline / e2e)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for c in ${CONFIGS:-C1 C3 C4 C5}; do
  timeout 400 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.log 2>&1; echo "$c=$?"; tail -1 gpurun_out/bench_$c.log | cut -c1-400
done
