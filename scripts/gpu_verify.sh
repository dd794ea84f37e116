#!/bin/bash
# full GPU parity suite + smoke + default bench line (round-end equivalent)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke=$?"
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests.log 2>&1; echo "tests=$?"; tail -3 gpurun_out/gpu_tests.log
timeout 600 python bench.py > gpurun_out/bench_default.log 2>&1; echo "bench=$?"; tail -1 gpurun_out/bench_default.log | cut -c1-1500
