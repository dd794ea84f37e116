#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/c1 gpurun_out/check2
timeout 300 python scripts/c1_tiles.py > gpurun_out/c1/scan.log 2>&1; echo "scan=$?"; tail -10 gpurun_out/c1/scan.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/check2/gpu_tests.log 2>&1; echo "tests=$?"; tail -2 gpurun_out/check2/gpu_tests.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/check2/smoke.log 2>&1; echo "smoke=$?"
