#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest_gpu=$?"; tail -3 gpurun_out/pytest_gpu.log
python scripts/exp_compute_only.py 4 512x512x512 64 ${T4:-8,8,8,64:512 8,4,8,64:256 4,4,16,64:256 8,4,8,32:256}
python scripts/exp_compute_only.py 5 768x768x768 32 ${T5:-8,4,8,64:256 8,4,32,32:512}
