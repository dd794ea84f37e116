#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest_gpu=$?"; tail -3 gpurun_out/pytest_gpu.log
HHC_EXP_T=256 timeout 600 python scripts/exp_tiles.py C2 32,12,512:384 24,16,512:384 16,6,512:192 16,6,512:256 12,8,512:192
HHC_EXP_T=64 timeout 600 python scripts/exp_tiles.py C4 10,8,8,64:512 8,8,8,32:256 10,6,8,32:256
HHC_EXP_T=32 timeout 600 python scripts/exp_tiles.py C5 8,6,8,64:256 8,4,8,64:256
