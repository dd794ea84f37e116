#!/bin/bash
# iteration check: GPU parity tests (2D or all), then the C2 bench line + sweep of a few tiles
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest_gpu=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_iter.log 2>&1; echo "bench=$?"; tail -1 gpurun_out/bench_iter.log | cut -c1-200
if [ -n "$TILES2" ]; then HHC_EXP_T=256 timeout 600 python scripts/exp_tiles.py C2 $TILES2; fi
