#!/bin/bash
# 2D kernel iteration: 2D parity subset, C2 bench line, a few C2 tiles; 3D tS2=16 tiles
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "2d or pair or threads or tiny or coeff or mid_size" > gpurun_out/gpu_k1_tests.log 2>&1; echo "tests=$?"; tail -1 gpurun_out/gpu_k1_tests.log
HHC_BENCH_ALLOW_SHORT=1 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | cut -c1-260
HHC_EXP_T=256 timeout 600 python scripts/exp_tiles.py C2 ${T2:-32,12,512:384 24,16,512:384 32,10,512:384 40,8,512:384 32,12,256:256} 2>&1 | sed 's/^/C2 /'
HHC_EXP_T=64 timeout 600 python scripts/exp_tiles.py C4 ${T4:-10,8,8,64:512 8,8,16,64:512 6,8,16,64:512 8,6,16,64:512 8,4,16,64:512 6,6,16,64:512 4,8,16,64:512} 2>&1 | sed 's/^/C4 /'
HHC_EXP_T=32 timeout 600 python scripts/exp_tiles.py C5 ${T5:-8,6,8,64:256 8,8,16,64:512 6,8,16,64:512 8,4,16,64:512} 2>&1 | sed 's/^/C5 /'
