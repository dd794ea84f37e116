#!/bin/bash
# 3D kernel iteration: 3D parity subset, then C4/C5 tile timings (TMA path and, for A/B, the cp.async path)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "3d or mid_size or virtual or tiny or HEAT3D or LAPLACIAN3D" > gpurun_out/gpu_k2_tests.log 2>&1; echo "tests=$?"; tail -3 gpurun_out/gpu_k2_tests.log
T4=${T4:-"10,8,8,64:512 6,16,8,64:512 8,16,4,64:512 8,8,8,64:256 8,8,16,32:512 8,12,8,64:512"}
T5=${T5:-"8,6,8,64:256 8,16,4,64:256 8,8,8,64:256 8,12,4,64:512"}
HHC_EXP_T=64 timeout 600 python scripts/exp_tiles.py C4 $T4 2>&1 | sed 's/^/C4 tma /'
HHC_EXP_T=32 timeout 600 python scripts/exp_tiles.py C5 $T5 2>&1 | sed 's/^/C5 tma /'
if [ -n "$AB" ]; then
HHC_NO_TMA=1 HHC_EXP_T=64 timeout 600 python scripts/exp_tiles.py C4 $T4 2>&1 | sed 's/^/C4 old /'
fi
