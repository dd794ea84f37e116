#!/bin/bash
# f3 on one B200: GPU parity of the wavefront schedule, smoke, the W1 tile sweep
cd "$(dirname "$0")/.."
O=gpurun_out/wave; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k wavefront > $O/tests.log 2>&1; echo "tests=$?"; tail -3 $O/tests.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke=$?"; tail -2 $O/smoke.log
timeout 900 python scripts/wave_sweep.py > $O/sweep.log 2>&1; echo "sweep=$?"; tail -1 $O/sweep.log | cut -c1-1500
