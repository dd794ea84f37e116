#!/bin/bash
# f3 on one B200 after a K3 change: parity, smoke, sweep, the W1 bench line
cd "$(dirname "$0")/.."
O=gpurun_out/wave; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k wavefront > $O/tests.log 2>&1; echo "tests=$?"; tail -2 $O/tests.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke=$?"; tail -1 $O/smoke.log
timeout 900 python scripts/wave_sweep.py > $O/sweep.log 2>&1; echo "sweep=$?"; tail -1 $O/sweep.log | cut -c1-1200
timeout 600 python bench.py --config W1 > $O/bench_W1.json 2> $O/bench_W1.err; echo "benchW1=$?"; tail -1 $O/bench_W1.json | cut -c1-1500; tail -3 $O/bench_W1.err
