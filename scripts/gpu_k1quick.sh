#!/bin/bash
# K1 change check: 2D GPU parity + the default bench line
cd "$(dirname "$0")/.."
O=gpurun_out/k1q; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "2d or pair or threads or C1 or C2 or C3 or T0 or custom or mid" > $O/tests.log 2>&1; echo "tests=$?"; tail -2 $O/tests.log
timeout 600 python bench.py --no-cpu-baseline > $O/bench_C2.json 2> $O/bench_C2.err; echo "bench=$?"; tail -1 $O/bench_C2.json | cut -c1-200
timeout 600 python bench.py --no-cpu-baseline --config C3 > $O/bench_C3.json 2> $O/bench_C3.err; echo "bench3=$?"; tail -1 $O/bench_C3.json | cut -c1-200
