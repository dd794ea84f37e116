#!/bin/bash
# quick re-verification of the current build on one B200: smoke, full GPU suite, default bench line, X1
cd "$(dirname "$0")/.."
O=gpurun_out/check; mkdir -p $O
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke=$?"
timeout 1500 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "tests=$?"; tail -2 $O/gpu_tests.log
timeout 600 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "benchC2=$?"; tail -1 $O/bench_C2.json | cut -c1-300
timeout 600 python bench.py --config X1 > $O/bench_X1.json 2> $O/bench_X1.err; echo "benchX1=$?"; tail -1 $O/bench_X1.json | cut -c1-300
