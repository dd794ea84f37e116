#!/bin/bash
# end-of-session evidence: full GPU suite, smoke, C2/C3/C1 bench lines, ncu launch list + full capture of C2
cd "$(dirname "$0")/.."
O=gpurun_out/final2; mkdir -p $O
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke=$?"
timeout 1500 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "tests=$?"; tail -2 $O/gpu_tests.log
for c in C2 C3 C1; do
  timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "bench$c=$?"; tail -1 $O/bench_$c.json | cut -c1-200
done
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_C2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $O/ncu_launch.log 2>&1; echo "ncu_launch=$?"
HHC_BENCH_ALLOW_SHORT=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 60 -c 1 -o $O/prof_c2 -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $O/ncu_full.log 2>&1; echo "ncu_full=$?"
