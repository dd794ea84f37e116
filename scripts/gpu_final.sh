#!/bin/bash
# round-end evidence on one B200: full GPU suite, smoke, every config's bench line, the reference arm,
# the ncu launch list of the default bench command and one full capture of its dominant kernel
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/final
O=gpurun_out/final
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke=$?"
timeout 1800 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "tests=$?"; tail -2 $O/gpu_tests.log
timeout 600 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "benchC2=$?"; tail -1 $O/bench_C2.json | cut -c1-300
for c in C1 C3 C4 C5; do
  timeout 900 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "bench$c=$?"; tail -1 $O/bench_$c.json | cut -c1-200
done
timeout 600 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err; echo "ref=$?"; tail -1 $O/bench_ref.json | cut -c1-200
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_C2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $O/ncu_launch.log 2>&1; echo "ncu_launch=$?"
HHC_BENCH_ALLOW_SHORT=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 60 -c 1 -o $O/prof_c2 -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $O/ncu_full.log 2>&1; echo "ncu_full=$?"
[ -f $O/prof_c2.ncu-rep ] && ncu -i $O/prof_c2.ncu-rep --page raw --csv > $O/prof_c2_raw.csv 2>/dev/null
