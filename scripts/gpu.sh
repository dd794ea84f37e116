#!/bin/bash
# One documented GPU-box runner (called through gpurun; logs under gpurun_out/$OUT).
#   scripts/gpu.sh tests            full `pytest -m gpu` + smoke
#   scripts/gpu.sh bench C2 C3 ...  bench lines (default arguments) per config
#   scripts/gpu.sh ncu CFG          ncu --set full of the dominant kernel of one bench step
#   scripts/gpu.sh launches CFG     ncu launch list (gpu__time_duration) of one bench step
#   scripts/gpu.sh quick CFG [tile:threads ...]   short bench lines for tiles (no cpu baseline / e2e)
cd "$(dirname "$0")/.."
OUT=gpurun_out/${OUT:-run}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()" > "$OUT/build.log" 2>&1 || { echo "build failed"; tail -20 "$OUT/build.log"; exit 1; }
cmd=$1; shift
case "$cmd" in
tests)
  timeout 300 python __graft_entry__.py smoke > "$OUT/smoke.log" 2>&1; echo "smoke=$? $(tail -1 $OUT/smoke.log)"
  timeout ${TEST_TIMEOUT:-2400} python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} > "$OUT/gpu_tests.log" 2>&1
  echo "tests=$?"; tail -3 "$OUT/gpu_tests.log";;
bench)
  for c in "$@"; do
    timeout 900 python bench.py --config $c ${BENCH_ARGS} > "$OUT/bench_$c.json" 2> "$OUT/bench_$c.err"
    echo "bench $c rc=$?: $(tail -c 600 $OUT/bench_$c.json)"
  done;;
quick)
  c=$1; shift
  for t in "$@"; do
    HHC_BENCH_ALLOW_SHORT=1 timeout 300 python bench.py --config $c --tile ${t%%:*} --threads ${t##*:} --steps ${STEPS:-3} --warmup 3 --no-cpu-baseline --no-e2e > "$OUT/q.json" 2> "$OUT/q.err"
    python -c "import json;d=json.loads(open('$OUT/q.json').read().splitlines()[-1]);print('$c $t', d['value'], d['ms_per_step'], d['roofline']['frac'])" 2>/dev/null | tee -a $OUT/quick.txt || { echo "$c $t FAILED"; tail -3 "$OUT/q.err"; }
  done;;
ncu)
  c=$1; k=${KREGEX:-hex}
  HHC_BENCH_ALLOW_SHORT=1 timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$k -s ${SKIP:-40} -c ${COUNT:-1} \
     -o "$OUT/prof_$c" -f python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > "$OUT/ncu_$c.log" 2>&1
  echo "ncu=$?"; tail -3 "$OUT/ncu_$c.log";;
launches)
  c=$1
  HHC_BENCH_ALLOW_SHORT=1 timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file "$OUT/launches_$c.csv" python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > "$OUT/launches_$c.log" 2>&1
  echo "launches=$?";;
*) echo "unknown command $cmd"; exit 2;;
esac
