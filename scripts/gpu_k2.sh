#!/bin/bash
# 3D (K2) iteration: 3D parity subset, then quick C4/C5 bench lines
cd "$(dirname "$0")/.."
OUT=gpurun_out/${OUT:-k2}; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { echo build failed; tail $OUT/build.log; exit 1; }
timeout ${TT:-900} python -m pytest tests -m gpu -x -q -k "${PYTEST_K:-3d or threads or mid_size or dist_local or tiny or C4 or C5 or flag}" > $OUT/tests.log 2>&1
echo "tests=$?"; tail -5 $OUT/tests.log
for c in ${CFGS:-C4 C5}; do
  HHC_BENCH_ALLOW_SHORT=1 timeout 300 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --no-e2e ${BARGS} > $OUT/q_$c.json 2> $OUT/q_$c.err
  python -c "import json;d=json.loads(open('$OUT/q_$c.json').read().splitlines()[-1]);print('$c', d['config'].get('tile'), d['config'].get('threads'), round(d['value'],1), round(d['ms_per_step'],2), d['roofline']['frac'])" 2>/dev/null || { echo "$c FAILED"; tail -3 $OUT/q_$c.err; }
done
