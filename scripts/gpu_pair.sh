#!/bin/bash
cd "$(dirname "$0")/.."
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "pair" > gpurun_out/pair.log 2>&1; echo pair=$?; grep -E "Error|passed|failed" gpurun_out/pair.log | head -3
for t in ${TILES}; do
  HHC_BENCH_ALLOW_SHORT=1 timeout 120 python bench.py --config C2 --tile ${t%%:*} --threads ${t##*:} --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/q_$t.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/q_$t.log').read().splitlines()[-1]);print('$t', d['value'], d['ms_per_step'], d['roofline']['frac'])" 2>/dev/null || tail -1 gpurun_out/q_$t.log
done
if [ -n "$NCUTILE" ]; then
HHC_BENCH_ALLOW_SHORT=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 20 -c 1 -o gpurun_out/prof_pair -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --tile ${NCUTILE%%:*} --threads ${NCUTILE##*:} > gpurun_out/ncu.log 2>&1; echo ncu=$?
fi
