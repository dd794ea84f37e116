#!/bin/bash
# usage: TILES="t,s1,s2,s3:threads[:ng] ..." CONFIG=C2 bash scripts/gpu_tiles.sh
cd "$(dirname "$0")/.."
for t in ${TILES}; do
  IFS=: read -r tile thr ng <<< "$t"
  HHC_FORCE_NG=${ng:-0} HHC_BENCH_ALLOW_SHORT=1 timeout 120 python bench.py --config ${CONFIG:-C2} --tile $tile --threads $thr --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/q.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/q.log').read().splitlines()[-1]);print('$t', d['value'], d['ms_per_step'], d['roofline']['frac'])" 2>/dev/null || (echo "$t FAIL"; tail -2 gpurun_out/q.log)
done
