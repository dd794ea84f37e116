#!/bin/bash
# quick check: smoke, 2D parity subset, C2 bench + a few tiles, ncu of one C2 launch
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke=$?"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "small or threads or tiny or coeff or mid or virtual" > gpurun_out/gpu_small.log 2>&1; echo "tests=$?"; tail -1 gpurun_out/gpu_small.log
rm -f gpurun_out/q_*.log
for t in ${TILES:-16,20,512,0:512 32,12,512,0:512 32,12,512,0:256 24,16,512,0:512 12,8,512,0:256}; do
  HHC_BENCH_ALLOW_SHORT=1 timeout 120 python bench.py --config C2 --tile ${t%%:*} --threads ${t##*:} --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/q_$t.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/q_$t.log').read().splitlines()[-1]);print('$t', d['value'], d['ms_per_step'], d['roofline']['frac'])" 2>/dev/null || tail -2 gpurun_out/q_$t.log
done
if [ -n "$NCU" ]; then
HHC_BENCH_ALLOW_SHORT=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 20 -c 1 -o gpurun_out/prof_c2 -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu.log 2>&1; echo "ncu=$?"
fi
