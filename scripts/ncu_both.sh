#!/bin/bash
# one full ncu capture of the bench's steady-state K1 launch (C2) and of K2 (C4, C5), exported as CSV pages
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
export HHC_BENCH_ALLOW_SHORT=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 60 -c 1 -o gpurun_out/prof_c2 -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_c2.log 2>&1; echo "ncu2=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex3d -s 40 -c 1 -o gpurun_out/prof_c4 -f python bench.py --config C4 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_c4.log 2>&1; echo "ncu4=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex3d -s 20 -c 1 -o gpurun_out/prof_c5 -f python bench.py --config C5 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_c5.log 2>&1; echo "ncu5=$?"
for r in c2 c4 c5; do
  [ -f gpurun_out/prof_$r.ncu-rep ] || continue
  ncu -i gpurun_out/prof_$r.ncu-rep --page raw --csv > gpurun_out/prof_${r}_raw.csv 2>/dev/null
  ncu -i gpurun_out/prof_$r.ncu-rep --page details --csv > gpurun_out/prof_${r}_details.csv 2>/dev/null
done
