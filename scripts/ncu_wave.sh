#!/bin/bash
# ncu full capture of one steady-state wave1d_kernel launch (W1 best tile) + the launch list
cd "$(dirname "$0")/.."
O=gpurun_out/wave; mkdir -p $O
timeout 600 ncu --set full --clock-control none --import-source on -k regex:wave1d -s 300 -c 1 -o $O/prof_wave -f python scripts/wave_one.py ${1:-4} ${2:-8192} > $O/ncu_full.log 2>&1; echo "ncu_full=$?"
[ -f $O/prof_wave.ncu-rep ] && ncu -i $O/prof_wave.ncu-rep --page raw --csv > $O/prof_wave_raw.csv 2>/dev/null
[ -f $O/prof_wave.ncu-rep ] && ncu -i $O/prof_wave.ncu-rep --page details > $O/prof_wave_details.txt 2>/dev/null
echo done
