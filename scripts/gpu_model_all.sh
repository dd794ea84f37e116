#!/bin/bash
# a12/a13 on one GPU on the current kernels: calibration, tile sweeps (RMSE, chosen-tile gaps) and
# model-driven selection for C2 (2D), C4 and C5 (3D)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
M="python -m paper_conf_ppopp_prajapatirradg17_b200.tune"
timeout 1200 $M calibrate --out gpurun_out/hw_params_b200.json > gpurun_out/calibrate.log 2>&1; echo "calibrate=$?"; tail -1 gpurun_out/calibrate.log | cut -c1-300
CAL=gpurun_out/hw_params_b200.json
timeout 1300 $M sweep --config C2 --cal $CAL --budget 1000 --out gpurun_out/sweep_C2_r01.json > gpurun_out/sweep_C2.log 2>&1; echo "sweepC2=$?"; tail -1 gpurun_out/sweep_C2.log | cut -c1-600
timeout 900 $M select --config C2 --cal $CAL --out gpurun_out/select_C2_r01.json > gpurun_out/select_C2.log 2>&1; echo "selectC2=$?"; tail -1 gpurun_out/select_C2.log | cut -c1-400
for c in C4 C5; do
timeout 900 $M sweep --config $c --cal $CAL --budget 500 --limit 200 --reps 2 --out gpurun_out/sweep_${c}_r01.json > gpurun_out/sweep_$c.log 2>&1; echo "sweep$c=$?"; tail -1 gpurun_out/sweep_$c.log | cut -c1-600
timeout 900 $M select --config $c --cal $CAL --reps 2 --max-measure 30 --out gpurun_out/select_${c}_r01.json > gpurun_out/select_$c.log 2>&1; echo "select$c=$?"; tail -1 gpurun_out/select_$c.log | cut -c1-400
done
