#!/bin/bash
# f2: the 1D model validated directly -- Jacobi-1D calibration added to the committed constants, X1 sweep, selection
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/x1m
O=gpurun_out/x1m
M="python -m paper_conf_ppopp_prajapatirradg17_b200.tune"
timeout 900 $M calibrate --kinds 7 --base profiles/hw_params_b200.json --out $O/hw_params_b200.json > $O/calibrate.log 2>&1; echo "calibrate=$?"; tail -3 $O/calibrate.log | cut -c1-400
CAL=$O/hw_params_b200.json
timeout 900 $M sweep --config X1 --cal $CAL --budget 600 --reps 2 --out $O/sweep_X1_r01.json > $O/sweep_X1.log 2>&1; echo "sweepX1=$?"; tail -1 $O/sweep_X1.log | cut -c1-1200
timeout 900 $M select --config X1 --cal $CAL --reps 2 --max-measure 20 --out $O/select_X1_r01.json > $O/select_X1.log 2>&1; echo "selectX1=$?"; tail -1 $O/select_X1.log | cut -c1-400
