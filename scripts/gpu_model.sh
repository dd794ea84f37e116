#!/bin/bash
# a12/a13 on one GPU: calibration micro-benchmarks, C2 tile sweep (RMSE, chosen-tile gaps), model-driven selection
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m paper_conf_ppopp_prajapatirradg17_b200.tune calibrate --out gpurun_out/hw_params_b200.json > gpurun_out/calibrate.log 2>&1; echo "calibrate=$?"; tail -1 gpurun_out/calibrate.log | cut -c1-300
timeout 1500 python -m paper_conf_ppopp_prajapatirradg17_b200.tune sweep --config C2 --cal gpurun_out/hw_params_b200.json --budget 1100 --out gpurun_out/sweep_C2_r01.json > gpurun_out/sweep.log 2>&1; echo "sweep=$?"; tail -1 gpurun_out/sweep.log | cut -c1-600
timeout 900 python -m paper_conf_ppopp_prajapatirradg17_b200.tune select --config C2 --cal gpurun_out/hw_params_b200.json --out gpurun_out/select_C2_r01.json > gpurun_out/select.log 2>&1; echo "select=$?"; tail -1 gpurun_out/select.log | cut -c1-400
HHC_EXP_T=64 timeout 600 python scripts/exp_tiles.py C4 ${T4X:-10,8,8,64:512 8,6,8,64:256 6,6,8,64:256 8,8,8,32:256 8,6,8,32:128 8,6,8,32:256 10,6,8,32:256 8,4,8,32:128}
