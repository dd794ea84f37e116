#!/bin/bash
# one GPU session: parity tests, calibration, sweep, selection, bench, ncu launch list
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_info.txt
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest_gpu=$?"
timeout 600 python -m paper_conf_ppopp_prajapatirradg17_b200.tune calibrate > gpurun_out/calibrate.log 2>&1; echo "calibrate=$?"
cp profiles/hw_params_b200.json gpurun_out/ 2>/dev/null
timeout 900 python -m paper_conf_ppopp_prajapatirradg17_b200.tune sweep --config C2 --budget 500 --out gpurun_out/sweep_C2_r01.json > gpurun_out/sweep.log 2>&1; echo "sweep=$?"
timeout 600 python -m paper_conf_ppopp_prajapatirradg17_b200.tune select --config C2 --out gpurun_out/select_C2_r01.json > gpurun_out/select.log 2>&1; echo "select=$?"
timeout 600 python bench.py > gpurun_out/bench_full.log 2>&1; echo "bench=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_C2.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1; echo "ncu_launch=$?"
