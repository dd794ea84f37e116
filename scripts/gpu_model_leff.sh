#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/m4
O=gpurun_out/m4
M="python -m paper_conf_ppopp_prajapatirradg17_b200.tune"
timeout 1500 $M calibrate --out $O/hw_params_b200.json > $O/calibrate.log 2>&1; echo "calibrate=$?"; tail -1 $O/calibrate.log | cut -c1-400
CAL=$O/hw_params_b200.json
for c in C4 C5; do
timeout 900 $M sweep --config $c --cal $CAL --budget 500 --limit 200 --reps 2 --out $O/sweep_${c}_r01.json > $O/sweep_$c.log 2>&1; echo "sweep$c=$?"; tail -1 $O/sweep_$c.log | cut -c1-900
timeout 900 $M select --config $c --cal $CAL --reps 2 --max-measure 30 --out $O/select_${c}_r01.json > $O/select_$c.log 2>&1; echo "select$c=$?"; tail -1 $O/select_$c.log | cut -c1-400
done
timeout 1300 $M sweep --config C2 --cal $CAL --budget 900 --out $O/sweep_C2_r01.json > $O/sweep_C2.log 2>&1; echo "sweepC2=$?"; tail -1 $O/sweep_C2.log | cut -c1-900
timeout 900 $M select --config C2 --cal $CAL --out $O/select_C2_r01.json > $O/select_C2.log 2>&1; echo "selectC2=$?"; tail -1 $O/select_C2.log | cut -c1-400
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke=$?"; tail -1 $O/smoke.log
timeout 1800 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "tests=$?"; tail -2 $O/gpu_tests.log
