#!/bin/bash
# a12/a13 for the 3D configs on the current kernels: recalibrate the 3D kinds, then
# full-space and near-best sweeps of C5 and C4 (min of 5), logs + JSON under gpurun_out/sw3
cd "$(dirname "$0")/.."
O=gpurun_out/sw3; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || exit 1
T=python
timeout 1500 $T -m paper_conf_ppopp_prajapatirradg17_b200.tune calibrate --kinds 4,5 --base profiles/hw_params_b200.json --out $O/hw_params_b200.json > $O/calibrate.log 2>&1; echo "cal=$?"
for c in C5 C4; do
  timeout 2400 $T -m paper_conf_ppopp_prajapatirradg17_b200.tune sweep --config $c --space full --limit 100000 --budget ${BUDGET:-1500} --cal $O/hw_params_b200.json --out $O/sweep_$c.json > $O/sweep_$c.log 2>&1; echo "sweep $c=$?"
done
