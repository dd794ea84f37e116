#!/bin/bash
# a13 for the 3D configs on the current kernels: full-space sweeps of C5 and C4 (min of 5) with the
# committed calibration (CAL=1 first recalibrates the 3D kinds); logs + JSON under gpurun_out/sw3
cd "$(dirname "$0")/.."
O=gpurun_out/sw3; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || exit 1
CALF=profiles/hw_params_b200.json
if [ -n "$CAL" ]; then
  timeout 1500 python -m paper_conf_ppopp_prajapatirradg17_b200.tune calibrate --kinds 4,5 --base $CALF --out $O/hw_params_b200.json > $O/calibrate.log 2>&1; echo "cal=$?"
  CALF=$O/hw_params_b200.json
fi
for c in ${CFGS:-C5 C4}; do
  timeout 2400 python -m paper_conf_ppopp_prajapatirradg17_b200.tune sweep --config $c --space full --limit 100000 --budget ${BUDGET:-1500} --cal $CALF --out $O/sweep_$c.json > $O/sweep_$c.log 2>&1; echo "sweep $c=$?"
done
