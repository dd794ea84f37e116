#!/bin/bash
# Refit the EXACT/EXACT_G/EXACT_GW/Leff constants from the recorded calibration instances (device
# registers for Eq. 11), then re-predict every committed sweep with them and time the model argmins.
cd "$(dirname "$0")/.."
O=gpurun_out/mdl; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || exit 1
M=paper_conf_ppopp_prajapatirradg17_b200.tune
timeout 1200 python -m $M refit --cal profiles/hw_params_b200.json --out $O/hw_params_b200.json > $O/refit.log 2>&1; echo "refit=$?"
for c in ${CFGS:-C2 C3 C4 C5}; do
  timeout 1500 python -m $M finish --config $c --cal $O/hw_params_b200.json --src profiles/r02/sweep_$c.json --repredict --measure --out $O/sweep_$c.json > $O/finish_$c.log 2>&1; echo "finish $c=$?"
done
