#!/bin/bash
# a12/a13 on the GPU box: calibration, then sweeps (SURVEY 8(d) full space) and Eq. 31 selections.
#   scripts/gpu_model.sh calibrate | sweep CFG BUDGET_S [LIMIT] | select CFG GEOM BUDGET_S
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/model profiles/r02
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/model/build.log 2>&1 || exit 1
case "$1" in
calibrate) timeout 3000 python -m paper_conf_ppopp_prajapatirradg17_b200.tune calibrate ${KINDS:+--kinds $KINDS} ${BASE:+--base $BASE} > gpurun_out/model/calibrate.log 2>&1
           echo "calibrate=$?"; cp profiles/hw_params_b200.json gpurun_out/model/; tail -2 gpurun_out/model/calibrate.log;;
sweep) timeout $(( $3 + 600 )) python -m paper_conf_ppopp_prajapatirradg17_b200.tune sweep --config $2 --space ${SPACE:-full} --budget $3 --limit ${4:-100000} --out gpurun_out/model/sweep_$2_${SPACE:-full}.json > gpurun_out/model/sweep_$2_${SPACE:-full}.log 2>&1
       echo "sweep $2 = $?"; tail -c 600 gpurun_out/model/sweep_$2_${SPACE:-full}.log;;
finish) timeout 1500 python -m paper_conf_ppopp_prajapatirradg17_b200.tune finish --config $2 --measure --src $3 --out gpurun_out/model/sweep_$2.json > gpurun_out/model/finish_$2.log 2>&1
       echo "finish $2 = $?"; tail -c 1500 gpurun_out/model/finish_$2.log;;
select) timeout $(( $4 + 900 )) python -m paper_conf_ppopp_prajapatirradg17_b200.tune select --config $2 --geometry $3 --budget $4 > gpurun_out/model/select_$2_$3.log 2>&1
        echo "select $2 $3 = $?"; cp profiles/r02/select_$2_$3.json gpurun_out/model/ 2>/dev/null; tail -c 800 gpurun_out/model/select_$2_$3.log;;
esac
