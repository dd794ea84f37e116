cd "$(dirname "$0")/.."
mkdir -p gpurun_out/n35
export HHC_BENCH_ALLOW_SHORT=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 30 -c 1 -o gpurun_out/n35/prof_c3 -f python bench.py --config C3 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/n35/ncu_c3.log 2>&1; echo "ncu3=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex3d -s 20 -c 1 -o gpurun_out/n35/prof_c5 -f python bench.py --config C5 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/n35/ncu_c5.log 2>&1; echo "ncu5=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex1d -s 20 -c 1 -o gpurun_out/n35/prof_x1 -f python bench.py --config X1 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/n35/ncu_x1.log 2>&1; echo "ncux1=$?"
