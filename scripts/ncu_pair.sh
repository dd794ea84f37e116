cd "$(dirname "$0")/.."
mkdir -p gpurun_out
export HHC_BENCH_ALLOW_SHORT=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 60 -c 1 -o gpurun_out/prof_c2d -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_c2d.log 2>&1; echo "ncu2=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex3d -s 40 -c 1 -o gpurun_out/prof_c4d -f python bench.py --config C4 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_c4d.log 2>&1; echo "ncu4=$?"
