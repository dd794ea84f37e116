cd "$(dirname "$0")/.."
mkdir -p gpurun_out
export HHC_BENCH_ALLOW_SHORT=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hex3d -s 40 -c 1 -o gpurun_out/prof_c4b -f python bench.py --config C4 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_c4b.log 2>&1; echo "ncu4=$?"
