cd "$(dirname "$0")/.."
mkdir -p gpurun_out
HHC_BENCH_ALLOW_SHORT=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:hex2d -s 60 -c 1 -o gpurun_out/prof_c2b -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS} > gpurun_out/ncu.log 2>&1; echo "ncu=$?"
