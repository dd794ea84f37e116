cd "$(dirname "$0")/.."
mkdir -p gpurun_out/last
timeout 600 python bench.py > gpurun_out/last/bench_C2.json 2> gpurun_out/last/bench_C2.err; echo "benchC2=$?"; tail -1 gpurun_out/last/bench_C2.json | cut -c1-300
timeout 600 python bench.py --config X1 > gpurun_out/last/bench_X1.json 2> gpurun_out/last/bench_X1.err; echo "benchX1=$?"; tail -1 gpurun_out/last/bench_X1.json | cut -c1-300
