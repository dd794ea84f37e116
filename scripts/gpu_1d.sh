cd "$(dirname "$0")/.."
mkdir -p gpurun_out/x1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "1d or tiny or small" > gpurun_out/x1/tests.log 2>&1; echo "tests=$?"; tail -3 gpurun_out/x1/tests.log
timeout 600 python bench.py --config X1 > gpurun_out/x1/bench_X1.json 2> gpurun_out/x1/bench_X1.err; echo "benchX1=$?"; tail -1 gpurun_out/x1/bench_X1.json | cut -c1-600; tail -3 gpurun_out/x1/bench_X1.err
HHC_EXP_T=256 timeout 600 python scripts/exp_tiles.py X1 64,2048:256 128,4096:256 32,1024:256 64,4096:256 128,2048:256 256,4096:256 2>&1 | sed 's/^/X1 /'
