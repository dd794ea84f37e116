#!/bin/bash
cd "$(dirname "$0")/.."
OUT=r9 PYTEST_K="hexdist" bash scripts/gpu.sh tests
OUT=r9 KREGEX=hex2d SKIP=20 bash scripts/gpu.sh ncu C3
mkdir -p gpurun_out/model
timeout 900 python scripts/slab_tiles.py --config C5 --gpus 8 --budget 600 --out gpurun_out/model/slab_C5.json > gpurun_out/model/slab_C5.log 2>&1; echo "slab C5 $?"; tail -2 gpurun_out/model/slab_C5.log
timeout 900 python scripts/slab_tiles.py --config C3 --gpus 2 4 8 --budget 500 --out gpurun_out/model/slab_C3.json > gpurun_out/model/slab_C3.log 2>&1; echo "slab C3 $?"; tail -3 gpurun_out/model/slab_C3.log
timeout 900 python scripts/slab_tiles.py --config C4 --gpus 2 4 8 --budget 500 --out gpurun_out/model/slab_C4.json > gpurun_out/model/slab_C4.log 2>&1; echo "slab C4 $?"; tail -3 gpurun_out/model/slab_C4.log
SPACE=near bash scripts/gpu_model.sh sweep C3 900
