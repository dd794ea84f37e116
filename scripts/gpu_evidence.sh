#!/bin/bash
# Round evidence on the current build: GPU suite + smoke, bench lines (default = C3, then the other
# BASELINE configs and the extensions), the ncu launch list of one C3 bench step and `--set full`
# captures of the dominant kernels of C3 (K1) and C4 (K2).
cd "$(dirname "$0")/.."
O=${OUT:-ev}
OUT=$O bash scripts/gpu.sh tests
OUT=$O bash scripts/gpu.sh bench C3 C2 C4 C5 C1 X1 X2 W1
OUT=$O bash scripts/gpu.sh launches C3
OUT=$O KREGEX=hex2d SKIP=20 bash scripts/gpu.sh ncu C3
OUT=$O KREGEX=hex3d SKIP=30 bash scripts/gpu.sh ncu C4
