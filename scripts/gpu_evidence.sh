#!/bin/bash
# Round evidence on the current build: GPU suite + smoke, bench lines (default = C3, then C2 C4 C5),
# the ncu launch list of one C3 bench step and one `--set full` capture of its dominant kernel.
cd "$(dirname "$0")/.."
O=${OUT:-ev}
OUT=$O bash scripts/gpu.sh tests
OUT=$O bash scripts/gpu.sh bench C3 C2 C4 C5
OUT=$O bash scripts/gpu.sh launches C3
OUT=$O KREGEX=hex2d SKIP=20 bash scripts/gpu.sh ncu C3
