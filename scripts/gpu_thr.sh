cd "$(dirname "$0")/.."
HHC_EXP_T=256 timeout 600 python scripts/exp_tiles.py C2 32,12,512:384 32,12,512:448 32,12,512:320 24,16,512:448 32,12,512:384 2>&1 | sed 's/^/C2 /'
