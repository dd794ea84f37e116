cd "$(dirname "$0")/.."
HHC_EXP_T=256 timeout 600 python scripts/exp_tiles.py C2 32,12,512:384 32,14,512:384 34,12,512:384 30,16,512:384 32,13,512:384 28,18,512:384 2>&1 | sed 's/^/C2 /'
HHC_EXP_T=64 timeout 600 python scripts/exp_tiles.py C5 8,6,8,64:256 12,9,8,32:256 12,9,8,32:512 10,8,8,32:256 2>&1 | sed 's/^/C5 /'
HHC_EXP_T=128 timeout 600 python scripts/exp_tiles.py C4 8,8,16,64:512 10,7,10,32:0 10,8,16,32:512 2>&1 | sed 's/^/C4 /'
