cd "$(dirname "$0")/.."
mkdir -p gpurun_out
T4="10,8,8,64:512 8,16,4,64:256 8,16,4,64:512 8,16,8,64:512 8,24,4,64:256 8,24,4,64:512 10,16,4,64:512 6,16,8,64:512 8,12,8,64:512 12,12,4,64:512 8,16,4,32:256 8,32,4,32:256 8,32,2,64:256 6,24,4,64:512 8,16,2,128:512 8,8,16,32:512"
HHC_EXP_T=64 timeout 900 python scripts/exp_tiles.py C4 $T4 > gpurun_out/sweep3d_wide_C4.log 2>&1; echo C4=$?
T5="8,6,8,64:256 8,6,8,64:512 8,16,4,64:256 8,16,4,64:512 8,12,4,64:512 6,16,4,64:512 8,24,2,64:256 8,16,8,32:512 8,16,2,128:512"
HHC_EXP_T=32 timeout 900 python scripts/exp_tiles.py C5 $T5 > gpurun_out/sweep3d_wide_C5.log 2>&1; echo C5=$?
cat gpurun_out/sweep3d_wide_C4.log gpurun_out/sweep3d_wide_C5.log
