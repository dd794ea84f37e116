cd /root/repo
T4="8,4,4,32:0 8,4,4,32:256 8,4,8,32:256 8,4,8,32:512 8,4,16,32:512 8,4,8,64:256 8,4,8,64:512 8,8,8,64:512 4,4,16,64:256 4,4,8,64:512 8,2,16,64:256 16,4,8,32:256 16,4,8,32:512 12,4,8,64:512 8,4,32,32:256 8,4,32,32:512 4,2,32,64:512 6,4,16,64:256"
HHC_EXP_T=64 timeout 600 python scripts/exp_tiles.py C4 $T4 > gpurun_out/sweep3d_C4.log 2>&1; echo C4=$?
HHC_EXP_T=32 timeout 600 python scripts/exp_tiles.py C5 $T4 > gpurun_out/sweep3d_C5.log 2>&1; echo C5=$?
