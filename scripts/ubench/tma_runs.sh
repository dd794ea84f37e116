T=scripts/ubench/tma_test2
for a in "1 36 5 1 0 2 0" "1 36 5 3 0 2 0" "1 36 5 0 -1 2 0" "1 36 5 -4 0 2 0" "1 36 5 -3 0 2 0" "1 36 5 2 0 2 0" "1 36 5 0 0 -1 0" "1 36 5 -1 0 2 0"; do timeout 30 $T $a; done
