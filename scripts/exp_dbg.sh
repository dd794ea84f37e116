#!/bin/bash
# timing experiments with the HHC_DBG switches (results are wrong by design; timing only)
cd "$(dirname "$0")/.."
for d in 0 1 4 5 2 6; do
  echo "dbg=$d $(HHC_DBG=$d python scripts/exp_compute_only.py 2 8194 256 32,12,512:384 2>&1 | tail -1)"
done
