#!/bin/bash
cd "$(dirname "$0")/.."
for d in 0 32 16; do
  echo "dbg=$d $(HHC_DBG=$d python scripts/exp_compute_only.py 2 16384 192 32,12,512:384 2>&1 | tail -1)"
done
