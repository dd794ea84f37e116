cd "$(dirname "$0")/.."
export CUDA_LAUNCH_BLOCKING=1 HHC_NO_GRAPH=1
for v in "HHC_NO_TMA=1" "HHC_DBG=48" "HHC_DBG=32" "HHC_DBG=16" "HHC_DBG=0"; do
  echo "== $v"; env $v timeout 120 python scripts/dbg3d.py 20,22,40 4,2,3,32 7 2>&1 | tail -2
done
echo "== sanitizer"
timeout 300 compute-sanitizer --print-limit 5 python scripts/dbg3d.py 20,22,40 4,2,3,32 7 2>&1 | head -40
