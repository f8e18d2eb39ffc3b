#!/bin/bash
# compute-sanitizer evidence (run through gpurun): memcheck, racecheck (shared
# memory hazards), synccheck (barrier misuse) on tools/sanitize_run.py.
# Usage: tools/sanitize.sh TAG
TAG=${1:-r2}
cd "$(dirname "$0")/.."
O=gpurun_out
export CADV_SCAN_CTAS=2   # a small scan grid: many steps per warp, faster under the tools
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 --target-processes all \
    python tools/sanitize_run.py > $O/${TAG}_sanitizer_${tool}.log 2>&1
  echo "rc=$?" >> $O/${TAG}_sanitizer_${tool}.log
done
