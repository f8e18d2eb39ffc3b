#!/bin/bash
# Profile evidence of ONE workload for the current build (run through gpurun):
#   TAG_launches_WL.csv   ncu launch list of one bench step (gpu__time_duration, cold-cache, serialised)
#   TAG_full_WL.ncu-rep   `ncu --set full` of every launch of one step (source-mapped: -lineinfo build)
#   TAG_ncu_full_summary_WL.csv  per-kernel summary (tools/ncu_summary.py)
#   profiles/ncu_traffic.json    DRAM bytes per launch of each kernel, stamped with the
#                                library source hash bench.py checks (tools/ncu_traffic.py)
# Usage: tools/ncu_capture.sh TAG [WORKLOAD] [extra bench args]
TAG=${1:-latest}; WL=${2:-c4_srad}; shift 2 2>/dev/null
cd "$(dirname "$0")/.."
O=gpurun_out
mkdir -p $O
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $O/${TAG}_launches_${WL}.csv \
    python bench.py --workload $WL --profile-run --steps 1 --warmup 2 --no-cpu-baseline "$@" > /dev/null 2>&1
ncu --profile-from-start off --set full --import-source on --clock-control none -o $O/${TAG}_full_${WL} -f \
    python bench.py --workload $WL --profile-run --steps 1 --warmup 2 --no-cpu-baseline "$@" > $O/${TAG}_ncu_full_${WL}.log 2>&1
python tools/ncu_summary.py $O/${TAG}_ncu_full_summary_${WL}.csv $O/${TAG}_full_${WL}.ncu-rep
python tools/ncu_traffic.py $WL $O/${TAG}_ncu_full_summary_${WL}.csv "$TAG"
echo "capture $TAG $WL done"
