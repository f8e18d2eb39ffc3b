#!/bin/bash
# Profile evidence of ONE workload for the current build (run through gpurun):
#   TAG_launches_WL.csv          ncu launch list of one bench step (gpu__time_duration, cold-cache, serialised)
#   TAG_ncu_full_summary_WL.csv  per-kernel summary of `ncu --set full` over the step's main kernels
#                                (NCU_KERNELS regex; tools/ncu_summary.py)
#   TAG_scan_sass_WL.csv         SASS-level source page of the first k_scan launch (-lineinfo build)
#   profiles/ncu_traffic.json    DRAM bytes per launch of each kernel, stamped with the library
#                                source hash bench.py checks (tools/ncu_traffic.py)
# The .ncu-rep reports stay in /tmp on the box (they exceed gpurun's copy-back limit).
# Usage: tools/ncu_capture.sh TAG [WORKLOAD] [extra bench args]
TAG=${1:-latest}; WL=${2:-c4_srad}; shift 2 2>/dev/null
cd "$(dirname "$0")/.."
O=gpurun_out
R=/tmp/ncu_${TAG}_$WL
mkdir -p $O $R
timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $O/${TAG}_launches_${WL}.csv \
    python bench.py --workload $WL --profile-run --steps 1 --warmup 2 --no-cpu-baseline "$@" > /dev/null 2>&1
timeout 1200 ncu --profile-from-start off --set full --import-source on --clock-control none -o $R/full -f \
    -k regex:"${NCU_KERNELS:-k_scan|k_rd_seg|k_rd_tile|k_rg_scatter|k_rg_count}" \
    python bench.py --workload $WL --profile-run --steps 1 --warmup 2 --no-cpu-baseline "$@" > $O/${TAG}_ncu_full_${WL}.log 2>&1
python tools/ncu_summary.py $O/${TAG}_ncu_full_summary_${WL}.csv $R/full.ncu-rep
ncu -i $R/full.ncu-rep --page source --csv --print-source sass -k regex:k_scan 2>/dev/null | head -c 20000000 > $O/${TAG}_scan_sass_${WL}.csv
python tools/ncu_traffic.py $WL $O/${TAG}_ncu_full_summary_${WL}.csv "$TAG"
cp profiles/ncu_traffic.json $O/${TAG}_ncu_traffic.json
echo "capture $TAG $WL done"
