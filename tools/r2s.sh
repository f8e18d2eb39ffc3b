#!/bin/bash
# scan split sweep (C4, C3), source-level profile of k_rd_seg and of C3's k_scan, C2 launch list.
cd "$(dirname "$0")/.."
O=gpurun_out
for w in c4_srad c3_bfs; do for sp in 0 2 3 6; do
  CADV_SCAN_SPLIT=$sp timeout 300 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 \
     --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2s_${w}_split$sp.json
done; done
timeout 600 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:"k_rd_seg|k_scan" -c 2 \
  -o /tmp/r2s_c4 -f python bench.py --profile-run --steps 1 --warmup 2 --no-cpu-baseline > $O/r2s_ncu_c4.log 2>&1
python tools/ncu_summary.py $O/r2s_ncu_c4_summary.csv /tmp/r2s_c4.ncu-rep >> $O/r2s_ncu_c4.log 2>&1
ncu -i /tmp/r2s_c4.ncu-rep --page source --csv --print-source sass -k regex:k_rd_seg 2>/dev/null > $O/r2s_seg_sass.csv
timeout 600 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:"k_scan|k_rd_tile" -c 2 \
  -o /tmp/r2s_c3 -f python bench.py --workload c3_bfs --profile-run --steps 1 --warmup 2 --no-cpu-baseline > $O/r2s_ncu_c3.log 2>&1
python tools/ncu_summary.py $O/r2s_ncu_c3_summary.csv /tmp/r2s_c3.ncu-rep >> $O/r2s_ncu_c3.log 2>&1
ncu -i /tmp/r2s_c3.ncu-rep --page source --csv --print-source sass -k regex:k_scan 2>/dev/null > $O/r2s_c3_scan_sass.csv
timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $O/r2s_launches_c2_sgemm.csv python bench.py --workload c2_sgemm --profile-run --steps 1 --warmup 2 --no-cpu-baseline > /dev/null 2>&1
echo done
