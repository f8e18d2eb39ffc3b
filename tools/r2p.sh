#!/bin/bash
cd "$(dirname "$0")/.."
O=gpurun_out
bash tools/r2o.sh r2p "c4_srad" a g
timeout 600 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:"k_rd_seg" -c 1 \
  -o /tmp/r2p_seg -f python bench.py --profile-run --steps 1 --warmup 2 --no-cpu-baseline > $O/r2p_ncu_seg.log 2>&1
python tools/ncu_summary.py $O/r2p_ncu_seg_summary.csv /tmp/r2p_seg.ncu-rep >> $O/r2p_ncu_seg.log 2>&1
ncu -i /tmp/r2p_seg.ncu-rep --page source --csv --print-source sass -k regex:k_rd_seg 2>/dev/null > $O/r2p_seg_sass.csv
timeout 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:"k_scan" -c 1 \
  -o /tmp/r2p_dc -f python tools/dc_profile.py > $O/r2p_ncu_dc.log 2>&1
python tools/ncu_summary.py $O/r2p_ncu_dc_summary.csv /tmp/r2p_dc.ncu-rep >> $O/r2p_ncu_dc.log 2>&1
ncu -i /tmp/r2p_dc.ncu-rep --page source --csv --print-source sass -k regex:k_scan 2>/dev/null > $O/r2p_dc_sass.csv
echo done
