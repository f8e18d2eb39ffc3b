#!/bin/bash
# A/B of library builds (libcadv_<v>.so) on C4 and C3 + parity of the current build.
# Usage: tools/r2n.sh TAG VARIANT...
TAG=$1; shift
cd "$(dirname "$0")/.."
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_datacentric.py tests/test_gpu_domain.py -x -q > $O/${TAG}_pytest.log 2>&1; echo "pytest=$?" >> $O/${TAG}_pytest.log
for w in c4_srad c3_bfs; do
for rep in 1 2; do for v in "$@"; do
  DC=--no-data-centric; [ $w = c4_srad ] && DC=
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 $DC --no-per-analysis 2>/dev/null | tail -1 > $O/${TAG}_${w}_${v}_$rep.json
done; done; done
# source-level profile of the segment kernel (current build)
timeout 600 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:"k_rd_seg|k_rg_scatter" -c 2 \
  -o /tmp/${TAG}_seg -f python bench.py --profile-run --steps 1 --warmup 2 --no-cpu-baseline > $O/${TAG}_ncu_seg.log 2>&1
python tools/ncu_summary.py $O/${TAG}_ncu_seg_summary.csv /tmp/${TAG}_seg.ncu-rep >> $O/${TAG}_ncu_seg.log 2>&1
ncu -i /tmp/${TAG}_seg.ncu-rep --page source --csv --print-source sass -k regex:k_rd_seg 2>/dev/null > $O/${TAG}_seg_sass.csv
echo done
