#!/bin/bash
# A/B r (e0989c3) vs s (speculative segment kernel) vs t (s + one-launch small scans); parity gate first.
cd "$(dirname "$0")/.."
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_datacentric.py tests/test_gpu_multirank.py -x -q > $O/r2v_pytest.log 2>&1; echo "pytest=$?" >> $O/r2v_pytest.log
for rep in 1 2; do for w in c4_srad c3_bfs c2_sgemm; do for v in r s t; do
  DC=--no-data-centric; [ $w = c4_srad ] && DC=
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 $DC --no-per-analysis 2>/dev/null | tail -1 > $O/r2v_${w}_${v}_$rep.json
done; done; done
timeout 600 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:"k_rd_seg" -c 1 \
  -o /tmp/r2v_seg -f python bench.py --profile-run --steps 1 --warmup 2 --no-cpu-baseline > $O/r2v_ncu_seg.log 2>&1
python tools/ncu_summary.py $O/r2v_ncu_seg_summary.csv /tmp/r2v_seg.ncu-rep >> $O/r2v_ncu_seg.log 2>&1
ncu -i /tmp/r2v_seg.ncu-rep --page source --csv --print-source sass -k regex:k_rd_seg 2>/dev/null > $O/r2v_seg_sass.csv
echo done
