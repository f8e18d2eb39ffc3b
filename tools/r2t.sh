#!/bin/bash
# parity of the packed segment-list tiles (p), tail-size sweep, A/B n vs p on C3 / C4 / data-centric.
cd "$(dirname "$0")/.."
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_datacentric.py tests/test_gpu_fullsize.py -k "not kernel_scope and not backprop" -x -q > $O/r2t_pytest.log 2>&1; echo "pytest=$?" >> $O/r2t_pytest.log
for w in c3_bfs c4_srad; do for tq in 2 4 8; do
  CADV_SCAN_TAIL=$tq timeout 300 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 \
     --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2t_${w}_tail$tq.json
done; done
for v in n o p; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload c3_bfs --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2t_c3_bfs_$v.json
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-per-analysis 2>/dev/null | tail -1 > $O/r2t_c4_srad_$v.json
done
echo done
