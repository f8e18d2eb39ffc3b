#!/bin/bash
# parity (multirank incl. per-rank segment paths, kernel scope full size, parity) of z = current; A/B w vs z.
cd "$(dirname "$0")/.."
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_parity.py "tests/test_gpu_fullsize.py::test_kernel_scope_full_exact" -x -q > $O/r2y_pytest.log 2>&1; echo "pytest=$?" >> $O/r2y_pytest.log
for rep in 1 2; do for w in c3_bfs c2_sgemm c4_srad; do for v in w z; do
  DC=--no-data-centric
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 $DC --no-per-analysis 2>/dev/null | tail -1 > $O/r2y_${w}_${v}_$rep.json
done; done; done
for v in w z; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --rd-scope kernel --steps 5 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2y_c4_kernel_${v}.json
done
echo done
