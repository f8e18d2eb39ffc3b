#!/bin/bash
# k2 = f + merge-path counts carried with the items: kernel-scope parity (incl. full size), domain tests, A/B.
cd "$(dirname "$0")/.."
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_domain.py tests/test_gpu_multirank.py tests/test_gpu_datacentric.py \
  "tests/test_gpu_parity.py" "tests/test_gpu_fullsize.py::test_kernel_scope_full_exact" -x -q > $O/r2k2_pytest.log 2>&1; echo "pytest=$?" >> $O/r2k2_pytest.log
for rep in 1 2; do for v in f k2; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --rd-scope kernel --steps 5 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2k2_c4_kernel_${v}_$rep.json
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload c2_sgemm --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2k2_c2_sgemm_${v}_$rep.json
done; done
echo done
