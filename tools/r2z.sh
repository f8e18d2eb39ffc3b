#!/bin/bash
cd "$(dirname "$0")/.."
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_parity.py tests/test_gpu_datacentric.py -x -q > $O/r2z_pytest.log 2>&1; echo "pytest=$?" >> $O/r2z_pytest.log
for rep in 1 2; do for w in c2_sgemm c3_bfs c4_srad; do for v in w zz; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2z_${w}_${v}_$rep.json
done; done; done
echo done
