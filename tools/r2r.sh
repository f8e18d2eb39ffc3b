#!/bin/bash
# A/B (a = round start, n = current) on the bench configs, then the full GPU suite on n.
cd "$(dirname "$0")/.."
O=gpurun_out
for w in c4_srad c3_bfs c2_sgemm; do
for rep in 1 2; do for v in a n; do
  DC=--no-data-centric; [ $w = c4_srad ] && DC=
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 $DC --no-per-analysis 2>/dev/null | tail -1 > $O/r2r_${w}_${v}_$rep.json
done; done; done
for v in a n; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --rd-scope kernel --steps 5 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2r_c4_kernel_${v}.json
done
timeout 2700 python -m pytest tests -m gpu -q --durations=15 > $O/r2r_pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/r2r_pytest_gpu.log
echo done
