cd "$(dirname "$0")/.."
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py tests/test_gpu_domain.py tests/test_gpu_datacentric.py tests/test_gpu_c5.py -k "not full" -q -x > $O/r2j_pytest.log 2>&1; echo "pytest=$?" >> $O/r2j_pytest.log
for w in c4_srad c3_bfs c2_sgemm; do
for rep in 1 2; do for v in e f; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2j_${w}_${v}_$rep.json
done; done; done
for sp in 1 2 8; do
  CADV_SCAN_SPLIT=$sp timeout 300 python bench.py --workload c3_bfs --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2j_c3_bfs_split$sp.json
  CADV_SCAN_SPLIT=$sp timeout 300 python bench.py --workload c4_srad --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2j_c4_srad_split$sp.json
done
