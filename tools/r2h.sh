cd "$(dirname "$0")/.."
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_multiprocess.py tests/test_gpu_multirank.py tests/test_gpu_domain.py tests/test_gpu_datacentric.py -q > $O/r2h_pytest.log 2>&1; echo "pytest=$?" >> $O/r2h_pytest.log
for w in c4_srad c3_bfs; do
for rep in 1 2; do for v in d e; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2h_${w}_${v}_$rep.json
done; done; done
