cd "$(dirname "$0")/.."
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_multiprocess.py tests/test_gpu_domain.py tests/test_gpu_parity.py tests/test_gpu_multirank.py -q > $O/r2g_pytest.log 2>&1; echo "pytest=$?" >> $O/r2g_pytest.log
for w in c4_srad c3_bfs; do
for rep in 1 2; do for v in a d n; do
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2g_${w}_${v}_$rep.json
done; done; done
for w in c4_srad c3_bfs; do
ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:k_scan -c 1 -o $O/r2g_scan_$w -f \
    python bench.py --workload $w --profile-run --steps 1 --warmup 1 --no-cpu-baseline > $O/r2g_ncu_$w.log 2>&1
done
