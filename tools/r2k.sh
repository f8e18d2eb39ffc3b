cd "$(dirname "$0")/.."
bash tools/ncu_capture.sh r2k c4_srad > gpurun_out/r2k_cap_c4.log 2>&1
bash tools/ncu_capture.sh r2k c3_bfs > gpurun_out/r2k_cap_c3.log 2>&1
for sp in 0 8; do
  CADV_SCAN_SPLIT=$sp timeout 300 python bench.py --workload c2_sgemm --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > gpurun_out/r2k_c2_split$sp.json
done
