cd "$(dirname "$0")/.."
O=gpurun_out
timeout 2000 python -m pytest tests -m gpu -q --durations=20 > $O/r2c_pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/r2c_pytest_gpu.log
for w in c4_srad c3_bfs c2_sgemm; do
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/r2c_bench_$w.json 2> $O/r2c_bench_$w.log
done
