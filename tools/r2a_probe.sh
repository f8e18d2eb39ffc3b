set -x
free -g; nproc; lscpu | head -20; nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv
df -h /tmp /root | head
for w in c3_bfs c2_sgemm; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --no-data-centric > gpurun_out/r2a_bench_$w.json 2> gpurun_out/r2a_bench_$w.log; done
timeout 600 python bench.py --workload c4_srad --rd-scope kernel --steps 10 --warmup 3 --no-cpu-baseline --no-data-centric > gpurun_out/r2a_bench_kernel.json 2> gpurun_out/r2a_bench_kernel.log
timeout 600 python bench.py --workload c4_backprop --steps 10 --warmup 3 --no-cpu-baseline --no-data-centric > gpurun_out/r2a_bench_bp.json 2> gpurun_out/r2a_bench_bp.log
