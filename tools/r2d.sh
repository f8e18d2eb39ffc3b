cd "$(dirname "$0")/.."
O=gpurun_out
for w in c3_bfs c4_srad; do
ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:k_scan -c 1 -o $O/r2d_scan_$w -f \
    python bench.py --workload $w --profile-run --steps 1 --warmup 1 --no-cpu-baseline > $O/r2d_ncu_$w.log 2>&1
done
