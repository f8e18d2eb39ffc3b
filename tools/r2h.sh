#!/bin/bash
# C3 scan chunks per warp: 6 (default below 2^28 records) vs 8 vs 12
cd "$(dirname "$0")/.."
O=gpurun_out
for rep in 1 2; do for sp in 0 8 12; do
  CADV_SCAN_SPLIT=$sp timeout 300 python bench.py --workload c3_bfs --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 \
     --no-data-centric --no-per-analysis 2>/dev/null | tail -1 > $O/r2h_c3_bfs_split${sp}_$rep.json
done; done
echo done
