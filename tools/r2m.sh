#!/bin/bash
# Round-2 evidence of the current tree on one B200 (run through gpurun):
# default bench line, one line per other config, the oracle arm, the ncu
# launch list + --set full summary of C4 and C3.  Usage: tools/r2m.sh TAG
TAG=${1:-r2m}
cd "$(dirname "$0")/.."
O=gpurun_out
mkdir -p $O
timeout 600 python bench.py > $O/${TAG}_bench.log 2>&1; echo "bench=$?" >> $O/${TAG}_bench.log
for w in c3_bfs c2_sgemm c4_backprop c5_mixed; do
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/${TAG}_bench_$w.log 2>&1; echo "bench=$?" >> $O/${TAG}_bench_$w.log
done
timeout 600 python bench.py --rd-scope kernel --steps 10 --warmup 3 --no-data-centric > $O/${TAG}_bench_c4_kernel.log 2>&1; echo "bench=$?" >> $O/${TAG}_bench_c4_kernel.log
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $O/${TAG}_reference.log 2>&1; echo "ref=$?" >> $O/${TAG}_reference.log
bash tools/ncu_capture.sh $TAG c4_srad > $O/${TAG}_cap_c4.log 2>&1
bash tools/ncu_capture.sh $TAG c3_bfs > $O/${TAG}_cap_c3.log 2>&1
echo done
