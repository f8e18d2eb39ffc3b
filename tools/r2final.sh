#!/bin/bash
# Evidence of the current build (run through gpurun): parity gate, A/B vs the
# round start, ncu capture (stamped traffic) of C4 then the bench lines that read
# it, every config, the oracle arm, C3 capture, the full GPU suite.
TAG=${1:-r2u}
cd "$(dirname "$0")/.."
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_datacentric.py tests/test_gpu_domain.py -x -q > $O/${TAG}_pytest_gate.log 2>&1
rc=$?; echo "pytest=$rc" >> $O/${TAG}_pytest_gate.log
[ $rc -ne 0 ] && exit 1
for w in c4_srad c3_bfs c2_sgemm; do for v in a f; do
  DC=--no-data-centric; [ $w = c4_srad ] && DC=
  CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 $DC --no-per-analysis 2>/dev/null | tail -1 > $O/${TAG}_ab_${w}_${v}.json
done; done
bash tools/ncu_capture.sh $TAG c4_srad > $O/${TAG}_cap_c4.log 2>&1
timeout 900 python bench.py > $O/${TAG}_bench.log 2>&1; echo "bench=$?" >> $O/${TAG}_bench.log
for w in c3_bfs c2_sgemm c4_backprop c5_mixed; do
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/${TAG}_bench_$w.log 2>&1; echo "bench=$?" >> $O/${TAG}_bench_$w.log
done
timeout 600 python bench.py --rd-scope kernel --steps 10 --warmup 3 --no-data-centric > $O/${TAG}_bench_c4_kernel.log 2>&1; echo "bench=$?" >> $O/${TAG}_bench_c4_kernel.log
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $O/${TAG}_reference.log 2>&1; echo "ref=$?" >> $O/${TAG}_reference.log
bash tools/ncu_capture.sh ${TAG} c3_bfs > $O/${TAG}_cap_c3.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke=$?" >> $O/${TAG}_smoke.log
timeout 2700 python -m pytest tests -m gpu -q --durations=15 > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/${TAG}_pytest_gpu.log
echo done
