#!/bin/bash
# Parity of the current build + A/B of library builds (libcadv_<v>.so; v:ENV=VAL sets an env var).
# Usage: tools/r2o.sh TAG "WORKLOADS" VARIANT...
TAG=$1; WLS=$2; shift 2
cd "$(dirname "$0")/.."
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_datacentric.py tests/test_gpu_domain.py tests/test_gpu_multirank.py -x -q > $O/${TAG}_pytest.log 2>&1; echo "pytest=$?" >> $O/${TAG}_pytest.log
for w in $WLS; do
for rep in 1 2; do for vv in "$@"; do
  v=${vv%%:*}; ev=; [ "$vv" != "$v" ] && ev=${vv#*:}
  DC=--no-data-centric; [ $w = c4_srad ] && DC=
  env $ev CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --workload $w --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 $DC --no-per-analysis 2>/dev/null | tail -1 > $O/${TAG}_${w}_${vv//[:=]/_}_$rep.json
done; done; done
echo done
