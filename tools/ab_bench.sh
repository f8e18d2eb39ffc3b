#!/bin/bash
# A/B timing of library builds: tools/ab_bench.sh VARIANT... (libcadv_<v>.so in the package dir)
cd "$(dirname "$0")/.."
for rep in 1 2; do
  for v in "$@"; do
    CADV_LIB=$PWD/paper_conf_cgo_shensll18_b200/libcadv_$v.so timeout 300 python bench.py --steps 10 --warmup 3 \
      --no-cpu-baseline --e2e-steps 0 --no-data-centric 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); k=d['kernels']
print('$v', round(d['value']/1e9,2), d['ms_per_step'], ' '.join(f'{n}={v[\"ms_per_step\"]:.3f}' for n,v in k.items() if v['ms_per_step']>0.05))"
  done
done
