#!/bin/bash
cd "$(dirname "$0")/.."
cp paper_conf_cgo_shensll18_b200/libcadv_g2.so paper_conf_cgo_shensll18_b200/libcadv.so
bash tools/r2o.sh r2q "c4_srad" a g2 h i j
bash tools/r2o.sh r2q3 "c3_bfs" a g2 > /dev/null 2>&1
echo done
