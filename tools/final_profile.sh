#!/bin/bash
# Round-end evidence on one B200 (run through gpurun): GPU tests, the default
# bench line, the reference arm, the ncu launch list of one bench step and a
# `--set full` summary of every kernel of one step.  Usage: tools/final_profile.sh TAG
TAG=${1:-latest}
cd "$(dirname "$0")/.."
O=gpurun_out
make -j4 all > /dev/null 2>&1
python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/${TAG}_pytest_gpu.log
python bench.py > $O/${TAG}_bench.log 2>&1; echo "bench=$?" >> $O/${TAG}_bench.log
python bench.py --impl reference --steps 2 --warmup 1 > $O/${TAG}_reference.log 2>&1; echo "ref=$?" >> $O/${TAG}_reference.log
# launch list of one step (warm-up step skipped): serialised, cold-cache times
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${TAG}_launches.csv \
    python bench.py --profile-run --steps 1 --warmup 2 > /dev/null 2>&1
# --set full over the launches of the last step
ncu --profile-from-start off --set full --clock-control none -o $O/${TAG}_full python bench.py --profile-run --steps 1 --warmup 2 > $O/${TAG}_ncu_full.log 2>&1
python tools/ncu_summary.py $O/${TAG}_ncu_full_summary.csv $O/${TAG}_full.ncu-rep > /dev/null 2>&1
echo done
