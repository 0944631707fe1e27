#!/bin/bash
# ncu launch list + one full capture of the top kernel for the bench command (1 GPU)
TAG=${1:-r01}
KREGEX=${2:-k_sliced}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
echo "launches rc=$?"
ncu --set full --clock-control none --import-source on -k regex:$KREGEX -s 3 -c 1 -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_full_$TAG.log 2>&1
echo "ncu full rc=$?"
tail -2 gpurun_out/ncu_full_$TAG.log
