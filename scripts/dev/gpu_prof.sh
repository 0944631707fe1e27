#!/bin/bash
TAG=${1:-r01}
mkdir -p gpurun_out
python scripts/diag_timing.py 2 > gpurun_out/diag_$TAG.txt 2>&1
python scripts/diag_timing.py 3 1000000 >> gpurun_out/diag_$TAG.txt 2>&1
python scripts/diag_timing.py 4 200000 >> gpurun_out/diag_$TAG.txt 2>&1
cat gpurun_out/diag_$TAG.txt | grep -v '^{'
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
echo "launches rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_sliced -s 3 -c 1 -o gpurun_out/prof_sliced_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_full_$TAG.log 2>&1
echo "ncu full rc=$?"
tail -3 gpurun_out/ncu_full_$TAG.log
