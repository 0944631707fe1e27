#!/bin/bash
# profiles for the rank-coded C2 path: launch list, full captures of both kernels, sanitizers
TAG=${1:-r01codes}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
echo "launches rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_sliced_codes -s 3 -c 1 -o gpurun_out/prof_slc_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_slc_$TAG.log 2>&1
echo "ncu slc rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_encode_rows -s 3 -c 1 -o gpurun_out/prof_enc_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_enc_$TAG.log 2>&1
echo "ncu enc rc=$?"
bash scripts/gpu_sanitize.sh
