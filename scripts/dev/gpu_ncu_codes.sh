#!/bin/bash
# ncu full captures of the coded pre-pass and the coded slice kernel on the bench command
TAG=${1:-codes}
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:k_encode_rows -s 3 -c 1 -o gpurun_out/prof_enc_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_enc_$TAG.log 2>&1
echo "ncu enc rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_sliced_codes -s 3 -c 1 -o gpurun_out/prof_slc_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_slc_$TAG.log 2>&1
echo "ncu slc rc=$?"
