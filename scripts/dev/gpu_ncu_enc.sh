#!/bin/bash
TAG=${1:-enc}
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:k_encode_rows -s 3 -c 1 -o gpurun_out/prof_enc_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_enc_$TAG.log 2>&1
echo "ncu enc rc=$?"
