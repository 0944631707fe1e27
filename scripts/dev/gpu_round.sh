#!/bin/bash
# one call: bench (default flags), launch list of the bench command, full ncu captures of the
# dominant kernel and the row-coding pre-pass
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
cat gpurun_out/bench_$TAG.json
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
echo "launches rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_sliced_codes -s 3 -c 1 -o gpurun_out/prof_slc_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_slc_$TAG.log 2>&1
echo "ncu slc rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_encode_rows -s 3 -c 1 -o gpurun_out/prof_enc_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_enc_$TAG.log 2>&1
echo "ncu enc rc=$?"
