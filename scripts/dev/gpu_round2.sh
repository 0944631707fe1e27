#!/bin/bash
# round check: GPU tests, default bench (C2), C4 bench + its launch list + ncu captures (wide codes)
TAG=${1:-r01w}
mkdir -p gpurun_out
timeout 1100 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 > gpurun_out/bench4_$TAG.json 2> gpurun_out/bench4_$TAG.err; echo "bench4 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches4_$TAG.csv python bench.py --config 4 --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sliced_codes8|k_encode_rows8" -s 6 -c 2 -o gpurun_out/prof4_$TAG python bench.py --config 4 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu4_$TAG.log 2>&1; echo "ncu rc=$?"
