#!/bin/bash
# rank-coded slices: parity tests, timing diagnostic, short bench
TAG=${1:-codes}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_parity_$TAG.log 2>&1; echo "parity rc=$?"
tail -15 gpurun_out/pytest_parity_$TAG.log
python scripts/diag_timing.py 2 2>&1 | grep -v '^{'
python scripts/diag_timing.py 3 1000000 2>&1 | grep -v '^{'
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
cat gpurun_out/bench_$TAG.json
tail -3 gpurun_out/bench_$TAG.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
echo "launches rc=$?"
