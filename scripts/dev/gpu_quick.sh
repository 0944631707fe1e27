#!/bin/bash
# quick loop: GPU parity tests + timing diagnostic + short bench
TAG=${1:-q}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_gpu_$TAG.log
python scripts/diag_timing.py 2 2>&1 | grep -v '^{'
python scripts/diag_timing.py 3 1000000 2>&1 | grep -v '^{'
python scripts/diag_timing.py 4 200000 2>&1 | grep -v '^{'
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/bench_$TAG.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'kernel', d['roofline']['kernel_ms'], 'frac', d['roofline']['frac'], 'e2e', d['e2e']['value'], 'clocks', d['clocks'])"
tail -3 gpurun_out/bench_$TAG.err
