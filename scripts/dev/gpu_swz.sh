#!/bin/bash
# A/B of the code-row swizzle: GPU tests, C3 / C2 bench lines
TAG=${1:-swz}
mkdir -p gpurun_out
timeout 1100 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_$TAG.log
timeout 600 python bench.py --config 3 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench3_$TAG.json 2> gpurun_out/bench3_$TAG.err; echo "bench3 rc=$?"
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
for f in bench3 bench; do python -c "
import json; d=json.loads(open('gpurun_out/${f}_$TAG.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$f', d['value']/1e6, d['ms_per_step'], r['kernel_ms'], r['frac'])"; done
