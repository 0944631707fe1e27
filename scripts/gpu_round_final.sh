#!/bin/bash
# End-of-round measurement on one B200: GPU tests, smoke, the default bench (C3) and its reference
# arm, the other configs' bench lines (C5 at its full 10M rows), then the profiles
# (scripts/gpu_profile_round.sh).  bash scripts/gpu_round_final.sh TAG
TAG=${1:-r02f}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1; echo "build rc=$?"
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err; echo "ref rc=$?"
timeout 600 python bench.py --config 2 > gpurun_out/bench2_$TAG.json 2> gpurun_out/bench2_$TAG.err; echo "bench2 rc=$?"
timeout 600 python bench.py --config 4 > gpurun_out/bench4_$TAG.json 2> gpurun_out/bench4_$TAG.err; echo "bench4 rc=$?"
timeout 1500 python bench.py --config 5 --steps 3 --warmup 3 > gpurun_out/bench5_$TAG.json 2> gpurun_out/bench5_$TAG.err; echo "bench5 rc=$?"
bash scripts/gpu_profile_round.sh $TAG
