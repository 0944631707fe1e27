#!/bin/bash
# end-of-round measurement: GPU tests, smoke, default bench (C2) + its launch list + ncu of the
# dominant kernel and the pre-pass, C4 bench, C3 / C5 bench lines, reference arm
TAG=${1:-r01f}
mkdir -p gpurun_out
timeout 1100 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_$TAG.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err; echo "ref rc=$?"
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 > gpurun_out/bench4_$TAG.json 2> gpurun_out/bench4_$TAG.err; echo "bench4 rc=$?"
timeout 600 python bench.py --config 3 --steps 10 --warmup 3 > gpurun_out/bench3_$TAG.json 2> gpurun_out/bench3_$TAG.err; echo "bench3 rc=$?"
timeout 900 python bench.py --config 5 --rows 1000000 --steps 3 --warmup 3 > gpurun_out/bench5_$TAG.json 2> gpurun_out/bench5_$TAG.err; echo "bench5 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sliced_codes|k_encode_rows_banks" -s 6 -c 2 -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_$TAG.log 2>&1; echo "ncu rc=$?"
