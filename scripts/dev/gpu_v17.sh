# HEAD validation: GPU suite, smoke, default bench (C3 with the path sector efficiency)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v17.log 2>&1; echo build rc=$?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v17.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_v17.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_v17.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench_v17.json 2> gpurun_out/bench_v17.err; echo "bench rc=$?"; cut -c1-200 gpurun_out/bench_v17.json
