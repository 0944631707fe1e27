mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v1.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v1.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_v1.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_v1.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench_v1.json 2> gpurun_out/bench_v1.err; echo "bench rc=$?"; cut -c1-300 gpurun_out/bench_v1.json
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v1.json 2> gpurun_out/bench4_v1.err; echo "bench4 rc=$?"; cut -c1-300 gpurun_out/bench4_v1.json
timeout 600 python bench.py --config 2 --no-cpu > gpurun_out/bench2_v1.json 2> gpurun_out/bench2_v1.err; echo "bench2 rc=$?"; cut -c1-300 gpurun_out/bench2_v1.json
