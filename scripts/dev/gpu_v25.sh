# final HEAD validation: GPU suite + smoke + C4 bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v25.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_v25.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_v25.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_v25.log 2>&1; echo "smoke rc=$?"
timeout 600 python bench.py --config 4 > gpurun_out/bench4_v25.json 2> gpurun_out/bench4_v25.err; echo "bench4 rc=$?"; cut -c1-200 gpurun_out/bench4_v25.json
