# two compute streams in predict_host (e2e), fuzz sweeps after the slot assignment, C3 bench with
# the oracle leg, C5 at its full 10M rows
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v5.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v5.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_v5.log
timeout 900 python bench.py > gpurun_out/bench3_v5.json 2> gpurun_out/bench3_v5.err; echo "bench3 rc=$?"; cut -c1-200 gpurun_out/bench3_v5.json
TAHOE_HOST_STREAMS=1 timeout 900 python bench.py --no-cpu > gpurun_out/bench3_v5_1s.json 2> gpurun_out/bench3_v5_1s.err; echo "bench3 1-stream rc=$?"
timeout 1800 python scripts/fuzz_big.py 0 400 > gpurun_out/fuzz_big_v5.log 2>&1; echo "fuzz_big rc=$?"; tail -n 2 gpurun_out/fuzz_big_v5.log
timeout 1200 python scripts/fuzz_configs.py 0 120 > gpurun_out/fuzz_configs_v5.log 2>&1; echo "fuzz_configs rc=$?"; tail -n 2 gpurun_out/fuzz_configs_v5.log
timeout 1500 python bench.py --config 5 --steps 3 --warmup 3 > gpurun_out/bench5_v5.json 2> gpurun_out/bench5_v5.err; echo "bench5 rc=$?"; cut -c1-300 gpurun_out/bench5_v5.json
