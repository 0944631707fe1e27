# robustness: fresh fuzz seeds (400-1200 shapes, 120-360 config subsets) and the GPU suite again
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v27.log 2>&1; echo build rc=$?
timeout 2400 python scripts/fuzz_big.py 400 1200 > gpurun_out/fuzz_big_v27.log 2>&1; echo "fuzz_big 400-1200 rc=$?"; tail -n 1 gpurun_out/fuzz_big_v27.log
timeout 2400 python scripts/fuzz_configs.py 120 360 > gpurun_out/fuzz_configs_v27.log 2>&1; echo "fuzz_configs 120-360 rc=$?"; tail -n 1 gpurun_out/fuzz_configs_v27.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_v27.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_v27.log
