mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v31.log 2>&1; echo build rc=$?
timeout 2400 python scripts/fuzz_big.py 1200 2000 > gpurun_out/fuzz_big_v31.log 2>&1; echo "fuzz_big 1200-2000 rc=$?"; tail -n 1 gpurun_out/fuzz_big_v31.log
timeout 2400 python scripts/fuzz_configs.py 360 600 > gpurun_out/fuzz_configs_v31.log 2>&1; echo "fuzz_configs 360-600 rc=$?"; tail -n 1 gpurun_out/fuzz_configs_v31.log
