# fuzz sweeps at HEAD (400 shapes + 120 config subsets, leaf ids and fingerprints from every strategy)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v18.log 2>&1; echo build rc=$?
timeout 1800 python scripts/fuzz_big.py 0 400 > gpurun_out/fuzz_big_v18.log 2>&1; echo "fuzz_big rc=$?"; tail -n 1 gpurun_out/fuzz_big_v18.log
timeout 1200 python scripts/fuzz_configs.py 0 120 > gpurun_out/fuzz_configs_v18.log 2>&1; echo "fuzz_configs rc=$?"; tail -n 1 gpurun_out/fuzz_configs_v18.log
