# C4 pre-pass with per-item group registers: wide-code tests, C4 bench, launch list
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v10.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests/test_gpu_wide.py -x -q > gpurun_out/pytest_v10.log 2>&1; echo "pytest wide rc=$?"; tail -2 gpurun_out/pytest_v10.log
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v10.json 2> gpurun_out/bench4_v10.err; echo "bench4 rc=$?"; cut -c1-200 gpurun_out/bench4_v10.json
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__inst_executed.sum --clock-control none --csv -k regex:"k_sliced_codes8|k_encode_rows8" -c 4 --log-file gpurun_out/launches4_v10.csv \
    python bench.py --config 4 --steps 2 --warmup 3 --no-cpu > gpurun_out/launches4_v10.log 2>&1; echo "launch list rc=$?"
