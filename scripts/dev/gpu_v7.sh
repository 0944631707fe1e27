# pre-pass probe rewrite (4 instructions per row-probe): GPU tests + C3/C2 bench + launch list C3
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v7.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v7.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_v7.log
for c in 3 2; do
timeout 600 python bench.py --config $c --no-cpu > gpurun_out/bench${c}_v7.json 2> gpurun_out/bench${c}_v7.err; echo "bench$c rc=$?"; cut -c1-200 gpurun_out/bench${c}_v7.json
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_sliced_codes|k_encode_rows|k_finalize" -c 6 --log-file gpurun_out/launches${c}_v7.csv \
    python bench.py --config $c --steps 2 --warmup 3 --no-cpu > gpurun_out/launches${c}_v7.log 2>&1; echo "launch list rc=$?"
done
