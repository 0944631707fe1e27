# A/B after the pre-pass loop-order + batched finalize change: GPU tests, benches, launch lists
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v2.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v2.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_v2.log
for c in 3 2 4; do
timeout 600 python bench.py --config $c --no-cpu > gpurun_out/bench${c}_v2.json 2> gpurun_out/bench${c}_v2.err; echo "bench$c rc=$?"; cut -c1-250 gpurun_out/bench${c}_v2.json
done
for c in 3 2 4; do
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches${c}_v2.csv \
    python bench.py --config $c --steps 3 --warmup 3 --no-cpu > gpurun_out/launches${c}_v2.log 2>&1; echo "launch list C$c rc=$?"
done
