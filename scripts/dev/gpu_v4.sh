# slot_attr fix for the L2 pre-pass, 4-step exit test in walk_coded2: GPU tests + C3/C2 bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v4.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v4.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_v4.log
for c in 3 2; do
timeout 600 python bench.py --config $c --no-cpu > gpurun_out/bench${c}_v4.json 2> gpurun_out/bench${c}_v4.err; echo "bench$c rc=$?"; cut -c1-250 gpurun_out/bench${c}_v4.json
done
