# A/B of the code-slot assignment (R10): GPU tests, C3/C2 bench, ncu of the C3 walk
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v3.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v3.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_v3.log
for c in 3 2 4; do
timeout 600 python bench.py --config $c --no-cpu > gpurun_out/bench${c}_v3.json 2> gpurun_out/bench${c}_v3.err; echo "bench$c rc=$?"; cut -c1-250 gpurun_out/bench${c}_v3.json
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_sliced_codes$" -s 3 -c 1 \
      -o gpurun_out/prof3_v3 python bench.py --config 3 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu3_v3.log 2>&1
echo "ncu C3 rc=$?"
