# replicated-lane pre-pass plan: GPU suite, C3/C2/C4 bench, pre-pass launch times, fuzz sweeps
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v13.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v13.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_v13.log
for c in 3 2 4; do
timeout 600 python bench.py --config $c --no-cpu > gpurun_out/bench${c}_v13.json 2> gpurun_out/bench${c}_v13.err; echo "bench$c rc=$?"; python -c "
import json; d=json.loads(open('gpurun_out/bench${c}_v13.json').read().strip().splitlines()[-1]); print(round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], round(d['roofline']['frac'],3), round(d['roofline']['peak']), round(d['e2e']['value']/1e6,1))"
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,sm__inst_executed.sum --clock-control none --csv -k regex:"k_encode_rows" -c 4 --log-file gpurun_out/launches3_v13.csv \
    python bench.py --config 3 --steps 2 --warmup 3 --no-cpu > gpurun_out/launches3_v13.log 2>&1; echo "launch list rc=$?"
timeout 1800 python scripts/fuzz_big.py 0 400 > gpurun_out/fuzz_big_v13.log 2>&1; echo "fuzz_big rc=$?"; tail -n 1 gpurun_out/fuzz_big_v13.log
timeout 1200 python scripts/fuzz_configs.py 0 120 > gpurun_out/fuzz_configs_v13.log 2>&1; echo "fuzz_configs rc=$?"; tail -n 1 gpurun_out/fuzz_configs_v13.log
