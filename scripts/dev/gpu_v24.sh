# C4 pre-pass: first bisection level loaded once per row group; wide/fuzz tests, C4 bench, pre-pass time
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v24.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests/test_gpu_wide.py tests/test_gpu_fuzz.py -x -q > gpurun_out/pytest_v24.log 2>&1; echo "pytest wide+fuzz rc=$?"; tail -1 gpurun_out/pytest_v24.log
for i in 1 2; do
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v24.json 2> gpurun_out/bench4_v24.err; python -c "
import json; d=json.loads(open('gpurun_out/bench4_v24.json').read().strip().splitlines()[-1]); print('C4', round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], round(d['roofline']['frac'],3))"
done
timeout 600 ncu --metrics gpu__time_duration.sum,sm__inst_executed.sum --clock-control none --csv -k regex:"k_encode_rows8" -c 2 --log-file gpurun_out/launches4_v24.csv \
    python bench.py --config 4 --steps 2 --warmup 3 --no-cpu > gpurun_out/launches4_v24.log 2>&1; echo "launch list rc=$?"; grep -o '"gpu__time_duration.sum","[a-z]*","[0-9,]*"' gpurun_out/launches4_v24.csv | head -3
