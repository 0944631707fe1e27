# C4: split slot hoisted out of the unit loop; wide tests + C4 bench x2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v23.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests/test_gpu_wide.py tests/test_gpu_fuzz.py -x -q > gpurun_out/pytest_v23.log 2>&1; echo "pytest wide+fuzz rc=$?"; tail -1 gpurun_out/pytest_v23.log
for i in 1 2; do
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v23.json 2> gpurun_out/bench4_v23.err; python -c "
import json; d=json.loads(open('gpurun_out/bench4_v23.json').read().strip().splitlines()[-1]); print('C4', round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], round(d['roofline']['frac'],3))"
done
