mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v30.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_v30.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_v30.log
timeout 600 python bench.py --config 2 > gpurun_out/bench2_v30.json 2> gpurun_out/bench2_v30.err; python -c "
import json; d=json.loads(open('gpurun_out/bench2_v30.json').read().strip().splitlines()[-1]); print('C2', round(d['value']/1e6,1), 'e2e', round(d['e2e']['value']/1e6,1), d['parity'])"
