# e2e: ramped chunks for C2's 1M rows (TAHOE_HOST_RAMP=1) vs default; C4 bench at HEAD
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v14.log 2>&1; echo build rc=$?
for r in -1 1 -1 1; do
if [ $r = -1 ]; then unset TAHOE_HOST_RAMP; else export TAHOE_HOST_RAMP=$r; fi
timeout 600 python bench.py --config 2 --no-cpu > gpurun_out/bench2_v14.json 2> gpurun_out/bench2_v14.err; python -c "
import json; d=json.loads(open('gpurun_out/bench2_v14.json').read().strip().splitlines()[-1]); print('ramp $r', round(d['value']/1e6,2), round(d['e2e']['value']/1e6,1))"
done
unset TAHOE_HOST_RAMP
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v14.json 2> gpurun_out/bench4_v14.err; python -c "
import json; d=json.loads(open('gpurun_out/bench4_v14.json').read().strip().splitlines()[-1]); print('C4', round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], round(d['roofline']['frac'],3), round(d['roofline']['peak']))"
timeout 600 python bench.py --config 3 --no-cpu > gpurun_out/bench3_v14.json 2> gpurun_out/bench3_v14.err; python -c "
import json; d=json.loads(open('gpurun_out/bench3_v14.json').read().strip().splitlines()[-1]); print('C3', round(d['value']/1e6,2), d['ms_per_step'], round(d['e2e']['value']/1e6,1))"
