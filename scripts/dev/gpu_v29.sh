# e2e A/B on C2 (1M rows): ramped chunks vs eight equal chunks, 20 e2e steps each, alternating
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v29.log 2>&1; echo build rc=$?
for r in 0 1 0 1 0 1; do
TAHOE_HOST_RAMP=$r timeout 600 python bench.py --config 2 --no-cpu > gpurun_out/bench2_v29.json 2> gpurun_out/bench2_v29.err; python -c "
import json; d=json.loads(open('gpurun_out/bench2_v29.json').read().strip().splitlines()[-1]); print('ramp $r', round(d['e2e']['value']/1e6,1))"
done
