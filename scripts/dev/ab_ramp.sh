for cfg in 3; do
for r in 0 1 0 1; do
TAHOE_HOST_RAMP=$r timeout 900 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_rp.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_rp.json').read().strip().splitlines()[-1]); print('cfg $cfg ramp $r', round(d['value']/1e6,1), round(d['e2e']['value']/1e6,1))
"
done; done
python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "host" -p no:cacheprovider 2>&1 | tail -1
