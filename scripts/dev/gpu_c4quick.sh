python -m pytest tests -m gpu -x -q -k "wide or codes8 or C4" 2>&1 | tail -2
for i in 1 2; do timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_k4.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_k4.json').read().strip().splitlines()[-1]); print('C4', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"; done
