# C4 pre-pass: TMA-staged rows vs rows through L1 (same box), step and walk time
for t in 1 0 1 0; do
TAHOE_CODE8_TMA=$t timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_k4.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_k4.json').read().strip().splitlines()[-1]); print('tma=$t', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3))
"; done
