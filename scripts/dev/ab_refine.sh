for cfg in 3 2; do
for it in 0 200 1000 3000; do
TAHOE_REFINE_ITERS=$it timeout 900 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_rf.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_rf.json').read().strip().splitlines()[-1]); print('cfg $cfg iters $it', round(d['value']/1e6,1), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3), d['config']['lockstep_eff_sim'], round(d['layout_s'],1))
"
done; done
