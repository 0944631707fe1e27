# fused finalize (coded walks) vs the separate finalize launch, same box: step time per config
for cfg in 3 2 4; do for f in 0 1 0 1; do
TAHOE_FUSE_FINALIZE=$f timeout 600 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_ff.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_ff.json').read().strip().splitlines()[-1]); print('C$cfg fuse=$f', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"; done; done
