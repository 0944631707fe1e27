set -x
python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -m gpu -q -x -p no:cacheprovider > gpurun_out/gputest_d.log 2>&1; echo rc=$? >> gpurun_out/gputest_d.log
for cfg in 3 2; do
for r in 3 9 3 9; do
TAHOE_CODES_RING=$r python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu > gpurun_out/ring_${cfg}_${r}.json 2>/dev/null
python -c "
import json,sys
d=json.loads(open('gpurun_out/ring_${cfg}_${r}.json').read().strip().splitlines()[-1]); print('cfg $cfg ring $r', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"
done; done
tail -2 gpurun_out/gputest_d.log
