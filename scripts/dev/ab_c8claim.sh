# C4 wide-code walk: tiles per claim x L2 prefetch distance (same box)
for cfg in "8 32" "16 32" "16 64" "32 64" "32 128" "8 0" "16 0" "8 32"; do set -- $cfg
TAHOE_CODE8_CLAIM=$1 TAHOE_CODE8_PREFETCH=$2 timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_k4.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_k4.json').read().strip().splitlines()[-1]); print('claim $1 pf $2', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3), (d.get('parity') or {}).get('mismatches'))
"
done
