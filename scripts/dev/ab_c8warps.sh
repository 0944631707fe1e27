for lib in w256 w320 cur w256 w320 cur; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_w.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_w.json').read().strip().splitlines()[-1]); print('$lib', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"
done
