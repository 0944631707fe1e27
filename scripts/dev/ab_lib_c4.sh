# same-box A/B: libtahoe_ab.so (ticket-protocol k_sliced_codes8) vs libtahoe.so (producer warp)
for lib in ab cur ab cur; do
if [ $lib = ab ]; then export TAHOE_LIB_AB=libtahoe_ab.so; else unset TAHOE_LIB_AB; fi
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_ab4.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_ab4.json').read().strip().splitlines()[-1]); print('$lib', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"
done
