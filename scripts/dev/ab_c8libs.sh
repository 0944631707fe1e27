# C4 wide-code walk: A/B of in-tree builds (ring depth x warps), same box
for lib in cur "$@" cur; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_k4.json 2>gpurun_out/bench_k4.err
python -c "
import json
d=json.loads(open('gpurun_out/bench_k4.json').read().strip().splitlines()[-1]); print('$lib', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3), d['config'].get('n_slices', d['config'].get('slices')))
" || tail -3 gpurun_out/bench_k4.err
done
