# A/B: staged slice partials of the u16 coded walk in swizzled slots (part_slot) vs plain; parity
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v19.log 2>&1; echo build rc=$?
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_p0.so -DTAHOE_PART_SWZ=0 >> gpurun_out/build_v19.log 2>&1
for lib in cur p0 cur p0; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
for c in 3 2; do
timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_p.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_p.json').read().strip().splitlines()[-1]); print('$lib C$c', round(d['value']/1e6,2), round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4))
"
done; done
unset TAHOE_LIB_AB
rm -f paper_conf_eurosys_xiedlll21_b200/libtahoe_p0.so
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/pytest_v19.log 2>&1; echo "pytest parity+fullsize rc=$?"; tail -1 gpurun_out/pytest_v19.log
