# A/B: exit test every 4 / 6 / 8 steps per chain in the u16 coded walk (C3, C2)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v15.log 2>&1; echo build rc=$?
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_e8.so -DTAHOE_CODED_EXIT=8 >> gpurun_out/build_v15.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_e6.so -DTAHOE_CODED_EXIT=6 >> gpurun_out/build_v15.log 2>&1
for lib in cur e6 e8 cur e6 e8; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
for c in 3 2; do
timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_e.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_e.json').read().strip().splitlines()[-1]); print('$lib C$c', round(d['value']/1e6,2), round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4))
"
done; done
unset TAHOE_LIB_AB
rm -f paper_conf_eurosys_xiedlll21_b200/libtahoe_e*.so
