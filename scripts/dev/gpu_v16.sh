# A/B (C4): exit test every 2 / 4 / 8 steps per chain of the two-row wide-code walk; 18 / 20 warps
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v16.log 2>&1; echo build rc=$?
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_x2.so -DTAHOE_CODE8_EXIT=2 >> gpurun_out/build_v16.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_x8.so -DTAHOE_CODE8_EXIT=8 >> gpurun_out/build_v16.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_w18.so -DTAHOE_CODE8_THREADS=576 >> gpurun_out/build_v16.log 2>&1
for lib in cur x2 x8 w18 cur x2 x8 w18; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_x.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_x.json').read().strip().splitlines()[-1]); print('$lib', round(d['value']/1e6,2), round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4))
"
done
unset TAHOE_LIB_AB
rm -f paper_conf_eurosys_xiedlll21_b200/libtahoe_x*.so paper_conf_eurosys_xiedlll21_b200/libtahoe_w18.so
