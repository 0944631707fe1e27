# A/B (C4): ring depth 5 tiles with two-row units (bigger slices, fewer of them) at 16 / 18 warps
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v26.log 2>&1; echo build rc=$?
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_r5w16.so -DTAHOE_CODE8_RING=5 -DTAHOE_CODE8_THREADS=512 >> gpurun_out/build_v26.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_r5w18.so -DTAHOE_CODE8_RING=5 -DTAHOE_CODE8_THREADS=576 >> gpurun_out/build_v26.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_r7w24.so -DTAHOE_CODE8_RING=7 -DTAHOE_CODE8_THREADS=768 >> gpurun_out/build_v26.log 2>&1
for lib in cur r5w16 r5w18 r7w24 cur r5w16 r5w18 r7w24; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_r.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_r.json').read().strip().splitlines()[-1]); print('$lib', round(d['value']/1e6,2), round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4), d['config'].get('n_slices'))
"
done
unset TAHOE_LIB_AB
rm -f paper_conf_eurosys_xiedlll21_b200/libtahoe_r*.so
