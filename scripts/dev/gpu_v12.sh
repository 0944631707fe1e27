# A/B: two-row wide-code units with 20 (default now) / 22 / 24 warps, and the old four-row units
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v12.log 2>&1; echo build rc=$?
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_w22.so -DTAHOE_CODE8_THREADS=704 >> gpurun_out/build_v12.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_w24.so -DTAHOE_CODE8_THREADS=768 >> gpurun_out/build_v12.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_u4.so -DTAHOE_CODE8_UROWS=4 -DTAHOE_CODE8_THREADS=320 >> gpurun_out/build_v12.log 2>&1
for lib in cur w22 w24 u4 cur w22 w24 u4; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_u.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_u.json').read().strip().splitlines()[-1]); print('$lib', round(d['value']/1e6,2), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"
done
unset TAHOE_LIB_AB
rm -f paper_conf_eurosys_xiedlll21_b200/libtahoe_w2*.so paper_conf_eurosys_xiedlll21_b200/libtahoe_u4.so
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v12.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_v12.log
