# A/B: wide-code work units of 4 rows (10 warps) vs 2 rows (20 / 16 warps); parity of the variants
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v11.log 2>&1; echo build rc=$?
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_u2.so -DTAHOE_CODE8_UROWS=2 -DTAHOE_CODE8_THREADS=640 >> gpurun_out/build_v11.log 2>&1
python -m paper_conf_eurosys_xiedlll21_b200.build --out libtahoe_u2w16.so -DTAHOE_CODE8_UROWS=2 -DTAHOE_CODE8_THREADS=512 >> gpurun_out/build_v11.log 2>&1
for lib in cur u2 u2w16 cur u2 u2w16; do
if [ $lib = cur ]; then unset TAHOE_LIB_AB; else export TAHOE_LIB_AB=libtahoe_$lib.so; fi
timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_u.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_u.json').read().strip().splitlines()[-1]); print('$lib', round(d['value']/1e6,2), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"
done
for lib in u2 u2w16; do
TAHOE_LIB_AB=libtahoe_$lib.so timeout 900 python -m pytest tests/test_gpu_wide.py -x -q > gpurun_out/pytest_v11_$lib.log 2>&1; echo "pytest wide $lib rc=$?"; tail -1 gpurun_out/pytest_v11_$lib.log
done
