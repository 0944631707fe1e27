# wide-code row swizzle for the second half-warp's rows: wide tests, GPU suite, C4 bench x2, ncu C4 walk
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v21.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests/test_gpu_wide.py -x -q > gpurun_out/pytest_v21w.log 2>&1; echo "pytest wide rc=$?"; tail -1 gpurun_out/pytest_v21w.log
for i in 1 2; do
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v21.json 2> gpurun_out/bench4_v21.err; python -c "
import json; d=json.loads(open('gpurun_out/bench4_v21.json').read().strip().splitlines()[-1]); print('C4', round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], round(d['roofline']['frac'],3))"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_sliced_codes8$" -s 3 -c 1 -o gpurun_out/prof4_v21 python bench.py --config 4 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu4_v21.log 2>&1; echo "ncu rc=$?"
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_v21.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_v21.log
