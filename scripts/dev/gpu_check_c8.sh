timeout 1200 python -m pytest tests/test_gpu_wide.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py "tests/test_gpu_fullsize.py::test_fullsize_c4_all_rows" -m gpu -q -x -p no:cacheprovider > gpurun_out/gputest_j.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/gputest_j.log
for cfg in 4 3; do
timeout 600 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_j$cfg.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_j$cfg.json').read().strip().splitlines()[-1]); print('cfg $cfg', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"
done
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python scripts/sanitize_case.py > gpurun_out/sanitize_racecheck_j.log 2>&1; echo "racecheck rc=$?"; tail -2 gpurun_out/sanitize_racecheck_j.log
