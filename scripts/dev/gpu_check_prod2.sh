python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -m gpu -q -x -p no:cacheprovider > gpurun_out/gputest_i.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/gputest_i.log
for cfg in 3 2; do
python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_i$cfg.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_i$cfg.json').read().strip().splitlines()[-1]); print('cfg $cfg', round(d['value']/1e6,1), round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), round(d['roofline']['frac'],3))
"
done
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rc scripts/dev/racecheck_mbarrier_canonical.cu && for m in A B C; do compute-sanitizer --tool racecheck /tmp/rc $m 2>&1 | tail -2; done
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python scripts/sanitize_case.py > gpurun_out/sanitize_racecheck_i.log 2>&1; echo "racecheck rc=$?"; tail -2 gpurun_out/sanitize_racecheck_i.log
