mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v34.log 2>&1; echo build rc=$?
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_v34.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_v34.log
timeout 1800 python scripts/fuzz_big.py 0 400 > gpurun_out/fuzz_big_v34.log 2>&1; echo "fuzz_big rc=$?"; tail -n 1 gpurun_out/fuzz_big_v34.log
timeout 1200 python scripts/fuzz_configs.py 0 120 > gpurun_out/fuzz_configs_v34.log 2>&1; echo "fuzz_configs rc=$?"; tail -n 1 gpurun_out/fuzz_configs_v34.log
timeout 2000 python scripts/ablation.py 2 3 4 5 > gpurun_out/ablation.log 2>&1; echo "ablation rc=$?"
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v34.json 2> gpurun_out/bench4_v34.err; python -c "
import json; d=json.loads(open('gpurun_out/bench4_v34.json').read().strip().splitlines()[-1]); print('C4', round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], d['config']['n_slices'], d['config']['lockstep_eff_sim'])"
