# packer re-cuts failing chunks before raising k: C4 slices / lockstep / walk; GPU suite
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v32.log 2>&1; echo build rc=$?
for i in 1 2; do
timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v32.json 2> gpurun_out/bench4_v32.err; python -c "
import json; d=json.loads(open('gpurun_out/bench4_v32.json').read().strip().splitlines()[-1]); print('C4', round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], round(d['roofline']['frac'],3), d['config']['n_slices'], d['config']['lockstep_eff_sim'])"
done
for c in 3 2; do
timeout 600 python bench.py --config $c --no-cpu > gpurun_out/bench${c}_v32.json 2> gpurun_out/bench${c}_v32.err; python -c "
import json; d=json.loads(open('gpurun_out/bench${c}_v32.json').read().strip().splitlines()[-1]); print('C$c', round(d['value']/1e6,2), d['ms_per_step'], d['roofline']['kernel_ms'], d['config']['n_slices'], d['config']['lockstep_eff_sim'])"
done
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_v32.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_v32.log
