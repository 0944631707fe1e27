# A/B: four chains per lane in the u16 coded walk (TAHOE_CODED_SPLIT) on C3 / C2, parity with it on
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v9.log 2>&1; echo build rc=$?
for s in 0 1 0 1; do for c in 3 2; do
TAHOE_CODED_SPLIT=$s timeout 600 python bench.py --config $c --no-cpu > gpurun_out/bench${c}_v9_$s.json 2> gpurun_out/bench${c}_v9_$s.err; echo "C$c split=$s rc=$?"; python -c "
import json; d=json.loads(open('gpurun_out/bench${c}_v9_$s.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['roofline']['kernel_ms'])"
done; done
TAHOE_CODED_SPLIT=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "coded or rank" > gpurun_out/pytest_v9.log 2>&1; echo "pytest split rc=$?"; tail -2 gpurun_out/pytest_v9.log
