# C4 slice count re-measured on the final wide-code walk (33 default vs 37 slices by expected work)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v28.log 2>&1; echo build rc=$?
for t in 0 37 0 37; do
TAHOE_SLICES_TARGET=$t timeout 600 python bench.py --config 4 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_s.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/bench_s.json').read().strip().splitlines()[-1]); print('slices_target $t', round(d['value']/1e6,2), round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4), d['config'].get('n_slices'))
"
done
TAHOE_SLICES_TARGET=37 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none --csv -k regex:"k_sliced_codes8" -c 2 --log-file gpurun_out/launches4_v28.csv \
    python bench.py --config 4 --steps 2 --warmup 3 --no-cpu > gpurun_out/launches4_v28.log 2>&1; echo "launch list rc=$?"; grep -o '"dram__bytes_read.sum","[a-z]*","[0-9,]*"' gpurun_out/launches4_v28.csv | head -2
