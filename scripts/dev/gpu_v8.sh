# C3 per-GPU step at the row counts of 2/4/8-way strong scaling (4M/G rows)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v8.log 2>&1; echo build rc=$?
for r in 500000 1000000 2000000; do
timeout 600 python bench.py --config 3 --rows $r --no-cpu > gpurun_out/bench3_v8_$r.json 2> gpurun_out/bench3_v8_$r.err; echo "rows $r rc=$?"; cut -c1-220 gpurun_out/bench3_v8_$r.json
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv -k regex:"k_sliced_codes|k_encode_rows|k_finalize" -c 6 --log-file gpurun_out/launches3_v8_500k.csv \
    python bench.py --config 3 --rows 500000 --steps 2 --warmup 3 --no-cpu > gpurun_out/launches3_v8.log 2>&1; echo "launch list rc=$?"
