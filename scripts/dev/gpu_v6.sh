# C4: 33 slices (default) vs 37 slices cut by expected work (4 CTAs per slice on 148 SMs); walk DRAM
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v6.log 2>&1; echo build rc=$?
./scripts/dev/smem_random > gpurun_out/smem_random.txt 2>&1; echo "smem_random rc=$?"; cat gpurun_out/smem_random.txt
for t in 0 37 74; do
TAHOE_SLICES_TARGET=$t timeout 600 python bench.py --config 4 --no-cpu > gpurun_out/bench4_v6_$t.json 2> gpurun_out/bench4_v6_$t.err; echo "bench4 $t rc=$?"; cut -c1-200 gpurun_out/bench4_v6_$t.json
TAHOE_SLICES_TARGET=$t timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_sliced_codes8|k_encode_rows8" -c 6 --log-file gpurun_out/launches4_v6_$t.csv \
    python bench.py --config 4 --steps 2 --warmup 3 --no-cpu > gpurun_out/launches4_v6_$t.log 2>&1; echo "launch list rc=$?"
done
