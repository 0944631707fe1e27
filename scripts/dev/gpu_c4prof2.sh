python -m pytest tests -m gpu -x -q -k "wide or codes8 or C4" 2>&1 | tail -3
ncu --set full --clock-control none --import-source on -k regex:"^k_sliced_codes8$" -s 3 -c 1 -o gpurun_out/prof4_r02b python bench.py --config 4 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu4_r02b.log 2>&1
echo ncu rc=$?
