ncu --set full --clock-control none --import-source on -k regex:"k_encode_rows8" -s 1 -c 1 -o gpurun_out/prof4enc_r02 python bench.py --config 4 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu4enc_r02.log 2>&1
echo ncu rc=$?
