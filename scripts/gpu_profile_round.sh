#!/bin/bash
# Profiles of the bench kernels (B200_PROFILING.md recipe): the launch list of the default bench
# command (C3) and one `ncu --set full` capture of the dominant kernel per config (full-size inputs).
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r02.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/launches_r02.log 2>&1
echo "launch list rc=$?"
for cfg in 3 2 4; do
  k=k_sliced_codes; [ $cfg = 4 ] && k=k_sliced_codes8
  ncu --set full --clock-control none --import-source on -k regex:"^${k}$" -s 3 -c 1 \
      -o gpurun_out/prof${cfg}_r02 python bench.py --config $cfg --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu${cfg}_r02.log 2>&1
  echo "ncu C$cfg rc=$?"
done
ncu --set full --clock-control none --import-source on -k regex:k_encode_rows_banks -s 3 -c 1 \
    -o gpurun_out/prof3enc_r02 python bench.py --config 3 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu3enc_r02.log 2>&1
echo "ncu C3 pre-pass rc=$?"
