#!/bin/bash
# Profiles of the bench kernels (B200_PROFILING.md recipe): the launch list of the default bench
# command (C3) and one `ncu --set full` capture of the dominant kernel per config (full-size
# inputs), plus the C3 row-coding pre-pass and the C5 direct walk.  bash scripts/gpu_profile_round.sh TAG
TAG=${1:-r02}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/launches_$TAG.log 2>&1
echo "launch list rc=$?"
for cfg in 3 2 4; do
  k=k_sliced_codes; [ $cfg = 4 ] && k=k_sliced_codes8
  ncu --set full --clock-control none --import-source on -k regex:"^${k}$" -s 3 -c 1 \
      -o gpurun_out/prof${cfg}_$TAG python bench.py --config $cfg --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu${cfg}_$TAG.log 2>&1
  echo "ncu C$cfg rc=$?"
done
ncu --set full --clock-control none --import-source on -k regex:k_encode_rows_banks -s 3 -c 1 \
    -o gpurun_out/prof3enc_$TAG python bench.py --config 3 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu3enc_$TAG.log 2>&1
echo "ncu C3 pre-pass rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_encode_rows8 -s 3 -c 1 \
    -o gpurun_out/prof4enc_$TAG python bench.py --config 4 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu4enc_$TAG.log 2>&1
echo "ncu C4 pre-pass rc=$?"
ncu --set full --clock-control none --import-source on -k regex:k_direct_tlp -s 20 -c 1 \
    -o gpurun_out/prof5_$TAG python bench.py --config 5 --rows 1000000 --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu5_$TAG.log 2>&1
echo "ncu C5 rc=$?"
