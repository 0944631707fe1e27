#!/bin/bash
# C4 wide codes: timing + ncu captures of the pre-pass and the walk (500K rows)
TAG=${1:-c4p}
mkdir -p gpurun_out
timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep -v '^{'
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_sliced_codes8|k_encode_rows8" -s 2 -c 2 -o gpurun_out/prof_$TAG python scripts/diag_timing.py 4 500000 > gpurun_out/ncu_$TAG.log 2>&1
echo "ncu rc=$?"
