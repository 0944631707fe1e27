#!/bin/bash
# A/B of two builds of libtahoe.so on one box (C3 bench): libtahoe_{old,new}.bin
L=paper_conf_eurosys_xiedlll21_b200
mkdir -p gpurun_out
for v in old new old new; do
  cp $L/libtahoe_$v.bin $L/libtahoe.so; touch $L/libtahoe.so
  timeout 300 python bench.py --config 3 --steps 10 --warmup 3 --no-cpu > gpurun_out/ab3_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/ab3_$v.json').read().strip().splitlines()[-1]); print('$v C3', round(d['value']/1e6,2), round(d['roofline']['kernel_ms'],4))"
done
