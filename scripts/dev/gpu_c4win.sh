#!/bin/bash
# C4 wide codes: window sweep (kernel times), clocks
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv
for w in 0 96 384 2000; do echo "window $w"; TAHOE_CODE8_WINDOW=$w timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep "strategy=[12]"; done
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv
