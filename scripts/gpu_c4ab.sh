#!/bin/bash
# C4 wide codes A/B in one box: walked tile rows (8 x 6 ring vs 16 x 3 ring), threads per CTA
for rep in 1 2; do
for cfg in "8 512" "16 512" "8 384" "16 384"; do set -- $cfg; echo "tile $1 threads $2"; TAHOE_CODE8_TILE=$1 TAHOE_CODE8_THREADS=$2 timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep "strategy=2"; done
done
timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep "strategy=1"
