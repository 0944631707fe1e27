#!/bin/bash
# C4 wide codes: L2 prefetch distance (tiles ahead of each claim), same box
for rep in 1 2; do for p in 0 8 24 64; do echo "prefetch $p"; TAHOE_CODE8_PREFETCH=$p timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep "strategy=2"; done; done
