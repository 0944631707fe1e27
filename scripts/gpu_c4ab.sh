#!/bin/bash
# C4 wide codes: back-off between ticket polls (ns), same box
for rep in 1 2; do for sl in 128 32 0 512; do echo "sleep $sl"; TAHOE_CODE8_SLEEP=$sl timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep "strategy=2"; done; done
