#!/bin/bash
# C4 wide codes: two vs four chains per lane (column halves), same box
TAHOE_CODE8_SPLIT=1 timeout 600 python -m pytest tests/test_gpu_wide.py -q -x 2>&1 | tail -1
for rep in 1 2; do for sp in 0 1; do echo "split $sp"; TAHOE_CODE8_SPLIT=$sp timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep "strategy=2"; done; done
