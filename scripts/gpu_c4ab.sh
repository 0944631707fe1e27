#!/bin/bash
# C4 wide-code pre-pass variants (same box): 0 = 512 threads x 8 rows, 1 = 1024 x 8, 2 = 1024 x 4
for rep in 1 2; do for v in 0 1 2; do echo "enc8 $v"; TAHOE_ENC8=$v timeout 200 python scripts/diag_timing.py 4 500000 2>&1 | grep "strategy=2"; done; done
