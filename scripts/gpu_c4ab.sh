#!/bin/bash
# C4 wide codes: tail / switching experiments
for n in 500000 1000000; do
for sw in 1 0; do echo "n $n switch $sw"; TAHOE_CODE8_SWITCH=$sw timeout 200 python scripts/diag_timing.py 4 $n 2>&1 | grep "strategy=2"; done
echo "n $n chunk 256"; TAHOE_CODE8_CHUNK_MB=256 timeout 200 python scripts/diag_timing.py 4 $n 2>&1 | grep "strategy=2"
done
