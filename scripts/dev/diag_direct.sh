#!/bin/bash
for v in 0 1 2; do
  echo "TAHOE_DIRECT_VARIANT=$v"
  TAHOE_DIRECT_VARIANT=$v python scripts/diag_c5.py 200000 2>&1 | grep "C5 shard"
  TAHOE_DIRECT_VARIANT=$v python scripts/diag_timing.py 2 2>&1 | grep "strategy=0"
  TAHOE_DIRECT_VARIANT=$v python scripts/diag_timing.py 1 100000 2>&1 | grep "strategy=0"
done
TAHOE_DIRECT_VARIANT=2 timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
