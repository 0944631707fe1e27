#!/bin/bash
# C5 shard direct walk: threads per row x rows per CTA x CTAs per SM (L1 share)
for cfg in "4 3" "4 4" "5 3" "5 4" "5 6" "5 8" "6 4" "6 6" "7 4" "7 6" "7 8"; do set -- $cfg; echo "variant $1 persm $2"; TAHOE_DIRECT_VARIANT=$1 TAHOE_DIRECT_PERSM=$2 timeout 300 python scripts/diag_c5.py 300000 2>&1 | grep "C5 shard"; done
