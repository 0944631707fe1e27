#!/bin/bash
# u16 coded slices: L2 prefetch distance (entries of the CTA's own tile sequence ahead), same box
for rep in 1 2; do for p in 0 1 3; do echo "prefetch $p"; TAHOE_CODES_PREFETCH=$p timeout 200 python scripts/diag_timing.py 3 4000000 2>&1 | grep "strategy=2"; TAHOE_CODES_PREFETCH=$p timeout 200 python scripts/diag_timing.py 2 2>&1 | grep "strategy=2"; done; done
