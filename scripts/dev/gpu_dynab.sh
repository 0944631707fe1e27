#!/bin/bash
# u16 coded slices: static (k_sliced_codes) vs dynamic walk (k_sliced_codes8<..., W16>), same box
TAHOE_CODES_DYNAMIC=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "rank_code or parity_configs or full_size_c2 or full_size_c3" 2>&1 | tail -2
for rep in 1 2; do for dy in 0 1; do echo "dynamic $dy"; TAHOE_CODES_DYNAMIC=$dy timeout 200 python scripts/diag_timing.py 3 4000000 2>&1 | grep "strategy=2"; TAHOE_CODES_DYNAMIC=$dy timeout 200 python scripts/diag_timing.py 2 2>&1 | grep "strategy=2"; done; done
