#!/bin/bash
# wide codes (reading R8): C4 parity + timing
TAG=${1:-c4}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "c4 or rank_code or parity_configs" > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_$TAG.log
timeout 300 python scripts/diag_timing.py 4 500000 2>&1 | grep -v '^{'
timeout 300 python scripts/diag_timing.py 2 2>&1 | grep -v '^{'
