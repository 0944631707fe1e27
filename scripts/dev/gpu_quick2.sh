#!/bin/bash
# quick loop: parity file + timing diagnostic + ncu launch list of the bench command
TAG=${1:-q}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_parity_$TAG.log 2>&1; echo "parity rc=$?"
tail -3 gpurun_out/pytest_parity_$TAG.log
python scripts/diag_timing.py 2 2>&1 | grep -v '^{'
python scripts/diag_timing.py 3 1000000 2>&1 | grep -v '^{'
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
python - <<PY
import csv
rows=list(csv.reader(open('gpurun_out/launches_$TAG.csv')))
hdr=None
for r in rows:
    if 'Kernel Name' in r: hdr=r; continue
    if hdr and len(r)==len(hdr):
        d=dict(zip(hdr,r)); print(d['Kernel Name'][:60], d['Metric Value'])
PY
python -c "
import gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
for c in (2,3):
    F=T.Forest(gen.make_forest(c),device=0).layout(gen.make_calibration(c))
    print(c, F.stats()['cta_split'])
"
