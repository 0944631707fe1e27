"""Top SASS lines by warp-stall samples of one kernel in an ncu report (source page), with the
per-reason split: python scripts/ncu_stalls.py report.ncu-rep [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
h = r[1]
rows = r[2:]
si = h.index("Warp Stall Sampling (All Samples)")
reasons = ["stall_long_sb", "stall_short_sb", "stall_wait", "stall_selected", "stall_branch_resolving",
           "stall_barrier", "stall_sleep", "stall_mio", "stall_math"]
ri = [h.index(k) for k in reasons if k in h]
tot = sum(int(x[si]) for x in rows)
print(f"total samples {tot}")
sums = {h[j]: sum(int(x[j]) for x in rows) for j in ri}
print({k[6:]: f"{v / tot:.1%}" for k, v in sums.items()})
for x in sorted(rows, key=lambda x: -int(x[si]))[:top]:
    print(f"{int(x[si]) / tot:6.1%} {x[0][-5:]} {x[1][:58]:58s}", {h[j][6:]: x[j] for j in ri if x[j] != '0'})
