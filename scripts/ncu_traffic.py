"""Refresh profiles/ncu_traffic.json from the round's `ncu --set full` captures (one kernel per
report): DRAM bytes read / written per launch and the LSU global-load sector use, the `traffic`
field of bench.py's roofline.  python scripts/ncu_traffic.py C3=gpurun_out/prof3_r02.ncu-rep ..."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = os.path.join(ROOT, "profiles", "ncu_traffic.json")


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--print-units", "base"],
                         capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return dict(zip(r[0], r[2]))   # row 1: units


def num(v):
    return float(v.replace(",", ""))


d = json.load(open(P)) if os.path.exists(P) else {}
for arg in sys.argv[1:]:
    cfg, rep = arg.split("=", 1)
    m = raw(rep)
    rd, wr = num(m["dram__bytes_read.sum"]), num(m["dram__bytes_write.sum"])
    e = d.setdefault(cfg, {})
    prev = {k: e.get(k) for k in ("kernel", "dram_bytes_per_launch")}
    k = m["Kernel Name"]
    e["kernel"] = k[5:] if k.startswith("void ") else k
    e["kernel"] = e["kernel"].split(">(")[0] + ">" if ">(" in e["kernel"] else e["kernel"]
    e["dram_read_bytes"] = int(rd)
    e["dram_write_bytes"] = int(wr)
    e["dram_bytes_per_launch"] = int(rd + wr)
    sec = m.get("smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.ratio")
    if sec:
        e["global_ld_bytes_per_sector"] = num(sec)
        e["global_ld_sector_efficiency"] = num(sec) / 32.0
    e["source"] = f"{os.path.relpath(rep, ROOT)} (scripts/gpu_profile_round.sh: ncu --set full, full size, round 2 HEAD)"
    if prev["dram_bytes_per_launch"] and prev["dram_bytes_per_launch"] != e["dram_bytes_per_launch"]:
        e["previous"] = prev
    print(cfg, e["kernel"], e["dram_bytes_per_launch"])
json.dump(d, open(P, "w"), indent=1)
