"""Per-kernel summary of an ncu launch-list CSV (gpu__time_duration.sum, optional DRAM bytes):
count, mean time and mean DRAM bytes per launch, in launch order of first appearance."""
import collections
import csv
import sys


def summarize(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    idi = hdr.index("ID")
    per = collections.OrderedDict()
    for r in rows[h + 1:]:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0][:70]
        per.setdefault(name, collections.defaultdict(dict))[r[idi]][r[mi]] = float(r[vi].replace(",", ""))
    out = []
    for name, launches in per.items():
        n = len(launches)
        t = sum(m.get("gpu__time_duration.sum", 0) for m in launches.values()) / n
        rd = sum(m.get("dram__bytes_read.sum", 0) for m in launches.values()) / n
        wr = sum(m.get("dram__bytes_write.sum", 0) for m in launches.values()) / n
        out.append((name, n, t, rd, wr))
    return out


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(p)
        for name, n, t, rd, wr in summarize(p):
            print(f"  {name:70s} n={n:4d} {t / 1e6:9.4f} ms  DRAM rd {rd / 1e9:8.3f} GB wr {wr / 1e9:8.3f} GB")
