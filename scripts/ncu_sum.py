"""Print the key ncu metrics of every kernel in a .ncu-rep (details page, CSV)."""
import csv, subprocess, sys
KEYS = ("Duration", "DRAM Throughput", "Issue Slots Busy", "L1/TEX Cache Throughput", "L2 Cache Throughput",
        "Achieved Active Warps Per SM", "Registers Per Thread", "Eligible Warps Per Scheduler", "Grid Size",
        "Block Size", "L1/TEX Hit Rate", "L2 Hit Rate", "Executed Instructions", "Avg. Active Threads Per Warp",
        "No Eligible", "Memory Throughput")
RULES = ("CPIStall", "SharedMemoryConflicts", "WorkloadImbalance", "MemoryCacheAccessPattern", "UncoalescedSharedAccess")
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "details", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[0]
ki, si, mi, ui, vi = h.index("Kernel Name"), h.index("Section Name"), h.index("Metric Name"), h.index("Metric Unit"), h.index("Metric Value")
ri = h.index("Rule Name") if "Rule Name" in h else None
last = None
for r in rows[1:]:
    if r[ki] != last:
        last = r[ki]
        print("==", last)
    if r[mi] in KEYS:
        print(f"  {r[mi]}: {r[vi]} {r[ui]}")
    elif ri is not None and r[ri] in RULES:
        print(f"  [{r[ri]}] {r[ri+2][:260]}")
