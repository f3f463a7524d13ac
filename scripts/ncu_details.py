"""Print the key metrics of an `ncu --page details --csv` export (one block per profiled launch).

    python scripts/ncu_details.py gpurun_out/x.details.csv [more.csv ...]
"""
import csv
import sys

WANT = ["Duration", "DRAM Throughput", "Memory Throughput", "Compute (SM) Throughput", "Issue Slots Busy",
        "Executed Instructions", "Registers Per Thread", "Theoretical Occupancy", "Achieved Occupancy",
        "Eligible Warps Per Scheduler", "No Eligible", "Warp Cycles Per Issued Instruction", "L1/TEX Hit Rate",
        "L2 Hit Rate", "Mem Busy", "Max Bandwidth", "Mem Pipes Busy"]

for f in sys.argv[1:]:
    rows = list(csv.reader(open(f)))
    h = rows[0]
    ki, ii, mn, mv, mu = (h.index(x) for x in ("Kernel Name", "ID", "Metric Name", "Metric Value", "Metric Unit"))
    cur = None
    for r in rows[1:]:
        if r[ii] != cur:
            cur = r[ii]
            print(f"== {f} #{cur} {r[ki][:90]}")
        if r[mn] in WANT:
            print(f"    {r[mn]:<36} {r[mv]} {r[mu]}")
