"""Summarise an ncu report (details page) per captured launch: python scripts/ncu_summary.py rep.ncu-rep"""
import csv
import io
import subprocess
import sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "Compute (SM) Throughput", "Executed Ipc Active",
        "Issue Slots Busy", "Registers Per Thread", "Achieved Occupancy", "Theoretical Occupancy",
        "L1/TEX Hit Rate", "L2 Hit Rate", "Eligible Warps Per Scheduler", "No Eligible", "Executed Instructions",
        "Avg. Active Threads Per Warp", "Dynamic Shared Memory Per Block", "Grid Size", "Block Size",
        "Block Limit Registers", "Block Limit Shared Mem"]
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
by = {}
for r in rows[1:]:
    d = dict(zip(h, r))
    k = (d["ID"], d["Kernel Name"][:70])
    by.setdefault(k, {})[d["Metric Name"]] = (d["Metric Value"], d["Metric Unit"])
for (i, name), m in by.items():
    print(f"== launch {i}: {name}")
    for k in KEYS:
        if k in m:
            print(f"   {k:36s} {m[k][0]} {m[k][1]}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
if len(rr) > 2:
    hh = rr[0]
    want = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum",
            "sm__inst_executed_pipe_fma.sum", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
            "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
            "lts__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
            "smsp__thread_inst_executed_per_inst_executed.ratio"]
    idx = {w: hh.index(w) for w in want if w in hh}
    for r in rr[2:]:
        print("  raw:", {w: r[i] for w, i in idx.items()})
