"""Warp-stall breakdown (pc sampling) and DRAM bytes of each launch in an `ncu --page raw --csv` export.

    python scripts/ncu_stalls.py gpurun_out/x.raw.csv [...]
"""
import csv
import sys

for f in sys.argv[1:]:
    rows = list(csv.reader(open(f)))
    h = rows[0]
    for v in rows[1:]:
        if not v or not v[0].strip().isdigit():
            continue  # units row
        d = dict(zip(h, v))
        print(f"== {f} #{d['ID']} {d['Kernel Name'][:80]}")
        st = []
        for k in h:
            if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
                try:
                    st.append((float(d[k].replace(",", "")), k[len("smsp__pcsamp_warps_issue_stalled_"):]))
                except ValueError:
                    pass
        tot = sum(x for x, _ in st) or 1.0
        print("   stalls: " + ", ".join(f"{k} {100 * x / tot:.1f}%" for x, k in sorted(st, reverse=True)[:9]))
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum"):
            if k in d:
                print(f"   {k} {d[k]}")
