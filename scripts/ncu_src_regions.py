"""Aggregate the pc-sampling stall samples of an `ncu --page source --csv --print-source sass` export by
SASS opcode and by code region (contiguous address ranges split at BAR/branch targets are too fine, so
regions are opcode classes), to see where a kernel's warps wait.

    python scripts/ncu_src_regions.py gpurun_out/x.src.csv [top]
"""
import collections
import csv
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
rows = list(csv.reader(open(path)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Address"][0]
h = rows[hi]
si, ni, ei = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
by_op = collections.Counter()
lines = []
tot = 0
for r in rows[hi + 1:]:
    if len(r) <= max(si, ni):
        continue
    try:
        n = int(r[ni] or 0)
    except ValueError:
        continue
    src = r[si].strip()
    op = src.split()[0] if src else "?"
    if op.startswith("@"):
        op = src.split()[1]
    by_op[op.split(".")[0]] += n
    tot += n
    lines.append((n, r[0], src[:90]))
print(f"total samples {tot}")
for op, n in by_op.most_common(top):
    print(f"  {op:12s} {n:8d} {100 * n / max(tot, 1):5.1f}%")
print("top lines:")
for n, a, s in sorted(lines, reverse=True)[:top]:
    print(f"  {n:7d} {a} {s}")
