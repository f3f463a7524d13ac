"""Write a markdown summary of one round's measurements for profiles/:
    python scripts/profile_summary.py <bench.json> <launches.csv> <full.raw.csv | full.ncu-rep> > profiles/rNN_summary.md
Launch shares come from the ncu launch list (cold-cache, serialised: compare SHARES, not absolutes)."""
import collections
import csv
import io
import json
import subprocess
import sys

bench, launches, rep = sys.argv[1:4]
b = json.load(open(bench))
print("# Measurement summary\n")
print(f"* metric: {b['metric']}; value **{b['value']:.4g} {b['unit']}**, {b['ms_per_step']:.3f} ms/step "
      f"({b['config']['workload']}, t={b['config']['t']}, s={b['config']['s']})")
r = b.get("roofline") or {}
if r:
    print(f"* dominant kernel `{r['kernel']}` ({r['bound']}-bound): achieved {r['achieved']:.1f} {r['unit']} of "
          f"{r['peak']:.1f} {r['unit']} ({r['peak_source']}) = **{100 * r['frac']:.1f}%**, {r['launches']} launches, "
          f"{100 * (r.get('share_of_step') or 0):.1f}% of the step (CUDA events, live)")
    if r.get("hbm"):
        print(f"  * its HBM traffic: {r['hbm']['achieved_gbs']:.0f} GB/s algorithmic ({100 * r['hbm']['frac']:.1f}% of HBM); "
              f"ncu DRAM bytes per launch {r.get('traffic')} ({r.get('traffic_source')})")
    if r.get("no_const_skip"):
        q = r["no_const_skip"]
        print(f"  * without the constant-row shortcut (pre_fused = 2): {q['avg_launch_ms']:.3f} ms, "
              f"{q['full_row_layers']} full row-layers, **{100 * q['frac']:.1f}%** of the FMA peak")
    if r.get("per_layer_kernels"):
        q = r["per_layer_kernels"]
        print(f"  * one launch per layer (pre_fused = 0): {q['ms_total']:.3f} ms over {q['launches']} launches, "
              f"{q['achieved']:.0f} GB/s = **{100 * q['frac']:.1f}%** of HBM; by stride {q.get('by_stride')}")
for k in ("uncompressed", "e2e", "cpu_baseline"):
    if b.get(k):
        print(f"* {k}: {b[k]['value']:.4g} {b[k]['unit']}" + (f" ({b[k].get('sample')}, {b[k].get('cores')} cores)" if k == "cpu_baseline" else ""))
print(f"* phases (ms): {b.get('phases_ms')}")
print(f"* dynamics: {b.get('dynamics')}")
print(f"* clocks: {b.get('clocks')}\n")

rows = list(csv.reader(open(launches)))
hi = [i for i, rr in enumerate(rows) if "Kernel Name" in rr][0]
h = rows[hi]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
agg = collections.OrderedDict()
for rr in rows[hi + 1:]:
    v = float(rr[vi].replace(",", ""))
    u = rr[ui]
    us = v / 1000 if u in ("ns", "nsecond") else (v if u in ("us", "usecond") else v * 1000)
    name = rr[ki].split("(")[0][:70]
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += us
tot = sum(v[1] for v in agg.values())
print("## Launch list of one step (ncu gpu__time_duration.sum, --clock-control none)\n")
print("| kernel | launches | total us | share |\n|---|---|---|---|")
for k, (n, us) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"| `{k}` | {n} | {us:.1f} | {100 * us / tot:.1f}% |")
print(f"\nTotal {sum(v[0] for v in agg.values())} launches, {tot:.1f} us serialised.\n")

out = open(rep).read() if rep.endswith(".csv") else \
    subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(out)))
hh = rr[0]
want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_sector_hit_rate.pct",
        "smsp__thread_inst_executed_per_inst_executed.ratio"]
idx = [hh.index(w) if w in hh else None for w in want]
print("## ncu --set full (per launch)\n")
print("| " + " | ".join(w.replace("|", "/") for w in want) + " |")
print("|" + "---|" * len(want))
units = rr[1]
for r2 in rr[2:]:
    cells = []
    for w, i in zip(want, idx):
        if i is None:
            cells.append("-")
        else:
            v = r2[i]
            if w == "Kernel Name":
                v = "`" + v.split("(")[0][:60] + "`"
            else:
                v = f"{v} {units[i]}".strip()
            cells.append(v)
    print("| " + " | ".join(cells) + " |")
