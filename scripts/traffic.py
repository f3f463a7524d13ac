"""DRAM traffic per launch of the a1 layer kernels from an ncu metric capture of one bench step:

    ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
        --profile-from-start off -k regex:layer_circ --csv --log-file traffic.csv \
        python scripts/profile_step.py --config C2
    python scripts/traffic.py traffic.csv C2 > profiles/rNN_traffic_C2.json

bench.py reports the mean (read + write) bytes per launch as roofline.traffic, next to the mean
algorithmic bytes of the same launches."""
import csv
import json
import sys

path, config = sys.argv[1], sys.argv[2]
rows = [r for r in csv.reader(open(path)) if r]
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ki, ii, mi, vi, ui = (h.index(x) for x in ("Kernel Name", "ID", "Metric Name", "Metric Value", "Metric Unit"))
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
         "ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}
launch = {}
for r in rows[hi + 1:]:
    d = launch.setdefault(r[ii], {"kernel": r[ki].split("(")[0]})
    d[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
L = [launch[k] for k in sorted(launch, key=int)]
per = [{"kernel": d["kernel"], "dram_bytes": d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0),
        "us": d.get("gpu__time_duration.sum")} for d in L]
out = {"config": config, "launches": len(per),
       "mean_dram_bytes_per_launch": sum(p["dram_bytes"] for p in per) / max(len(per), 1),
       "source": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum (one bench step, a1 layer kernels)",
       "per_launch": per}
print(json.dumps(out, indent=1))
