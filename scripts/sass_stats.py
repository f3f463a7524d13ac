"""Opcode histogram of one kernel's SASS in libsnicit.so: python scripts/sass_stats.py <name-substring> [--dump]"""
import collections
import re
import subprocess
import sys

lib = "paper_conf_icpp_jiangh0h23_b200/lib/libsnicit.so"
pat = sys.argv[1]
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s*Function : ", out)
for f in funcs[1:]:
    name = f.split("\n", 1)[0].strip()
    if pat not in name:
        continue
    ops = collections.Counter()
    lines = []
    for ln in f.split("\n"):
        m = re.match(r"\s*/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_]+)(\.[A-Z0-9_.]+)?", ln)
        if m:
            ops[m.group(2)] += 1
            lines.append(ln.strip())
    print(name, "instructions:", sum(ops.values()))
    print("  " + ", ".join(f"{k}:{v}" for k, v in ops.most_common(25)))
    if "--dump" in sys.argv:
        print("\n".join(lines))
