"""R32 measurement: C3 (or --config) step time with the popcount layer 0 (pre_fused 1: packed rows only,
7: fp32 two-valued rows too, 6: never, and without R30/R31) for fp32 device rows and packed device bits.
    python scripts/popc_timing.py [--config C2]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork, pack_rows  # noqa: E402
from workload import sdgc  # noqa: E402

p = argparse.ArgumentParser()
p.add_argument("--config", default="C3")
p.add_argument("--t", type=int, default=30)
a = p.parse_args()
c = sdgc.CONFIGS[a.config]
N, L, B = c["N"], c["L"], c["B"]
cn = sdgc.gen_circulant(N, L)
g = SnicitNetwork.circulant(cn.N, cn.L, cn.nu, cn.w, cn.bias, cn.ymax)
Y0 = sdgc.gen_inputs(N, B)
y0 = torch.from_numpy(Y0).cuda()
bits = torch.from_numpy(pack_rows(Y0).view(np.int32)).cuda()
out = torch.empty_like(y0)
st = torch.cuda.Stream()
g.set_stream(st)
for name, pf in (("fp32", 1), ("fp32", 7), ("packed", 1), ("packed", 6)):
    def run():
        if name == "fp32":
            g.infer(y0, t=a.t, s=32, y_out=out, pre_fused=pf)
        else:
            g.infer_packed(bits, t=a.t, s=32, y_out=out, pre_fused=pf)
    for _ in range(3):
        run()
    st.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(10):
        run()
    e1.record(st)
    st.synchronize()
    s_ = g.stats()
    print(f"pre_fused={pf} {a.config} t={a.t} {name}: "
          f"{e0.elapsed_time(e1) / 10:.3f} ms/step, pre_full_rows {s_['pre_full_rows']}, "
          f"pre_popc_rows {s_['pre_popc_rows']}", flush=True)
