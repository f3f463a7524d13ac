"""Per-stride-class timing of the plain layer kernel (Eq. 1) on B fully live rows.

For each layer of one stride cycle of an SDGC radix network (N neurons), runs snicit_debug_layer on
B device rows (MNIST-like inputs pushed through a few layers so values are 0..32 like the real path)
and reports CUDA-event time per launch and the achieved algorithmic GB/s (8 B per row-element:
DESIGN.md §7).  Inputs (B*N*4 bytes) are larger than L2 at the default sizes.

    python scripts/layer_bench.py [--N 4096] [--B 60000] [--iters 20] [--kernel auto|circ|ell|smem]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import KERNEL_AUTO, KERNEL_CIRC, KERNEL_CIRC_SMEM, KERNEL_ELL, SnicitNetwork  # noqa: E402
from workload import sdgc  # noqa: E402

p = argparse.ArgumentParser()
p.add_argument("--N", type=int, default=4096)
p.add_argument("--B", type=int, default=60000)
p.add_argument("--iters", type=int, default=20)
p.add_argument("--kernel", default="auto")
p.add_argument("--peak", type=float, default=6650.0)
a = p.parse_args()
kern = {"auto": KERNEL_AUTO, "circ": KERNEL_CIRC, "ell": KERNEL_ELL, "smem": KERNEL_CIRC_SMEM}[a.kernel]
strides = sdgc.radix_strides(a.N)
L = len(strides)
cn = sdgc.gen_circulant(a.N, L)
g = SnicitNetwork.circulant(cn.N, cn.L, cn.nu, cn.w, cn.bias, cn.ymax)
st = torch.cuda.current_stream()
g.set_stream(st)
y0 = torch.from_numpy(sdgc.gen_inputs(a.N, min(a.B, 4096))).cuda()
x = y0.repeat((a.B + y0.shape[0] - 1) // y0.shape[0], 1)[: a.B].contiguous()
y = torch.empty_like(x)
# two warm layers so the rows hold SDGC-like values (0 .. 32, not just 0/1)
g.debug_layer(0, x, y, kern)
g.debug_layer(1 % L, y, x, kern)
torch.cuda.synchronize()
res = []
for l in range(L):
    for _ in range(3):
        g.debug_layer(l, x, y, kern)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(a.iters):
        g.debug_layer(l, x, y, kern)
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.iters
    gbs = 8.0 * a.B * a.N / (ms * 1e-3) / 1e9
    res.append({"layer": l, "nu": int(strides[l]), "ms": round(ms, 4), "GBps": round(gbs, 1),
                "frac": round(gbs / a.peak, 4)})
    print(json.dumps({"N": a.N, "B": a.B, **res[-1]}), flush=True)
tot = sum(r["ms"] for r in res)
print(json.dumps({"N": a.N, "B": a.B, "cycle_ms": round(tot, 4),
                  "cycle_frac": round(8.0 * a.B * a.N * L / (tot * 1e-3) / 1e9 / a.peak, 4)}))
g.close()
