"""One SNICIT inference step (bench.py's configuration) inside a cudaProfilerStart/Stop range, after
warm-up, for `ncu --profile-from-start off` (launch lists and --set full captures).

    python scripts/profile_step.py [--config C2] [--t 30] [--mode radix] [--kernel auto] [--steps 1]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import KERNEL_AUTO, KERNEL_CIRC, KERNEL_ELL, SnicitNetwork, default_options  # noqa: E402
from workload import sdgc  # noqa: E402

p = argparse.ArgumentParser()
p.add_argument("--config", default="C2")
p.add_argument("--t", type=int, default=30)
p.add_argument("--s", type=int, default=32)
p.add_argument("--mode", default="radix")
p.add_argument("--kernel", default="auto")
p.add_argument("--steps", type=int, default=1)
p.add_argument("--batch", type=int, default=None)
p.add_argument("--pre-fused", type=int, default=1)
a = p.parse_args()
c = sdgc.CONFIGS[a.config]
B = a.batch or c["B"]
extra = {}
if a.config == "C5":  # config 5: medium MLP (random K = 26 columns, per-entry weights), s = 128, n = N
    Y0 = sdgc.gen_medium_inputs(c["N"], B)
    g = SnicitNetwork.from_network(sdgc.gen_medium_network(c["N"], c["L"]))
    extra = dict(n_segments=0)
    a.s = 128
elif a.mode == "radix" and c["N"] >= 16384:  # compact circulant ABI (the CSC would be 8-32 GB)
    Y0 = sdgc.gen_inputs(c["N"], B)
    cn = sdgc.gen_circulant(c["N"], c["L"])
    g = SnicitNetwork.circulant(cn.N, cn.L, cn.nu, cn.w, cn.bias, cn.ymax)
else:
    Y0 = sdgc.gen_inputs(c["N"], B)
    net = sdgc.gen_network(c["N"], c["L"], a.mode)
    g = SnicitNetwork.from_network(net)
st = torch.cuda.Stream()
g.set_stream(st)
y0 = torch.from_numpy(Y0).cuda()
out = torch.empty_like(y0)
opt = default_options(kernel={"auto": KERNEL_AUTO, "ell": KERNEL_ELL, "circ": KERNEL_CIRC}[a.kernel], pre_fused=a.pre_fused, **extra)
for _ in range(2):
    g.infer(y0, t=a.t, s=a.s, options=opt, y_out=out)
    g.num_categories()
torch.cuda.synchronize()
torch.cuda.profiler.start()
for _ in range(a.steps):
    g.infer(y0, t=a.t, s=a.s, options=opt, y_out=out)
    g.num_categories()
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("stats", g.stats())
g.close()
