"""Small parity repro of one configuration (debugging aid; compute-sanitizer friendly)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork  # noqa: E402
from workload import sdgc  # noqa: E402

p = argparse.ArgumentParser()
p.add_argument("--N", type=int, default=4096)
p.add_argument("--L", type=int, default=20)
p.add_argument("--B", type=int, default=300)
p.add_argument("--t", type=int, default=3)
p.add_argument("--mode", default="radix")
p.add_argument("--opt", default="")
a = p.parse_args()
opt = {k: float(v) if "." in v else int(v) for k, v in (kv.split("=") for kv in a.opt.split(",") if kv)}
net = sdgc.gen_network(a.N, a.L, a.mode)
Y0 = sdgc.gen_inputs(a.N, a.B)
ref = oracle.snicit(net, Y0, t=a.t)
with SnicitNetwork.from_network(net) as g:
    g.set_stream(torch.cuda.current_stream())
    y0 = torch.from_numpy(Y0).cuda()
    out = torch.empty_like(y0)
    g.infer(y0, t=a.t, s=32, y_out=out, **opt)
    cats = g.categories()
    st = g.stats()
    Y = out.cpu().numpy()
print({k: st[k] for k in ("residual_at_t", "residual_final", "res_nnz_at_t", "res_full_rl", "res_sparse_rl",
                          "res_scalar_rl", "n_centroids")})
print("Y equal:", np.array_equal(Y, ref["Y"]), "cats equal:", np.array_equal(cats, ref["categories"]))
