import sys; sys.path.insert(0, '.')
import numpy as np, torch, oracle
from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork, KERNEL_ELL
from workload import sdgc
from workload.sdgc import Network
N, L, B, t = 16384, 12, 60, 3
full = sdgc.gen_network(N, L, "radix"); Y0 = sdgc.gen_inputs(N, B)
def sub(k):
    P = full.ptr[: k * (N + 1)]
    nnz = int(P[-1])
    return Network(N=N, L=k, ptr=P, idx=full.idx[:nnz], val=full.val[:nnz], bias=full.bias[:k * N], ymax=full.ymax)
for rep in range(2):
  for k in range(t + 1, L + 1):
    net = sub(k)
    ref = oracle.snicit(net, Y0, t=t)
    res = []
    for pm, kern in ((1, 0), (0, 0), (1, KERNEL_ELL)):
        with SnicitNetwork.from_network(net) as g:
            g.set_stream(torch.cuda.current_stream())
            y0 = torch.from_numpy(Y0).cuda(); out = torch.empty_like(y0)
            g.infer(y0, t=t, s=32, y_out=out, post_mode=pm, kernel=kern)
            Y = out.cpu().numpy(); st = g.stats()
        d = np.abs(Y - ref['Y']); bad = np.nonzero(d.max(1) > 0)[0]
        res.append((pm, kern, len(bad), st['residual_final'], int((ref['ne'] & (ref['M'] >= 0)).sum())))
        if len(bad) and pm == 1 and kern == 0:
            r = bad[0]; cols = np.nonzero(d[r] > 0)[0]
            print("   k", k, "row", r, "ncols", len(cols), "cols mod 32", np.unique(cols % 32)[:8], "vals", Y[r, cols[:3]], ref['Y'][r, cols[:3]])
    print("rep", rep, "layers", k, "nu of last", full.strides[(k - 1) % 3], res, flush=True)
