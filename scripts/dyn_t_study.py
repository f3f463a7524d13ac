"""Dynamic threshold layer study (the paper's future work): per config,
step time (CUDA events, median of 5 after 2 warm-ups, device-resident inputs) with the fixed t, with
dyn_t (t chosen by the probe rule), uncompressed (t = L), and a t sweep for reference.

    python scripts/dyn_t_study.py [C1 C2 C5 C3] > gpurun_out/dyn_t.jsonl
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork, default_options  # noqa: E402
from workload import sdgc  # noqa: E402


def timed(fn, k=5):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(k):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(torch.cuda.current_stream())
        fn()
        e1.record(torch.cuda.current_stream())
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


for cfg in (sys.argv[1:] or ["C1", "C2", "C5"]):
    c = sdgc.CONFIGS[cfg]
    N, L, B = c["N"], c["L"], c["B"]
    if cfg == "C5":
        net = sdgc.gen_medium_network(N, L)
        Y0 = sdgc.gen_medium_inputs(N, B)
        t_fixed, s, n = sdgc.medium_t(L), 128, 0
        sweep = [2, 4, 6, 8, 10, 12, 14, 16]
    else:
        net = sdgc.gen_circulant(N, L) if N >= 16384 else sdgc.gen_network(N, L, "radix")
        Y0 = sdgc.gen_inputs(N, B)
        t_fixed, s, n = 30, 32, 16
        sweep = [5, 10, 15, 20, 25, 30, 40]
    if isinstance(net, sdgc.CirculantNetwork):
        g = SnicitNetwork.circulant(net.N, net.L, net.nu, net.w, net.bias, net.ymax)
    else:
        g = SnicitNetwork.from_network(net)
    g.set_stream(torch.cuda.current_stream())
    y0 = torch.from_numpy(Y0).cuda()
    out = torch.empty_like(y0)
    edges = B * net.nnz

    def run(t, dyn=0):
        o = default_options(n_segments=n, dyn_t=dyn)
        g.infer(y0, t=t, s=s, options=o, y_out=out)
        g.num_categories()

    res = {"config": cfg, "t_fixed": t_fixed}
    ms = timed(lambda: run(t_fixed))
    res["fixed"] = {"t": t_fixed, "ms": ms, "edges_per_s": edges / (ms * 1e-3)}
    ms = timed(lambda: run(t_fixed, 1))
    res["dyn_t"] = {"t": g.stats()["threshold_layer"], "ms": ms, "edges_per_s": edges / (ms * 1e-3),
                    "upper_bound": t_fixed}
    ms = timed(lambda: run(L))
    res["uncompressed"] = {"t": L, "ms": ms, "edges_per_s": edges / (ms * 1e-3)}
    res["sweep"] = {}
    for t in sweep:
        if t < L:
            res["sweep"][t] = timed(lambda: run(t), 3)
    print(json.dumps(res), flush=True)
    g.close()
    del y0, out
    torch.cuda.empty_cache()
