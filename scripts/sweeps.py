"""SURVEY 8(f) studies on one B200 (one process, networks loaded once), JSON lines to stdout:

  t-sweep   (Fig. 8 analog, P:1221-1245 / P:1390-1391): C2 step time vs threshold layer t
  B-sweep   (Fig. 9 analog, P:1248-1351 / P:1399-1408): C2 edges/s vs batch size B (t = 30)
  prune_eps (approximate relaxation, P:883-888 / P:1469-1472): residue-heavy C2 (small t) with
            near-zero residual pruning: time, surviving residues, category flips and max |dY| vs exact
  fig6      (Fig. 6 analog): post-convergence time per layer (fused and per-layer post
            modes) vs the uncompressed per-layer kernels' time per layer on the same layers
  C5        (conventional-DNN path): medium sparse MLP 256 x 18, B = 60000, ELL kernel

    python scripts/sweeps.py [--quick]
Times: CUDA events on the library stream, median of 3 after 2 warm-ups (device-resident inputs).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork, default_options  # noqa: E402
from workload import sdgc  # noqa: E402


def timed(g, y0, out, t, s, opt, reps=3, warm=2):
    st = torch.cuda.current_stream()
    for _ in range(warm):
        g.infer(y0, t=t, s=s, options=opt, y_out=out)
        g.num_categories()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(st)
        g.infer(y0, t=t, s=s, options=opt, y_out=out)
        g.num_categories()
        e1.record(st)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def emit(**kw):
    print(json.dumps(kw), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    args = ap.parse_args()
    N, L = 4096, 480
    net = sdgc.gen_network(N, L, "radix")
    B = 60000
    Yh = sdgc.gen_inputs(N, B)
    g = SnicitNetwork.from_network(net)
    g.set_stream(torch.cuda.current_stream())
    y0 = torch.from_numpy(Yh).cuda()
    out = torch.empty_like(y0)
    nnz = net.nnz

    # ---- t sweep (uncompressed = t >= L)
    for t in ([2, 10, 30, L] if args.quick else [2, 5, 10, 15, 20, 25, 30, 40, 60, L]):
        opt = default_options(timing=1)
        ms = timed(g, y0, out, t, 32, opt)
        st = g.stats()
        emit(study="t_sweep", config="C2", t=t, ms=ms, edges_per_s=B * nnz / (ms * 1e-3),
             phases={k: st[k] for k in ("t_pre_ms", "t_convert_ms", "t_post_ms", "t_recover_ms")},
             live_at_t=st["live_at_t"], centroids=st["n_centroids"], residual_at_t=st["residual_at_t"],
             residual_final=st["residual_final"])

    # ---- Fig. 6 analog: post-convergence time per layer vs uncompressed time per layer
    opt_u = default_options(timing=2, pre_fused=0)  # one launch per layer: per-layer CUDA-event times
    g.infer(y0, t=L, s=32, options=opt_u, y_out=out)
    g.infer(y0, t=L, s=32, options=opt_u, y_out=out)
    unc_ms = np.asarray(g.layer_profile(L)["ms"])
    for t in ([30] if args.quick else [10, 20, 30]):
        for pm in (0, 1):
            opt = default_options(timing=1, post_mode=pm)
            ms = timed(g, y0, out, t, 32, opt)
            st = g.stats()
            emit(study="fig6", config="C2", t=t, post_mode=pm, post_ms=st["t_post_ms"],
                 post_ms_per_layer=st["t_post_ms"] / (L - t),
                 uncompressed_ms_per_layer_same_layers=float(unc_ms[t:].mean()),
                 ratio=float(unc_ms[t:].mean()) / (st["t_post_ms"] / (L - t)),
                 residual_at_t=st["residual_at_t"], centroids=st["n_centroids"])

    # ---- B sweep (t = 30)
    for b in ([10000, 60000] if args.quick else [2000, 5000, 10000, 20000, 30000, 60000]):
        opt = default_options()
        ms = timed(g, y0[:b], out[:b], 30, 32, opt)
        emit(study="B_sweep", config="C2", B=b, t=30, ms=ms, edges_per_s=b * nnz / (ms * 1e-3))

    # ---- near-zero residual pruning (approximate) on a residue-heavy threshold
    for t in (3, 5):
        exact = default_options()
        ms0 = timed(g, y0, out, t, 32, exact)
        Y0 = out.cpu().numpy().copy()
        c0 = g.categories()
        st0 = g.stats()
        emit(study="prune_eps", config="C2", t=t, prune_eps=0.0, ms=ms0, residual_at_t=st0["residual_at_t"],
             residual_final=st0["residual_final"], category_flips=0, max_abs_dy=0.0)
        for pe in ([1e-3, 1e-1] if args.quick else [1e-6, 1e-4, 1e-3, 1e-2, 1e-1, 0.5]):
            opt = default_options(prune_eps=pe)
            ms = timed(g, y0, out, t, 32, opt)
            Y = out.cpu().numpy()
            c = g.categories()
            st = g.stats()
            flips = len(set(c.tolist()) ^ set(c0.tolist()))
            emit(study="prune_eps", config="C2", t=t, prune_eps=pe, ms=ms, speedup=ms0 / ms,
                 residual_at_t=st["residual_at_t"], residual_final=st["residual_final"], category_flips=flips,
                 max_abs_dy=float(np.abs(Y - Y0).max()), mean_abs_dy=float(np.abs(Y - Y0).mean()))
    g.close()
    del y0, out

    # ---- config 5: medium sparse MLP (ELL kernel, YMAX 1, per-neuron bias, s = 128, n = N)
    mnet = sdgc.gen_medium_network(256, 18)
    Ym = sdgc.gen_medium_inputs(256, 60000)
    gm = SnicitNetwork.from_network(mnet)
    gm.set_stream(torch.cuda.current_stream())
    y0 = torch.from_numpy(Ym).cuda()
    out = torch.empty_like(y0)
    for t in (sdgc.medium_t(18), 18):
        opt = default_options(n_segments=0, timing=1)
        ms = timed(gm, y0, out, t, 128, opt)
        st = gm.stats()
        emit(study="C5", config="C5 medium 256x18", t=t, ms=ms, edges_per_s=60000 * mnet.nnz / (ms * 1e-3),
             centroids=st["n_centroids"], residual_at_t=st["residual_at_t"], residual_final=st["residual_final"],
             n_categories=st["n_categories"],
             phases={k: st[k] for k in ("t_pre_ms", "t_convert_ms", "t_post_ms", "t_recover_ms")})
    gm.close()


if __name__ == "__main__":
    main()
