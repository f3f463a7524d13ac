"""Row-resident pre-phase kernel on stride patterns (icache / per-class efficiency study):
    python scripts/pf_experiment.py [N] [B] [t]
Prints, per stride pattern, the fused kernel time, full row-layer evaluations and the FMA-pipe fraction
(2*32*N flops per full row-layer vs 74.45 TFLOP/s)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork, default_options  # noqa: E402
from workload import sdgc  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
B = int(sys.argv[2]) if len(sys.argv) > 2 else 60000
t = int(sys.argv[3]) if len(sys.argv) > 3 else 30
PEAK = 148 * 128 * 2 * 1965e6 / 1e12
Y0 = torch.from_numpy(sdgc.gen_inputs(N, B)).cuda()
out = torch.empty_like(Y0)
std = sdgc.radix_strides(N)
pats = {"radix": std, "nu1": [1], "q32": [N // 32], "str32": [32]}
ONLY = os.environ.get("PF_ONLY")  # one pattern, pre_fused = 2, last iteration inside a profiler range
if ONLY:
    pats = {ONLY: pats[ONLY]}
bias = {1024: -0.3, 4096: -0.35, 16384: -0.4, 65536: -0.45}[N]
for name, pat in pats.items():
    for pf in ((2,) if ONLY else (1, 2)):
        L = t + 1
        nu = np.array([pat[l % len(pat)] for l in range(L)], np.int32)
        w = np.full((L, 32), 1.0 / 16.0, np.float32)
        g = SnicitNetwork.circulant(N, L, nu, w, np.full(L * N, bias, np.float32), 32.0)
        g.set_stream(torch.cuda.current_stream())
        o = default_options(timing=2, pre_fused=pf)
        ms = []
        for it in range(4):
            if ONLY and it == 3:
                torch.cuda.synchronize()
                torch.cuda.profiler.start()
            g.infer(Y0, t=t, s=32, options=o, y_out=out)
            if ONLY and it == 3:
                torch.cuda.synchronize()
                torch.cuda.profiler.stop()
            pr = g.layer_profile()
            if it:
                ms.append(float(np.sum(pr["ms"])))
        st = g.stats()
        k = float(np.median(ms))
        fl = 2.0 * 32 * N * st["pre_full_rows"]
        print(f"{name:6s} pre_fused={pf} kernel {k:7.3f} ms  full row-layers {st['pre_full_rows']:8d}  "
              f"{fl / k / 1e9:6.1f} TFLOP/s = {100 * fl / k / 1e9 / PEAK:5.1f}% of FMA peak  live@t {st['live_at_t']}", flush=True)
        g.close()
