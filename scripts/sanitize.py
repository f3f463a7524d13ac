"""Small SNICIT runs for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
    compute-sanitizer --tool memcheck python scripts/sanitize.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import KERNEL_ELL, SnicitNetwork  # noqa: E402
from workload import sdgc  # noqa: E402

for mode, N, L, B, t, kw in (("radix", 1024, 24, 300, 3, {}), ("radix", 4096, 12, 64, 2, {}),
                             ("perm", 1024, 10, 100, 2, {}), ("radix", 1024, 12, 200, 2, dict(post_mode=1)),
                             ("radix", 1024, 12, 100, 3, dict(kernel=KERNEL_ELL))):
    net = sdgc.gen_network(N, L, mode)
    Y0 = torch.from_numpy(sdgc.gen_inputs(N, B)).cuda()
    out = torch.empty_like(Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(Y0, t=t, s=32, y_out=out, **kw)
        cats = g.categories()
        torch.cuda.synchronize()
    print(mode, N, L, B, t, kw, "categories", len(cats), "sum", float(out.sum()))
# row-resident pre phase at N = 16384 (three row buffers), per-layer constant-row mode (segmented +
# column kernels, kernels_const.cu), packed rows streamed from pinned host memory (ready flags)
from paper_conf_icpp_jiangh0h23_b200 import pack_rows  # noqa: E402
for N, L, B, t, kw in ((16384, 7, 12, 3, {}), (16384, 7, 12, 7, dict(pre_fused=0)), (65536, 5, 4, 3, {})):
    net = sdgc.gen_network(N, L, "radix")
    Y0 = torch.from_numpy(sdgc.gen_inputs(N, B)).cuda()
    out = torch.empty_like(Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(Y0, t=t, s=32, y_out=out, **kw)
        cats = g.categories()
        torch.cuda.synchronize()
    print("radix", N, L, B, t, kw, "categories", len(cats), "sum", float(out.sum()))
net = sdgc.gen_network(4096, 12, "radix")
Yh = sdgc.gen_inputs(4096, 5000)
bits = torch.from_numpy(pack_rows(Yh).view(np.int32)).pin_memory()
out = torch.empty((5000, 4096), dtype=torch.float32, device="cuda")
with SnicitNetwork.from_network(net) as g:
    g.set_stream(torch.cuda.current_stream())
    g.infer_packed(bits.numpy(), t=4, s=32, y_out=out)
    cats = g.categories()
    torch.cuda.synchronize()
print("packed streamed 4096 12 5000 4 categories", len(cats), "sum", float(out.sum()))
# round 2: cluster-split row-resident kernel (pre_fused = 4), two-pass Alg. 2, sparse-entry residues,
# interleaved ELL tiles in constant-row mode, dynamic t probe, device category export
for N, L, B, t, kw in ((16384, 7, 9, 7, dict(pre_fused=4)), (65536, 5, 3, 5, dict(pre_fused=4))):
    net = sdgc.gen_network(N, L, "radix")
    Y0 = torch.from_numpy(sdgc.gen_inputs(N, B)).cuda()
    out = torch.empty_like(Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(Y0, t=t, s=32, y_out=out, **kw)
        cats = g.categories()
        torch.cuda.synchronize()
    print("cluster", N, L, B, t, "categories", len(cats), "sum", float(out.sum()))
for mode, N, L, B, t, kw in (("radix", 4096, 16, 200, 10, dict(timing=1)), ("perm", 1024, 12, 200, 12, {}),
                             ("random", 1024, 10, 150, 4, {}), ("radix", 1024, 40, 400, 30, dict(dyn_t=1))):
    net = sdgc.gen_network(N, L, mode)
    Y0 = torch.from_numpy(sdgc.gen_inputs(N, B)).cuda()
    out = torch.empty_like(Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(Y0, t=t, s=32, y_out=out, **kw)
        cats = g.categories()
        buf = torch.empty(1 + B, dtype=torch.int64, device="cuda")
        g.categories_device(buf)
        torch.cuda.synchronize()
    print(mode, N, L, B, t, kw, "categories", len(cats), "sum", float(out.sum()))
# sparse residues (near-duplicate rows, t = 0)
N, L, B = 4096, 8, 120
base = sdgc.gen_inputs(N, 8)
Yh = base[np.arange(B) % 8].copy()
rs = np.random.RandomState(0)
for r in range(32, B):
    k = rs.choice(N, 2, replace=False)
    Yh[r, k] = 1.0 - Yh[r, k]
net = sdgc.gen_network(N, L, "radix")
Y0 = torch.from_numpy(Yh).cuda()
out = torch.empty_like(Y0)
with SnicitNetwork.from_network(net) as g:
    g.set_stream(torch.cuda.current_stream())
    g.infer(Y0, t=0, s=32, y_out=out)
    st = g.stats()
    torch.cuda.synchronize()
print("sparse residues: sparse row-layers", st["res_sparse_rl"], "sum", float(out.sum()))
# round 2 (late): range prediction (R30/R31) near the fixed point, popcount layer 0 (R32) on packed and fp32
# rows, TMA stores of constant rows, Y(t) kept in y_out (recovery skip), per-layer path with R30
for N, B, kw in ((16384, 24, {}), (16384, 24, dict(pre_fused=7)), (4096, 200, dict(pre_fused=7)),
                 (65536, 6, {}), (1024, 300, dict(pre_fused=0, pre_const=1))):
    net = sdgc.gen_network(N, 40, "radix")
    rs = np.random.RandomState(N)
    Yh = (-sdgc.SDGC_BIAS[N] + rs.uniform(-0.05, 0.05, size=(B, 1)) + rs.uniform(-0.03, 0.03, size=(B, N)))
    Yh = Yh.clip(0, None).astype(np.float32)
    Yh[::3] = sdgc.gen_inputs(N, B)[::3]
    Y0 = torch.from_numpy(Yh).cuda()
    out = torch.empty_like(Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(Y0, t=30, s=32, y_out=out, **kw)
        cats = g.categories()
        bits = torch.from_numpy(pack_rows((Yh != 0).astype(np.float32)).view(np.int32)).cuda()
        g.infer_packed(bits, t=30, s=32, y_out=out)
        cats2 = g.categories()
        torch.cuda.synchronize()
    print("range/popc", N, B, kw, "categories", len(cats), len(cats2), "sum", float(out.sum()))
print("sanitize run done")
# round 2 (r02c): general-CSC row-interleaved kernel (kernels_gen.cu: G = 2 / 4 / 16 tiles, padded and ragged
# columns, PLAIN with constant-row ranges, CENTROID / RESIDUAL in the per-layer post phase) and the
# cluster pre kernel with R30 / R31 (the default for N = 65536)
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from test_gpu_round2c import random_k_net  # noqa: E402
for N, K, B in ((256, 26, 300), (1024, 30, 70), (4096, 32, 20)):
    net = random_k_net(N, 4, K, seed=N)
    Y0 = torch.rand(B, N, device="cuda") * 8
    out = torch.empty_like(Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(Y0, t=2, s=32, y_out=out)
        cats = g.categories()
        torch.cuda.synchronize()
    print("gen", N, K, B, "categories", len(cats), "sum", float(out.sum()))
net = sdgc.gen_medium_network(256, 18)
Y0 = torch.from_numpy(sdgc.gen_medium_inputs(256, 700)).cuda()
out = torch.empty_like(Y0)
with SnicitNetwork.from_network(net) as g:
    g.set_stream(torch.cuda.current_stream())
    g.infer(Y0, t=8, s=128, n_segments=0, y_out=out)
    torch.cuda.synchronize()
print("gen medium post per-layer sum", float(out.sum()))
net = sdgc.gen_network(65536, 6, "radix")
Y0 = torch.from_numpy(sdgc.gen_inputs(65536, 4)).cuda()
out = torch.empty_like(Y0)
with SnicitNetwork.from_network(net) as g:
    g.set_stream(torch.cuda.current_stream())
    g.infer(Y0, t=6, s=32, y_out=out)
    torch.cuda.synchronize()
print("cluster R30/R31 65536 sum", float(out.sum()))
