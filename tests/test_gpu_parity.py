"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on identical seeded inputs.

Bars (north_star / DESIGN.md): category set bit-exact; fp32 activations within 1e-4 abs or 1e-5 rel
of the plain oracle; the uncompressed path and every step that follows the oracle's evaluation
order are bit-exact (compared with ==, so +0 == -0, reading R19).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from paper_conf_icpp_jiangh0h23_b200 import KERNEL_CIRC, KERNEL_CIRC_SMEM, KERNEL_ELL, SnicitNetwork  # noqa: E402
from workload import sdgc  # noqa: E402
from workload.sdgc import Network  # noqa: E402

pytestmark = pytest.mark.gpu

ATOL, RTOL = 1e-4, 1e-5


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_jiangh0h23_b200 import build
    build.build()


def run_gpu(net, Y0, t, s=32, device_io=True, **opt):
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        if device_io:
            y0 = torch.from_numpy(np.ascontiguousarray(Y0)).cuda()
            out = torch.empty_like(y0)
            g.infer(y0, t=t, s=s, y_out=out, **opt)
            cats = g.categories()
            Y = out.cpu().numpy()
        else:
            out = np.empty_like(Y0)
            g.infer(np.ascontiguousarray(Y0), t=t, s=s, y_out=out, **opt)
            cats = g.categories()
            Y = out
        st = g.stats()
        clus = g.debug_clustering(n_segments=opt.get("n_segments", 16), s=s) if t < net.L else None
    return Y, cats, st, clus


def ragged_net(N, L, seed, ymax=32.0):
    rs = np.random.RandomState(seed)
    ptr, idx, val = [], [], []
    off = 0
    for l in range(L):
        p = [off]
        for j in range(N):
            kk = rs.choice(N, size=rs.randint(0, 40), replace=False)
            idx.extend(kk.tolist())
            val.extend(rs.uniform(-0.2, 0.4, size=len(kk)).tolist())
            off += len(kk)
            p.append(off)
        ptr.extend(p)
    bias = rs.uniform(-0.3, 0.2, size=L * N)
    return Network(N=N, L=L, ptr=np.array(ptr, np.int64), idx=np.array(idx, np.int32), val=np.array(val, np.float32),
                   bias=bias.astype(np.float32), ymax=ymax, mode="ragged")


# ------------------------------------------------------------------------------ single layer, bit-exact

@pytest.mark.parametrize("N,mode,rows", [(1024, "radix", 333), (4096, "radix", 97), (16384, "radix", 9),
                                         (65536, "radix", 3), (1024, "perm", 130), (4096, "random", 41)])
def test_layer_kernels_bit_exact(N, mode, rows):
    net = sdgc.gen_network(N, 4, mode)
    Y0 = sdgc.gen_inputs(N, rows) * np.float32(7.5)  # non-binary values exercise rounding
    Y0[::5] = np.random.RandomState(0).uniform(0, 32, size=Y0[::5].shape).astype(np.float32)
    with SnicitNetwork.from_network(net) as g:
        yin = torch.from_numpy(Y0).cuda()
        for l in range(net.L):
            ref = oracle.layers_f32(net, Y0, l, l + 1)
            kernels = [KERNEL_ELL] + ([KERNEL_CIRC, KERNEL_CIRC_SMEM] if g.layer_is_circulant(l) else [])
            assert g.layer_is_circulant(l) == (mode == "radix")  # N >= 16384: segmented circulant kernel
            for k in kernels:
                out = torch.full_like(yin, float("nan"))
                g.debug_layer(l, yin, out, kernel=k)
                assert np.array_equal(out.cpu().numpy(), ref), f"layer {l} kernel {k}"


@pytest.mark.parametrize("N,nus,rows", [(2048, (32, 64), 37), (3072, (32, 96), 29), (8192, (64, 256, 128), 11),
                                         (16384, (32, 512), 5), (65536, (1024, 2048, 32), 2)])
@pytest.mark.parametrize("uniform", [True, False])
def test_column_stream_kernel_bit_exact(N, nus, rows, uniform):
    """Column-streaming kernel (strided layers, Q = N/nu in {32, 64, 96, 128, 512, 2048}: whole-column
    and ring paths, odd chunk counts) vs the oracle's Eq. 1, per-n weights and per-neuron bias too."""
    rs = np.random.RandomState(N + len(nus))
    L = len(nus)
    if uniform:
        w = np.full((L, 32), 1.0 / 16.0, np.float32)
        bias = np.full(L * N, -0.35, np.float32)
    else:
        w = rs.uniform(-0.1, 0.2, size=(L, 32)).astype(np.float32)
        bias = rs.uniform(-0.4, 0.1, size=L * N).astype(np.float32)
    cn = sdgc.CirculantNetwork(N=N, L=L, nu=np.array(nus, np.int32), w=w, bias=bias, ymax=32.0)
    net = cn.to_network()
    Y0 = rs.uniform(0, 32, size=(rows, N)).astype(np.float32)
    Y0[1::3] = 0.0  # all-zero rows (row flags)
    with SnicitNetwork.circulant(cn.N, cn.L, cn.nu, cn.w, cn.bias, cn.ymax) as g:
        yin = torch.from_numpy(Y0).cuda()
        for l in range(L):
            ref = oracle.layers_f32(net, Y0, l, l + 1)
            for k in (KERNEL_CIRC, KERNEL_CIRC_SMEM):
                out = torch.full_like(yin, float("nan"))
                g.debug_layer(l, yin, out, kernel=k)
                assert np.array_equal(out.cpu().numpy(), ref), f"layer {l} nu {nus[l]} kernel {k}"


@pytest.mark.parametrize("N,L,B,t,dev", [(1024, 40, 700, 4, True), (1024, 40, 700, 40, False),
                                         (4096, 20, 300, 3, True), (16384, 6, 20, 2, False),
                                         (4096, 20, 300, 6, "pinned"), (16384, 6, 20, 3, "pinned"),
                                         (1024, 40, 700, 0, "pinned")])
def test_packed_inputs_equal_fp32(N, L, B, t, dev):
    """snicit_infer_packed (binary rows as a bitmap: expanded inside the row-resident kernel, or
    unpacked by a kernel when that path does not apply, e.g. t = 0) == snicit_infer on the equivalent
    fp32 rows, bit for bit, and == the oracle's categories.  Bits from device memory, pageable host
    memory (staged copy) and pinned host memory (read by the kernel over PCIe, zero-copy)."""
    from paper_conf_icpp_jiangh0h23_b200 import pack_rows
    net = sdgc.gen_network(N, L, "radix")
    Y0 = sdgc.gen_inputs(N, B)
    bits = pack_rows(Y0)
    plain = oracle.layers_f32(net, Y0)
    Y, cats, _, _ = run_gpu(net, Y0, t=t)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        out = torch.empty((B, N), dtype=torch.float32, device="cuda")
        if dev == "pinned":
            src = torch.from_numpy(bits.view(np.int32)).pin_memory().numpy()
        elif dev:
            src = torch.from_numpy(bits.view(np.int32)).cuda()
        else:
            src = bits
        g.infer_packed(src, t=t, s=32, y_out=out)
        cp = g.categories()
        Yp = out.cpu().numpy()
    assert np.array_equal(Yp, Y) and np.array_equal(cp, cats)
    assert np.array_equal(cp, oracle.categories(plain))


@pytest.mark.parametrize("N,L,B,t,pm", [(1024, 60, 1500, 30, 0), (1024, 60, 1500, 30, 1), (1024, 60, 1500, 12, 0),
                                        (1024, 60, 1500, 6, 0), (4096, 40, 400, 25, 0), (4096, 40, 400, 25, 1),
                                        (1024, 60, 1500, 2, 0), (4096, 40, 600, 3, 0)])
def test_constant_centroid_rows(N, L, B, t, pm):
    """post_const (constant centroid rows carried by one scalar chain per circulant layer; in the
    fused mode also constant residue rows over constant centroid pre-activations, small t) is
    bit-identical to the full-row evaluation and to the oracle's SNICIT reference, fused and
    per-layer post modes, with and without residue rows."""
    net = sdgc.gen_network(N, L, "radix")
    Y0 = sdgc.gen_inputs(N, B)
    ref = oracle.snicit(net, Y0, t=t)
    plain = oracle.layers_f32(net, Y0)
    Ya, ca, sa, _ = run_gpu(net, Y0, t=t, post_mode=pm, post_const=1)
    Yb, cb, sb, _ = run_gpu(net, Y0, t=t, post_mode=pm, post_const=0)
    assert sb["const_centroids"] == 0
    assert np.array_equal(Ya, Yb) and np.array_equal(ca, cb)
    assert np.array_equal(Ya, ref["Y"]) and np.array_equal(ca, oracle.categories(plain))
    if t >= 25:  # the synthetic rows have collapsed to the all-YMAX row
        assert sa["const_centroids"] >= 1


def test_layer_ell_ragged_and_values():
    net = ragged_net(64, 3, 1, ymax=4.0)
    Y0 = np.random.RandomState(2).uniform(0, 3, size=(50, 64)).astype(np.float32)
    with SnicitNetwork.from_network(net) as g:
        yin = torch.from_numpy(Y0).cuda()
        for l in range(3):
            out = torch.empty_like(yin)
            g.debug_layer(l, yin, out)
            assert np.array_equal(out.cpu().numpy(), oracle.layers_f32(net, Y0, l, l + 1))


# ------------------------------------------------------------------------------ whole path

@pytest.mark.parametrize("mode", ["radix", "perm"])
def test_uncompressed_path_bit_exact_c1(mode):
    net = sdgc.gen_network(1024, 120, mode)
    Y0 = sdgc.gen_inputs(1024, 2000)
    ref = oracle.layers_f32(net, Y0)
    Y, cats, st, _ = run_gpu(net, Y0, t=net.L)
    assert np.array_equal(Y, ref)
    assert np.array_equal(cats, oracle.categories(ref))
    assert st["n_categories"] == len(cats)


@pytest.mark.parametrize("t", [0, 2, 5, 10, 30])
def test_snicit_c1_vs_oracle(t):
    """C1 (SDGC 1024 x 120, B = 2000): the GPU SNICIT path equals the oracle's SNICIT pipeline
    bit-exactly (same clustering, same evaluation order) and the plain result within tolerance."""
    net = sdgc.gen_network(1024, 120, "radix")
    Y0 = sdgc.gen_inputs(1024, 2000)
    plain = oracle.layers_f32(net, Y0)
    ref = oracle.snicit(net, Y0, t=t, s=32, n=16)
    Y, cats, st, clus = run_gpu(net, Y0, t=t)
    assert np.array_equal(cats, oracle.categories(plain))
    assert np.array_equal(cats, ref["categories"])
    np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)
    assert np.array_equal(Y, ref["Y"])
    # step-level: sampled F, centroids, mapper, ne at t, live rows at t
    assert np.array_equal(clus["live_t"], ref["live_t"])
    assert np.array_equal(clus["F"], ref["F"])
    assert np.array_equal(clus["cent"], ref["cent"])
    assert np.array_equal(clus["M"], ref["M"])
    assert st["n_centroids"] == len(ref["cent"]) >= 1
    assert Y.min() >= 0 and Y.max() <= 32


def test_snicit_ell_forced_equals_auto():
    net = sdgc.gen_network(1024, 40, "radix")
    Y0 = sdgc.gen_inputs(1024, 700)
    a = run_gpu(net, Y0, t=4)
    b = run_gpu(net, Y0, t=4, kernel=KERNEL_ELL)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    assert a[2]["circ_layers"] == 40 and b[2]["circ_layers"] == 0


def test_snicit_perm_4096_small_t():
    net = sdgc.gen_network(4096, 24, "perm")
    Y0 = sdgc.gen_inputs(4096, 300)
    plain = oracle.layers_f32(net, Y0)
    ref = oracle.snicit(net, Y0, t=3)
    Y, cats, st, clus = run_gpu(net, Y0, t=3)
    assert np.array_equal(cats, oracle.categories(plain))
    assert np.array_equal(Y, ref["Y"])
    np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)
    assert st["residual_at_t"] > 0  # residual kernels exercised


def test_medium_net_config5():
    """Config 5 stand-in: YMAX 1, per-neuron values and biases (some > 0: no dead-row drop), no
    downsampling (n = N), s = 128."""
    net = sdgc.gen_medium_network(256, 18)
    Y0 = sdgc.gen_medium_inputs(256, 3000)
    plain = oracle.layers_f32(net, Y0)
    t = sdgc.medium_t(18)
    ref = oracle.snicit(net, Y0, t=t, s=128, n=0)
    Y, cats, st, clus = run_gpu(net, Y0, t=t, s=128, n_segments=0)
    assert np.array_equal(cats, oracle.categories(plain))
    np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)
    assert np.array_equal(Y, ref["Y"])
    assert np.array_equal(clus["cent"], ref["cent"])


def test_host_buffers_path():
    net = sdgc.gen_network(1024, 30, "radix")
    Y0 = sdgc.gen_inputs(1024, 333)
    ref = oracle.snicit(net, Y0, t=7)
    Y, cats, _, _ = run_gpu(net, Y0, t=7, device_io=False)
    assert np.array_equal(Y, ref["Y"]) and np.array_equal(cats, ref["categories"])


@pytest.mark.parametrize("B", [0, 1, 5, 33])
def test_edge_batches(B):
    net = sdgc.gen_network(1024, 16, "radix")
    Y0 = sdgc.gen_inputs(1024, max(B, 1))[:B]
    ref = oracle.snicit(net, Y0, t=3) if B else None
    Y, cats, st, _ = run_gpu(net, Y0, t=3)
    if B:
        assert np.array_equal(Y, ref["Y"]) and np.array_equal(cats, ref["categories"])
    else:
        assert len(cats) == 0


def test_s_one_and_no_dead_drop():
    net = sdgc.gen_network(1024, 20, "radix")
    Y0 = sdgc.gen_inputs(1024, 400)
    plain = oracle.layers_f32(net, Y0)
    for kw in (dict(s=1), dict(s=32, drop_dead_rows=0), dict(s=64, n_segments=0)):
        s = kw.pop("s")
        Y, cats, _, _ = run_gpu(net, Y0, t=5, s=s, **kw)
        assert np.array_equal(cats, oracle.categories(plain))
        np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)


def test_near_zero_pruning_runs():
    """prune_eps > 0 is the paper's approximate relaxation: outside exact parity; the
    outputs must stay in range and close to the exact result for a tiny eps."""
    net = sdgc.gen_network(1024, 30, "radix")
    Y0 = sdgc.gen_inputs(1024, 500)
    Y, cats, _, _ = run_gpu(net, Y0, t=4, prune_eps=1e-6)
    assert Y.min() >= -1e-6 and Y.max() <= 32


@pytest.mark.parametrize("mode,N,L,B,t", [("radix", 1024, 60, 1500, 2), ("radix", 1024, 60, 1500, 6),
                                          ("perm", 4096, 20, 300, 3), ("radix", 4096, 40, 400, 4)])
def test_post_modes_identical(mode, N, L, B, t):
    """Fused multi-layer post-convergence kernels (default) == per-layer Eq. 5 + ne_idx compaction
     == the oracle's SNICIT pipeline, bit for bit, with residue rows present."""
    net = sdgc.gen_network(N, L, mode)
    Y0 = sdgc.gen_inputs(N, B)
    ref = oracle.snicit(net, Y0, t=t)
    a = run_gpu(net, Y0, t=t, post_mode=0)
    b = run_gpu(net, Y0, t=t, post_mode=1)
    d = run_gpu(net, Y0, t=t, post_mode=0, res_sparse=0)
    assert a[2]["residual_at_t"] > 0
    for Y, cats, st, _ in (a, b, d):
        assert np.array_equal(Y, ref["Y"])
        assert np.array_equal(cats, ref["categories"])
    assert a[2]["residual_final"] == b[2]["residual_final"] == int((ref["ne"] & (ref["M"] >= 0)).sum())


@pytest.mark.parametrize("N,L,B,t", [(16384, 12, 60, 3), (65536, 8, 12, 2)])
def test_large_rows_segmented(N, L, B, t):
    """C3/C4-sized rows (16384 / 65536 neurons): segmented circulant kernel (A- and C-segments),
    per-layer post mode for N > 24576, both post modes for 16384; against the oracle."""
    net = sdgc.gen_network(N, L, "radix")
    Y0 = sdgc.gen_inputs(N, B)
    plain = oracle.layers_f32(net, Y0)
    ref = oracle.snicit(net, Y0, t=t)
    for pm in ((0, 1) if N <= 24576 else (1,)):
        Y, cats, st, clus = run_gpu(net, Y0, t=t, post_mode=pm)
        assert np.array_equal(cats, oracle.categories(plain))
        assert np.array_equal(Y, ref["Y"])
        np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)
        assert st["circ_layers"] > 0
    Yu, catsu, _, _ = run_gpu(net, Y0, t=L)  # uncompressed path, bit-exact
    assert np.array_equal(Yu, plain) and np.array_equal(catsu, oracle.categories(plain))
    Ys, catss, _, _ = run_gpu(net, Y0, t=t, kernel=KERNEL_CIRC_SMEM)  # staged kernels for strided layers
    assert np.array_equal(catss, oracle.categories(plain)) and np.array_equal(Ys, ref["Y"])


@pytest.mark.parametrize("N,L", [(1024, 10), (4096, 9)])
def test_post_modes_unsaturated_centroids(N, L):
    """Per-layer post mode with centroids far from saturation (random real-valued inputs), so the
    centroid pre-activations a_c differ per column: regression for the a_c of a row's tail outputs."""
    net = sdgc.gen_network(N, L, "radix")
    rs = np.random.RandomState(5)
    Y0 = (sdgc.gen_inputs(N, 200) * rs.uniform(0.2, 1.5, size=(200, N))).astype(np.float32)
    ref = oracle.snicit(net, Y0, t=2, n=0, eta=0.0, eps=0.01, s=8)
    for pm in (0, 1):
        Y, cats, st, _ = run_gpu(net, Y0, t=2, s=8, n_segments=0, eta=0.0, eps=0.01, post_mode=pm)
        assert st["residual_at_t"] > 0
        assert np.array_equal(Y, ref["Y"]) and np.array_equal(cats, ref["categories"])


@pytest.mark.parametrize("N,L,B,t", [(1024, 30, 500, 4), (16384, 9, 40, 3)])
def test_compact_circulant_loader_equals_csc(N, L, B, t):
    """snicit_load_network_circulant (compact RadiX form) == snicit_load_network (explicit CSC)."""
    c = sdgc.gen_circulant(N, L)
    net = c.to_network()
    Y0 = sdgc.gen_inputs(N, B)
    ref = run_gpu(net, Y0, t=t)
    with SnicitNetwork.circulant(N, L, c.nu, c.w, c.bias, c.ymax) as g:
        g.set_stream(torch.cuda.current_stream())
        y0 = torch.from_numpy(Y0).cuda()
        out = torch.empty_like(y0)
        g.infer(y0, t=t, s=32, y_out=out)
        cats = g.categories()
        Y = out.cpu().numpy()
        with pytest.raises(Exception):
            g.infer(y0, t=t, s=32, kernel=KERNEL_ELL)  # no ELL copy in compact form
    assert np.array_equal(Y, ref[0]) and np.array_equal(cats, ref[1])
    assert np.array_equal(cats, oracle.categories(oracle.layers_circulant_f32(c, Y0)))


@pytest.mark.parametrize("N,L,B,t", [(1024, 40, 800, 3), (4096, 24, 300, 3), (16384, 10, 40, 3)])
def test_cluster_centroid_trajectory(N, L, B, t):
    """Fused post mode: the 8-CTA cluster (DSMEM) centroid trajectory == one CTA per centroid == the
    oracle pipeline, with residue rows present (they consume the cluster kernel's a_c)."""
    net = sdgc.gen_network(N, L, "radix")
    Y0 = sdgc.gen_inputs(N, B)
    ref = oracle.snicit(net, Y0, t=t)
    a = run_gpu(net, Y0, t=t, post_cluster=1)
    b = run_gpu(net, Y0, t=t, post_cluster=0)
    assert a[2]["residual_at_t"] > 0
    for Y, cats, _, _ in (a, b):
        assert np.array_equal(Y, ref["Y"]) and np.array_equal(cats, ref["categories"])


# ------------------------------------------------------------------------------ row-resident pre phase

def _pf_inputs(N, B, seed):
    """Binary MNIST-like rows plus the degenerate rows the fused kernel branches on: all-zero rows,
    constant rows (0 < v < 32 and v = 32), rows that die after a few layers, random-valued rows."""
    rs = np.random.RandomState(seed)
    if int(np.sqrt(N)) ** 2 == N:
        Y0 = sdgc.gen_inputs(N, B)
    else:  # non-square N: binary rows at the SDGC-like density
        Y0 = (rs.uniform(size=(B, N)) < 0.25).astype(np.float32)
    Y0[1::7] = 0.0
    Y0[2::7] = np.float32(32.0)
    Y0[3::7] = np.float32(0.375)
    Y0[4::7] *= np.float32(0.02)  # sparse small values: dead after a few layers
    Y0[5::7] = rs.uniform(0, 32, size=Y0[5::7].shape).astype(np.float32)
    return Y0


@pytest.mark.parametrize("N,nus,B", [(1024, (1, 32), 301), (2048, (1, 32, 64), 97), (4096, (1, 32, 128), 150),
                                     (8192, (1, 64, 256, 32), 41), (16384, (1, 32, 512), 23),
                                     (16384, (512, 1, 32, 1), 17), (32768, (1, 32, 1024), 9),
                                     (65536, (1, 32, 1024, 2048), 9), (65536, (2048, 32, 1, 1024), 5)])
@pytest.mark.parametrize("drop", [1, 0])
def test_pre_fused_bit_exact(N, nus, B, drop):
    """Row-resident pre-convergence kernel (every stride class: nu = 1, Q = 32, STR with compile-time
    nu = 32 and runtime nu = 64) with and without the constant-row shortcut (R26) == the per-layer
    kernels == the oracle's Eq. 1, bit for bit, on the uncompressed path (t = L: every layer runs in the
    pre phase) and in the full SNICIT pipeline."""
    L = 3 * len(nus) + 1
    nu = np.array([nus[l % len(nus)] for l in range(L)], np.int32)
    w = np.full((L, 32), 1.0 / 16.0, np.float32)
    bias = np.repeat(np.array([-0.3 - 0.01 * (l % 3) for l in range(L)], np.float32), N)
    cn = sdgc.CirculantNetwork(N=N, L=L, nu=nu, w=w, bias=bias, ymax=32.0)
    net = cn.to_network()
    Y0 = _pf_inputs(N, B, N + B)
    plain = oracle.layers_f32(net, Y0)
    res = {}
    single = N <= 16384  # one CTA per row exists (kernels_pre_fused.cu); pre_fused = 4: cluster form (N >= 16384)
    for pf in (1, 2, 0, 5, 4):  # 1/2: split layout, 5: paired-half layout, 4: cluster form, 0: per layer
        if (pf == 4 and N < 16384) or (pf == 5 and not single):
            continue
        Y, cats, st, _ = run_gpu(net, Y0, t=L, drop_dead_rows=drop, pre_fused=pf)
        # N > 16384: pre_fused = 1 runs the cluster form (a row does not fit one CTA), 2 the per-layer path
        want = 2 if pf == 4 or (pf == 1 and not single) else (0 if pf == 0 or not single else 1)
        assert st["pre_fused"] == want, f"pre_fused={pf}"
        res[pf] = (Y, cats, st)
        assert np.array_equal(Y, plain), f"pre_fused={pf}"
        assert np.array_equal(cats, oracle.categories(plain))
    if single:
        assert res[1][2]["pre_const_rows"] > 0 and res[2][2]["pre_const_rows"] == 0
        assert res[1][2]["pre_full_rows"] < res[2][2]["pre_full_rows"]
    if 4 in res:
        assert res[4][2]["pre_const_rows"] > 0 and res[4][2]["live_at_t"] == res[0][2]["live_at_t"]
    assert res[1][2]["live_at_t"] == res[0][2]["live_at_t"] == res[2][2]["live_at_t"]
    # SNICIT pipeline with conversion at t = L // 2: fused pre phase == per-layer pre phase
    Ya, ca, sa, cla = run_gpu(net, Y0, t=L // 2, drop_dead_rows=drop, pre_fused=1)
    Yb, cb, sb, clb = run_gpu(net, Y0, t=L // 2, drop_dead_rows=drop, pre_fused=0)
    assert np.array_equal(Ya, Yb) and np.array_equal(ca, cb)
    if N >= 16384:
        Yc, cc, sc, _ = run_gpu(net, Y0, t=L // 2, drop_dead_rows=drop, pre_fused=4)
        assert sc["pre_fused"] == 2 and np.array_equal(Yc, Yb) and np.array_equal(cc, cb)
    assert np.array_equal(ca, oracle.categories(plain))
    assert np.allclose(Ya, plain, atol=ATOL, rtol=RTOL)


def test_pre_fused_positive_bias_and_fallbacks():
    """A positive bias (no dead-row dropping after it, R23) runs fused and stays exact; per-n weights,
    per-neuron bias or an unsupported N fall back to the per-layer kernels (stats.pre_fused == 0)."""
    N, L, B = 4096, 7, 80
    nu = np.array([1, 32, 128, 1, 32, 128, 1], np.int32)
    w = np.full((L, 32), 1.0 / 16.0, np.float32)
    bias = np.full(L * N, -0.35, np.float32)
    bias[4 * N:5 * N] = 0.05
    cn = sdgc.CirculantNetwork(N=N, L=L, nu=nu, w=w, bias=bias, ymax=32.0)
    net = cn.to_network()
    Y0 = _pf_inputs(N, B, 7)
    plain = oracle.layers_f32(net, Y0)
    Y, cats, st, _ = run_gpu(net, Y0, t=L)
    assert st["pre_fused"] == 1 and np.array_equal(Y, plain)
    # per-n weights -> per-layer kernels
    w2 = w.copy()
    w2[2, 5] = np.float32(0.07)
    cn2 = sdgc.CirculantNetwork(N=N, L=L, nu=nu, w=w2, bias=bias, ymax=32.0)
    net2 = cn2.to_network()
    Y2, _, st2, _ = run_gpu(net2, Y0, t=L)
    assert st2["pre_fused"] == 0 and np.array_equal(Y2, oracle.layers_f32(net2, Y0))
    # but a prefix of eligible layers before t still runs fused
    Y3, _, st3, _ = run_gpu(net2, Y0, t=2)
    assert st3["pre_fused"] == 1
    assert np.array_equal(oracle.categories(oracle.layers_f32(net2, Y0)), run_gpu(net2, Y0, t=2)[1])


@pytest.mark.parametrize("N,L,B", [(16384, 13, 40), (65536, 9, 14)])
@pytest.mark.parametrize("drop", [1, 0])
def test_pre_const_per_layer(N, L, B, drop):
    """Per-layer pre-convergence path (segmented + column-streaming kernels) in constant-row mode
    (R26: rows whose outputs are all equal leave the list and are carried by a scalar chain; with R30,
    rows whose range bounds Y(t) leave too) == R26 alone == the path without either == the oracle, bit
    for bit: uncompressed (t = L) and SNICIT (t = 4)."""
    net = sdgc.gen_network(N, L, "radix")
    Y0 = _pf_inputs(N, B, 3)
    plain = oracle.layers_f32(net, Y0)
    for t in (L, 4):
        res = {}
        for pc in (1, 2, 0):  # 2: R26 without the range prediction (R30)
            Y, cats, st, _ = run_gpu(net, Y0, t=t, drop_dead_rows=drop, pre_fused=0, pre_const=pc)
            assert st["pre_fused"] == 0
            res[pc] = (Y, cats, st)
            assert np.array_equal(cats, oracle.categories(plain))
            if t == L:
                assert np.array_equal(Y, plain), f"pre_const={pc}"
        assert np.array_equal(res[1][0], res[0][0]) and np.array_equal(res[1][1], res[0][1])
        assert np.array_equal(res[2][0], res[0][0]) and np.array_equal(res[2][1], res[0][1])
        assert res[1][2]["live_at_t"] == res[0][2]["live_at_t"]
        assert res[1][2]["pre_const_rows"] > 0 and res[0][2]["pre_const_rows"] == 0
