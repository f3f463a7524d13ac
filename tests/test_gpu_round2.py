"""GPU parity for the round-2 pieces of the path, through the C ABI against the CPU oracle:

* row sharding: G shards run one after another on one GPU with row_offset ("fake
  multi-GPU") give the category set of G = 1 and of the oracle, and the device category export;
* the two-rank bench step end to end through libsnicit (gloo hook, both ranks on cuda:0);
* the sparse-entry residue form (north_star "only the nonzero residual entries are propagated") on
  inputs whose residues are sparse, bit-identical to the dense form and the oracle;
* the approximate mode (near-zero residue pruning) element by element vs the oracle;
* the SNICIT_CSR loader branch; a non-blocking stream while the legacy default stream is busy.
"""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from paper_conf_icpp_jiangh0h23_b200 import CSR_FORMAT, SnicitNetwork, pack_rows, shard_capacity, shard_rows  # noqa: E402
from workload import sdgc  # noqa: E402
from workload.sdgc import Network  # noqa: E402

pytestmark = pytest.mark.gpu

ATOL, RTOL = 1e-4, 1e-5
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_jiangh0h23_b200 import build
    build.build()


def _infer(g, Y0, t, s=32, row_offset=0, **opt):
    y0 = torch.from_numpy(np.ascontiguousarray(Y0)).cuda()
    out = torch.empty_like(y0)
    g.infer(y0, t=t, s=s, y_out=out, row_offset=row_offset, **opt)
    return out.cpu().numpy(), g.categories(), g.stats()


# ------------------------------------------------------------------------------ sharding

@pytest.mark.parametrize("N,L,B,t,mode", [(4096, 60, 6000, 10, "radix"), (4096, 60, 6000, 30, "radix"),
                                          (1024, 120, 2000, 5, "radix"), (1024, 40, 2000, 6, "perm")])
def test_sharded_inference_matches_single_gpu_and_oracle(N, L, B, t, mode):
    """Rows are independent (Eq. 1), clustering runs per shard (reading R14): for G = 1, 2, 4,
    8 contiguous shards with row_offset, the concatenated category sets are identical to G = 1 and to the
    oracle's, and every shard's activations are within tolerance of the plain oracle (perm: the general-CSC
    kernel on every shard, ragged tiles included)."""
    net = sdgc.gen_network(N, L, mode)
    Y0 = sdgc.gen_inputs(N, B)
    plain = oracle.layers_f32_fast(net, Y0)
    ref_cats = oracle.categories(plain)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        for G in (1, 2, 4, 8):
            cats, Ys = [], []
            for r in range(G):
                a, b = shard_rows(B, G, r)
                Y, c, st = _infer(g, Y0[a:b], t, row_offset=a)
                assert np.all((c >= a) & (c < b))
                cats.append(c)
                Ys.append(Y)
                # device export of this shard's categories (the all-gather buffer)
                cap = shard_capacity(B, G)
                buf = torch.full((1 + cap,), -7, dtype=torch.int64, device="cuda")
                g.categories_device(buf)
                torch.cuda.synchronize()
                hb = buf.cpu().numpy()
                assert hb[0] == len(c) and np.array_equal(hb[1:1 + len(c)], c) and np.all(hb[1 + len(c):] == -7)
            assert np.array_equal(np.concatenate(cats), ref_cats), f"G = {G}"
            np.testing.assert_allclose(np.concatenate(Ys), plain, atol=ATOL, rtol=RTOL)


def test_bench_two_ranks_gloo_hook():
    """bench.py --gpus 2 (it launches torchrun itself) with SNICIT_DIST_BACKEND=gloo: both ranks share
    cuda:0, each infers its row shard through libsnicit, the padded category buffers are all-gathered;
    the line reports n_gpus 2 and the category count of a one-rank run."""
    env = dict(os.environ, SNICIT_DIST_BACKEND="gloo")
    common = ["--config", "C1", "--quick", "--steps", "2", "--warmup", "3"]

    def run(extra, e):
        p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + common + extra, env=e,
                           capture_output=True, text=True, timeout=900, cwd=ROOT)
        assert p.returncode == 0, p.stderr[-3000:]
        lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
        assert len(lines) == 1, p.stdout[-2000:]
        return json.loads(lines[0])

    two = run(["--gpus", "2"], env)
    one = run(["--gpus", "1"], dict(os.environ))
    assert two["n_gpus"] == 2 and one["n_gpus"] == 1
    assert two["categories"] == one["categories"] > 0
    assert len(two["per_rank"]) == 2 and sum(r["rows"] for r in two["per_rank"]) == 2000
    assert two["config"]["global_batch"] == one["config"]["global_batch"] == 2000


# ------------------------------------------------------------------------------ sparse-entry residues

def _near_duplicate_inputs(N, B, flips, seed):
    """Rows 0..31 are 8 distinct base images (the sampled rows: they become the centroids); every other
    row is a base image with `flips` pixels toggled, so its residue at t = 0 has ~`flips` non-zeros."""
    rs = np.random.RandomState(seed)
    base = sdgc.gen_inputs(N, 8, row0=seed * 8)
    Y = np.repeat(base, (B + 7) // 8, axis=0)[:B].copy()
    Y[:32] = base[np.arange(32) % 8]
    for r in range(32, B):
        Y[r] = base[r % 8]
        k = rs.choice(N, flips, replace=False)
        Y[r, k] = 1.0 - Y[r, k]
    return Y.astype(np.float32)


@pytest.mark.parametrize("N,L,B,t,flips", [(4096, 24, 600, 0, 3), (4096, 24, 600, 1, 1), (1024, 30, 800, 0, 2),
                                           (16384, 10, 64, 0, 5)])
def test_sparse_entry_residues(N, L, B, t, flips):
    """Residue rows with few non-zeros propagate only the outputs their non-zeros touch (fused post mode,
    circulant layers): bit-identical to the dense-row form (res_sparse = 0) and to the oracle's SNICIT
    pipeline; the stats show sparse row-layers evaluated."""
    net = sdgc.gen_network(N, L, "radix")
    Y0 = _near_duplicate_inputs(N, B, flips, N + t)
    ref = oracle.snicit(net, Y0, t=t)
    plain = oracle.layers_f32(net, Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        Ys, cs, sts = _infer(g, Y0, t, res_sparse=1)
        Yd, cd, std = _infer(g, Y0, t, res_sparse=0)
    assert sts["residual_at_t"] > 0 and sts["res_sparse_rl"] > 0 and std["res_sparse_rl"] == 0
    assert sts["res_nnz_at_t"] <= sts["residual_at_t"] * (flips if t == 0 else 32 * flips)
    assert np.array_equal(Ys, Yd) and np.array_equal(cs, cd)
    assert np.array_equal(Ys, ref["Y"]) and np.array_equal(cs, ref["categories"])
    assert np.array_equal(cs, oracle.categories(plain))
    np.testing.assert_allclose(Ys, plain, atol=ATOL, rtol=RTOL)


def test_sparse_entry_residues_per_n_weights_and_bias():
    """The sparse form with per-n weights and per-neuron biases (non-uniform circulant layers)."""
    N, L, B = 2048, 12, 300
    rs = np.random.RandomState(9)
    nu = np.array([[1, 32, 64][l % 3] for l in range(L)], np.int32)
    w = rs.uniform(0.02, 0.09, size=(L, 32)).astype(np.float32)
    bias = rs.uniform(-0.4, -0.1, size=L * N).astype(np.float32)
    cn = sdgc.CirculantNetwork(N=N, L=L, nu=nu, w=w, bias=bias, ymax=32.0)
    net = cn.to_network()
    base = (rs.uniform(size=(8, N)) < 0.3).astype(np.float32) * 3.0
    Y0 = base[np.arange(B) % 8].copy()
    for r in range(32, B):
        k = rs.choice(N, 2, replace=False)
        Y0[r, k] += 1.0
    ref = oracle.snicit(net, Y0, t=0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        Ys, cs, sts = _infer(g, Y0, 0, res_sparse=1)
        Yd, cd, _ = _infer(g, Y0, 0, res_sparse=0)
    assert sts["res_sparse_rl"] > 0
    assert np.array_equal(Ys, Yd) and np.array_equal(Ys, ref["Y"]) and np.array_equal(cs, ref["categories"])


# ------------------------------------------------------------------------------ approximate mode (f2)

@pytest.mark.parametrize("prune_eps", [0.1, 0.5])
@pytest.mark.parametrize("pm", [0, 1])
def test_prune_eps_matches_oracle(prune_eps, pm):
    """Near-zero residue pruning (|v| <= prune_eps -> 0, reading R8) is outside exact parity
    with the plain result, but the GPU's approximate pipeline equals the oracle's approximate pipeline
    (oracle_post_layer's prune_eps branch) element by element, fused and per-layer post modes."""
    net = sdgc.gen_network(1024, 40, "radix")
    Y0 = sdgc.gen_inputs(1024, 1500)
    ref = oracle.snicit(net, Y0, t=3, prune_eps=prune_eps)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        Y, cats, st = _infer(g, Y0, 3, prune_eps=prune_eps, post_mode=pm)
    assert st["residual_at_t"] > 0
    assert np.array_equal(Y, ref["Y"]) and np.array_equal(cats, ref["categories"])


# ------------------------------------------------------------------------------ loader / streams

def test_csr_loader_equals_csc():
    """SNICIT_CSR (per input k its outputs j): transposed on load, each output column ordered by
    ascending k.  A CSC net stored in ascending-k order loads to the same plan: identical results."""
    net = sdgc.gen_network(1024, 12, "random")  # columns stored ascending (workload recipe)
    N, L = net.N, net.L
    ptr_r, idx_r, val_r = [0], [], []
    for l in range(L):
        p, idx, val, _ = net.layer(l)
        cols = np.repeat(np.arange(N), np.diff(p))
        order = np.lexsort((cols, idx))  # by input k, then output j
        k_sorted = idx[order]
        idx_r.extend(cols[order].tolist())
        val_r.extend(val[order].tolist())
        counts = np.bincount(k_sorted, minlength=N)
        base = ptr_r[-1]
        ptr_r.extend((base + np.cumsum(counts)).tolist())
        if l < L - 1:
            ptr_r.append(ptr_r[-1])
    ptr_r = np.array(ptr_r, np.int64)
    csr = Network(N=N, L=L, ptr=ptr_r, idx=np.array(idx_r, np.int32), val=np.array(val_r, np.float32),
                  bias=net.bias, ymax=net.ymax, mode="csr")
    Y0 = sdgc.gen_inputs(N, 500)
    plain = oracle.layers_f32(net, Y0)
    with SnicitNetwork.from_network(net) as g1:
        g1.set_stream(torch.cuda.current_stream())
        Ya, ca, _ = _infer(g1, Y0, 4)
    with SnicitNetwork(N, L, csr.ptr, csr.idx, csr.val, csr.bias, csr.ymax, fmt=CSR_FORMAT) as g2:
        g2.set_stream(torch.cuda.current_stream())
        Yb, cb, _ = _infer(g2, Y0, 4)
        Yu, cu, _ = _infer(g2, Y0, L)
    assert np.array_equal(Ya, Yb) and np.array_equal(ca, cb)
    assert np.array_equal(Yu, plain) and np.array_equal(cu, oracle.categories(plain))


@pytest.mark.parametrize("pre_fused", [0, 1])
def test_nonblocking_stream_with_busy_default_stream(pre_fused):
    """All work of a handle (including the first-call workspace initialisation of the self-clearing
    counters) is ordered on the handle's stream: a fresh non-blocking stream while the legacy default
    stream is busy gives the oracle's result (per-layer path: column-streaming + segmented kernels)."""
    N, L, B = 16384, 8, 48
    net = sdgc.gen_network(N, L, "radix")
    Y0 = sdgc.gen_inputs(N, B)
    plain = oracle.layers_f32(net, Y0)
    y0 = torch.from_numpy(Y0).cuda()
    big = torch.randn(8192, 8192, device="cuda")
    torch.cuda.synchronize()
    s = torch.cuda.Stream()  # created cudaStreamNonBlocking
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(s)
        for _ in range(3):
            for _ in range(20):  # keep the legacy default stream busy
                big = big @ big
                big = big / big.norm()
            out = torch.empty_like(y0)
            with torch.cuda.stream(s):
                g.infer(y0, t=L, s=32, y_out=out, pre_fused=pre_fused)
                cats = g.categories()
                s.synchronize()
                got = out.cpu().numpy()
            assert np.array_equal(got, plain) and np.array_equal(cats, oracle.categories(plain))


def test_misaligned_device_pointer_rejected():
    net = sdgc.gen_network(1024, 4, "radix")
    Y0 = sdgc.gen_inputs(1024, 9)
    with SnicitNetwork.from_network(net) as g:
        flat = torch.from_numpy(np.ascontiguousarray(Y0)).cuda().flatten()
        buf = torch.empty(9 * 1024 + 1, dtype=torch.float32, device="cuda")
        buf[1:].copy_(flat)
        y0 = buf[1:].view(9, 1024)  # contiguous, 4-byte offset
        with pytest.raises(Exception):
            g.infer(y0, t=2, s=8)


@pytest.mark.parametrize("N,L,B,mode", [(1024, 12, 400, "perm"), (4096, 10, 150, "perm"), (1024, 9, 300, "random")])
@pytest.mark.parametrize("drop", [1, 0])
def test_general_layers_constant_rows(N, L, B, mode, drop):
    """Constant-row mode (R26) of the general (ELL) layer kernels: rows whose outputs are all equal leave
    the active list and are carried by a scalar chain, bit-identical to evaluating every live row (and
    to the oracle), uncompressed and SNICIT (t = 4); constant centroid rows likewise (R25)."""
    net = sdgc.gen_network(N, L, mode)
    rs = np.random.RandomState(N + L)
    Y0 = sdgc.gen_inputs(N, B)
    Y0[1::5] = 0.0
    Y0[2::5] = np.float32(32.0)
    Y0[3::5] = np.float32(0.5)
    plain = oracle.layers_f32(net, Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        for t in (L, 4):
            Ya, ca, sa = _infer(g, Y0, t, drop_dead_rows=drop, pre_const=1)
            Yb, cb, sb = _infer(g, Y0, t, drop_dead_rows=drop, pre_const=0, post_const=0)
            assert np.array_equal(Ya, Yb) and np.array_equal(ca, cb)
            assert np.array_equal(ca, oracle.categories(plain))
            if t == L:
                assert np.array_equal(Ya, plain)
                if mode == "perm":  # uniform weights, 32 per column: the constant-row mode applies
                    assert sa["pre_const_rows"] > 0 and sb["pre_const_rows"] == 0
            else:
                np.testing.assert_allclose(Ya, plain, atol=ATOL, rtol=RTOL)


# ------------------------------------------------------------------------------ dynamic t (f3)

def test_dynamic_threshold_layer():
    """dyn_t: t is chosen from the first s rows (the first layer after which all live probe rows are
    identical, at most threshold_layer; the uncompressed path when they stay distinct).  Any t gives the
    plain result: categories equal the oracle's, activations within tolerance, and the chosen t is the
    one the rule names on the oracle's own layer-by-layer rows."""
    net = sdgc.gen_network(1024, 120, "radix")
    Y0 = sdgc.gen_inputs(1024, 2000)
    plain = oracle.layers_f32_fast(net, Y0)
    # the rule on the oracle: first l with every live row among the first 32 identical
    want = None
    y = Y0[:32].copy()
    for l in range(30):
        y = oracle.layers_f32(net, y, l, l + 1)
        live = y[(y != 0).any(1)]
        if len(live) == 0 or (live == live[0]).all():
            want = l + 1
            break
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        Y, cats, st = _infer(g, Y0, 30, dyn_t=1)
        assert st["threshold_layer"] == (min(2 * want, 30) if want is not None else 30)
        assert np.array_equal(cats, oracle.categories(plain))
        np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)
        # packed input and host input choose the same t
        from paper_conf_icpp_jiangh0h23_b200 import pack_rows
        out = torch.empty((2000, 1024), dtype=torch.float32, device="cuda")
        g.infer_packed(pack_rows(Y0), t=30, s=32, y_out=out, dyn_t=1)
        assert g.stats()["threshold_layer"] == st["threshold_layer"]
        assert np.array_equal(g.categories(), cats)


def test_dynamic_t_non_converging_net_goes_uncompressed():
    """A random-init medium net (config 5) never converges: the probe rows stay distinct, so dyn_t takes
    the uncompressed path (t = L), bit-exact with the oracle."""
    net = sdgc.gen_medium_network(256, 18)
    Y0 = sdgc.gen_medium_inputs(256, 3000)
    plain = oracle.layers_f32(net, Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        Y, cats, st = _infer(g, Y0, sdgc.medium_t(18), s=128, n_segments=0, dyn_t=1)
    assert st["threshold_layer"] == 18
    assert np.array_equal(Y, plain) and np.array_equal(cats, oracle.categories(plain))


# ------------------------------------------------------------------------------ per-layer dynamics log

@pytest.mark.parametrize("N,drop", [(1024, 1), (1024, 0), (4096, 1), (16384, 1), (65536, 1)])
def test_range_prediction_bit_exact(N, drop):
    """R30 on rows built to sit near the repelling fixed point of out(m) = 2m + b0 (values -b0 +- small
    noise): rows drift to YMAX or to zero over many layers, so the range test fires at long and short
    horizons (k up to 32 and the clamped k > 32).  Uncompressed (t = L) outputs equal the oracle's bit for
    bit in the row-resident kernel (pre_fused 1, and 6 = without R30) and in the per-layer constant-row
    path (pre_const 1, and 2 = without R30); SNICIT (t < L) outputs agree across the pre paths."""
    L, B = 48, (240 if N <= 4096 else (40 if N <= 16384 else 8))
    net = sdgc.gen_network(N, L, "radix")
    fix = -sdgc.SDGC_BIAS[N]
    rs = np.random.RandomState(N + drop)
    base = rs.uniform(fix - 0.05, fix + 0.05, size=(B, 1))
    Y0 = (base + rs.uniform(-0.03, 0.03, size=(B, N))).clip(0, None).astype(np.float32)
    Y0[::5] = sdgc.gen_inputs(N, B)[::5]
    plain = oracle.layers_f32(net, Y0)
    want_c = oracle.categories(plain)
    runs = {}
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        modes = [("pl1", dict(pre_fused=0, pre_const=1)), ("pl2", dict(pre_fused=0, pre_const=2))]
        if N <= 16384:
            modes += [("pf1", dict(pre_fused=1)), ("pf6", dict(pre_fused=6))]
        else:  # a row does not fit one CTA: pre_fused = 1 is the cluster form (R26/R30/R31, round 2 (r02c))
            modes += [("pf1", dict(pre_fused=1))]
        if N >= 16384:
            modes += [("pf4", dict(pre_fused=4))]
        for name, kw in modes:
            runs[name] = _infer(g, Y0, L, drop_dead_rows=drop, **kw)
            assert np.array_equal(runs[name][0], plain), name
            assert np.array_equal(runs[name][1], want_c), name
            runs[name + "_t"] = _infer(g, Y0, 40, drop_dead_rows=drop, **kw)
    for name, _ in modes:
        assert np.array_equal(runs[name + "_t"][0], runs["pl2_t"][0]), name
        assert np.array_equal(runs[name + "_t"][1], runs["pl2_t"][1]), name
    assert np.allclose(runs["pl1_t"][0], plain, atol=ATOL, rtol=RTOL)
    if N <= 16384:
        assert runs["pf1"][2]["pre_fused"] == 1 and runs["pf6"][2]["pre_fused"] == 1
        assert runs["pf1"][2]["pre_full_rows"] < runs["pf6"][2]["pre_full_rows"]
    else:
        assert runs["pf1"][2]["pre_fused"] == 2
    if N >= 16384:
        assert runs["pf4"][2]["pre_fused"] == 2


@pytest.mark.parametrize("t", [7, 5])
def test_cluster_positive_bias_and_horizons(t):
    """Cluster pre kernel (the default at N = 65536) on a net with a positive-bias layer: a zero row is not
    absorbing before it (no dead-row drop, R23) and the range tables cover only layers that share one
    bias (R30 off here: the layers < t do not), so rows are carried by the constant-row rule and full
    evaluation alone; outputs equal the oracle's bit for bit and the per-layer path's."""
    N, L, B = 65536, 7, 6
    nu = np.array([1, 32, 1024, 2048, 1, 32, 1024], np.int32)
    w = np.full((L, 32), 1.0 / 16.0, np.float32)
    bias = np.full(L * N, -0.45, np.float32)
    bias[4 * N:5 * N] = 0.05
    cn = sdgc.CirculantNetwork(N=N, L=L, nu=nu, w=w, bias=bias, ymax=32.0)
    net = cn.to_network()
    rs = np.random.RandomState(t)
    Y0 = sdgc.gen_inputs(N, B)
    Y0[1] = np.float32(32.0)
    Y0[2] = 0.0
    Y0[3] = rs.uniform(0.4, 0.5, size=N).astype(np.float32)
    plain = oracle.layers_f32(net, Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        a = _infer(g, Y0, t)
        b = _infer(g, Y0, t, pre_fused=0)
    assert a[2]["pre_fused"] == 2 and b[2]["pre_fused"] == 0
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    assert np.array_equal(a[1], oracle.categories(plain))
    if t == L:
        assert np.array_equal(a[0], plain)
    else:
        np.testing.assert_allclose(a[0], plain, atol=ATOL, rtol=RTOL)


@pytest.mark.parametrize("N", [1024, 4096, 16384])
def test_popcount_layer0_bit_exact(N):
    """R32: layer 0 (stride 1) of a row of zeros and one value c runs as a table lookup by window count
    (k fmas of c from +0, in any order); on fp32 rows with pre_fused = 7 (and by default at N = 2048..4096), on
    packed rows by default.  Rows with c in {1, 0.3, 1.7, 0.02, YMAX, 1e-39 (subnormal)},
    all-zero rows, and rows with two different non-zero values (fma chains): the uncompressed outputs equal
    the oracle's and the run without R32 (pre_fused = 2 / 6) bit for bit; stats.pre_popc_rows counts
    exactly the two-valued rows; the packed path (binary) runs every row through it."""
    L = 9
    B = 70 if N <= 4096 else 21
    net = sdgc.gen_network(N, L, "radix")
    rs = np.random.RandomState(N)
    Y0 = (rs.uniform(size=(B, N)) < 0.3).astype(np.float32)
    cs = [1.0, 0.3, 1.7, 0.02, 32.0, 1e-39]
    for r in range(B):
        if r % 7 < len(cs):
            Y0[r] *= np.float32(cs[r % 7])
    Y0[6::7] = 0.0
    Y0[3::14, 5] = np.float32(0.5)  # a second non-zero value: not two-valued (c = 0.02 rows)
    two_valued = np.array([len(np.unique(y[y != 0])) <= 1 for y in Y0])
    assert 0 < two_valued.sum() < B
    plain = oracle.layers_f32(net, Y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        Y1, c1, st1 = _infer(g, Y0, L, pre_fused=7)  # R32 on fp32 rows too
        assert st1["pre_fused"] == 1 and st1["pre_popc_rows"] == int(two_valued.sum())
        assert np.array_equal(Y1, plain) and np.array_equal(c1, oracle.categories(plain))
        for pf in (1, 2, 6):  # 1: R32 on fp32 rows too at N = 2048..4096 (several CTAs per SM), else packed only
            Y2, c2, st2 = _infer(g, Y0, L, pre_fused=pf)
            want = int(two_valued.sum()) if (pf == 1 and 2048 <= N <= 4096) else 0
            assert st2["pre_popc_rows"] == want and np.array_equal(Y2, plain), pf
        # SNICIT path (t < L) agrees with the per-layer pre phase
        Y3, c3, _ = _infer(g, Y0, 4, pre_fused=7)
        Y4, c4, _ = _infer(g, Y0, 4, pre_fused=0)
        assert np.array_equal(Y3, Y4) and np.array_equal(c3, c4)
        # packed binary rows: every row takes R32, outputs equal the fp32 binary rows'
        Yb = (Y0 != 0).astype(np.float32)
        bits = torch.from_numpy(pack_rows(Yb).view(np.int32)).cuda()
        outp = torch.empty((B, N), dtype=torch.float32, device="cuda")
        g.infer_packed(bits, t=L, s=32, y_out=outp)
        stp = g.stats()
        assert stp["pre_popc_rows"] == B
        assert np.array_equal(outp.cpu().numpy(), oracle.layers_f32(net, Yb))


def test_dynamics_log(tmp_path):
    """snicit_dynamics (SURVEY 5 per-layer log) of the row-resident kernel.  Without the range rules
    (pre_fused = 6) it is modelled row by row on the oracle's layer-by-layer rows: pre_full[l] = rows not
    yet constant (R26) before layer l, pre_live[l] = rows with a non-zero output after layer l (all-zero
    rows drop at once, R23).  With them (default: R30 / R31 drop a row at the layer by which its range
    proves Y(t)), fewer rows are evaluated in full, pre_live counts rows not yet proven zero (>= the
    non-zero rows) and is exact after layer t - 1.  res_alive ends at stats.residual_final and never
    increases (zero residues are absorbing, R16)."""
    N, L, B, t = 1024, 40, 600, 6
    net = sdgc.gen_network(N, L, "radix")
    Y0 = sdgc.gen_inputs(N, B)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        _infer(g, Y0, t, timing=1, pre_fused=6)
        d6 = g.dynamics()
        _infer(g, Y0, t, timing=1)
        d = g.dynamics()
        st = g.stats()
        nlines = g.write_dynamics_jsonl(str(tmp_path / "dyn.jsonl"))
    y = Y0.copy()
    const_before = np.zeros(B, bool)
    alive = np.ones(B, bool)
    for l in range(t):
        full = alive & ~const_before
        assert d6["pre_full"][l] == int(full.sum()), l
        y = oracle.layers_f32(net, y, l, l + 1)
        alive = alive & (y != 0).any(1)
        assert d6["pre_live"][l] == int(alive.sum()), l
        assert d["pre_live"][l] >= int(alive.sum()), l
        assert d["pre_full"][l] <= d6["pre_full"][l], l
        const_before = const_before | (alive & (y == y[:, :1]).all(1))
    assert d["pre_live"][t - 1] == int(alive.sum())
    assert sum(d["pre_full"][:t]) < sum(d6["pre_full"][:t])  # the range rules fire on this workload
    ra = d["res_alive"][t:]
    assert ra[-1] == st["residual_final"] and np.all(np.diff(ra) <= 0) and ra[0] <= st["residual_at_t"]
    assert np.all(d["pre_full"][t:] == -1) and np.all(d["res_alive"][:t] == -1)
    lines = open(tmp_path / "dyn.jsonl").read().splitlines()
    assert nlines == len(lines) == L + 1
    assert json.loads(lines[1])["phase"] == "pre" and json.loads(lines[-1])["phase"] == "post"
