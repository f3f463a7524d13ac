"""Pins for the CPU oracle (oracle/) against things other than itself: brute force, closed forms,
the paper's worked examples (tests/golden/), special cases and invariants.

Each test names the PAPER.md passage it pins.  CPU only (-m "not gpu").
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden
from workload import sdgc
from workload.sdgc import Network


# ---------------------------------------------------------------- helpers (test-only)

def tiny_random_net(N, L, K, seed, ymax=32.0, pos_bias=True):
    """A small unstructured net with random values and mixed-sign biases (generic Eq. 1)."""
    rs = np.random.RandomState(seed)
    ptr, idx, val = [0], [], []
    for l in range(L):
        for j in range(N):
            kk = rs.choice(N, size=rs.randint(0, K + 1), replace=False)  # ragged, possibly empty
            rs.shuffle(kk)  # arbitrary stored order
            idx.extend(kk.tolist())
            val.extend(rs.uniform(-0.6, 0.9, size=len(kk)).astype(np.float32).tolist())
            ptr.append(len(idx))
    # per-layer absolute ptr with N+1 entries per layer
    p = np.asarray(ptr, dtype=np.int64)
    P = np.concatenate([p[l * N:(l + 1) * N + 1] for l in range(L)])
    lo = -0.5 if pos_bias else -0.5
    hi = 0.5 if pos_bias else 0.0
    bias = rs.uniform(lo, hi, size=L * N).astype(np.float32)
    return Network(N=N, L=L, ptr=P, idx=np.asarray(idx, np.int32), val=np.asarray(val, np.float32),
                   bias=bias, ymax=ymax, mode="test")


def dense_weights(net, l):
    """Dense N x N matrix of layer l (rows = inputs k, cols = outputs j), built by scatter."""
    p, idx, val, _ = net.layer(l)
    W = np.zeros((net.N, net.N), dtype=np.float64)
    cols = np.repeat(np.arange(net.N), np.diff(p))
    np.add.at(W, (idx.astype(np.int64), cols), val.astype(np.float64))
    return W


def dense_forward_f64(net, Y0, l0=0, l1=None):
    l1 = net.L if l1 is None else l1
    Y = Y0.astype(np.float64)
    for l in range(l0, l1):
        b = net.bias[l * net.N:(l + 1) * net.N].astype(np.float64)
        Y = np.clip(Y @ dense_weights(net, l) + b, 0.0, net.ymax)
    return Y


# ---------------------------------------------------------------- Eq. (1)

@pytest.mark.parametrize("N,L,K,seed", [(16, 3, 5, 1), (37, 5, 9, 2), (64, 6, 12, 3)])
def test_plain_f64_matches_dense_matmul(N, L, K, seed):
    """Eq. (1) PAPER.md:435-438 / problem statement PAPER.md:308-312, sigma of Table 2 PAPER.md:410:
    the oracle's sparse fp64 layer loop equals a dense fp64 matmul + bias + clamp."""
    net = tiny_random_net(N, L, K, seed, ymax=2.0)
    rs = np.random.RandomState(seed + 100)
    Y0 = rs.uniform(0, 1.5, size=(11, N)).astype(np.float32)
    ref = dense_forward_f64(net, Y0)
    got = oracle.layers_f64(net, Y0)
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("N,L,K,seed", [(16, 3, 5, 4), (64, 6, 12, 5)])
def test_plain_f32_close_to_dense(N, L, K, seed):
    net = tiny_random_net(N, L, K, seed, ymax=2.0)
    Y0 = np.random.RandomState(seed).uniform(0, 1.5, size=(9, N)).astype(np.float32)
    np.testing.assert_allclose(oracle.layers_f32(net, Y0), dense_forward_f64(net, Y0), rtol=2e-6, atol=2e-6)


def test_plain_layer_range_composes():
    net = tiny_random_net(24, 6, 6, 7, ymax=3.0)
    Y0 = np.random.RandomState(1).uniform(0, 1, size=(5, 24)).astype(np.float32)
    a = oracle.layers_f32(net, oracle.layers_f32(net, Y0, 0, 2), 2, 6)
    assert np.array_equal(a, oracle.layers_f32(net, Y0))


def test_closed_form_one_layer_binary_sdgc():
    """One SDGC layer on binary input: y'_j = sigma(cnt_j / 16 + b), cnt_j = #active inputs of j
    (weights 1/16, bias Table 1, YMAX 32).  Products and partial sums are exact."""
    for N in (1024, 4096):
        net = sdgc.gen_network(N, 2, "radix")
        Y0 = sdgc.gen_inputs(N, 40)
        p, idx, val, b = net.layer(0)
        cnt = np.array([[Y0[r, idx[p[j]:p[j + 1]]].sum() for j in range(N)] for r in range(4)])
        expect = np.minimum(np.maximum(np.float32(cnt / 16.0) + b, np.float32(0)), np.float32(32))
        got = oracle.layers_f32(net, Y0[:4], 0, 1)
        assert np.array_equal(got, expect.astype(np.float32))


def test_zero_row_fixed_point_and_all_ymax_fixed_point():
    """b <= 0: sigma(W.0 + b) = 0.  SDGC constants: 32 * 32/16 - 0.45 >= 32, so the all-32 row
    is a fixed point."""
    for N in (1024, 4096):
        net = sdgc.gen_network(N, 12, "perm")
        Y = np.zeros((2, N), np.float32)
        Y[1] = 32.0
        out = oracle.layers_f32(net, Y)
        assert np.array_equal(out[0], np.zeros(N, np.float32))
        assert np.array_equal(out[1], np.full(N, 32.0, np.float32))


def test_permutation_network_is_exact_permutation():
    """w = 1, b = 0, one input per column, huge YMAX: Eq. (1) reduces to y'[j] = y[pi(j)]."""
    N, L = 50, 3
    rs = np.random.RandomState(3)
    perms = [rs.permutation(N) for _ in range(L)]
    P = np.concatenate([l * N + np.arange(N + 1, dtype=np.int64) for l in range(L)])
    net = Network(N=N, L=L, ptr=P, idx=np.concatenate(perms).astype(np.int32), val=np.ones(N * L, np.float32),
                  bias=np.zeros(N * L, np.float32), ymax=1e30, mode="test")
    Y0 = rs.uniform(0, 10, size=(6, N)).astype(np.float32)
    expect = Y0.copy()
    for l in range(L):
        expect = expect[:, perms[l]]
    assert np.array_equal(oracle.layers_f32(net, Y0), expect)


def test_table1_connections_and_bias():
    """Table 1: Connections = 32 * N * L; bias per N."""
    table = {(1024, 120): 3932160, (1024, 480): 15728640, (1024, 1920): 62914560,
             (4096, 120): 15728640, (4096, 480): 62914560, (4096, 1920): 251658240,
             (16384, 120): 62914560, (16384, 480): 251658240, (16384, 1920): 1006632960,
             (65536, 120): 251658240, (65536, 480): 1006632960, (65536, 1920): 4026531840}
    for (N, L), c in table.items():
        assert 32 * N * L == c
    for N, L in ((1024, 120), (4096, 8)):
        net = sdgc.gen_network(N, L)
        assert net.nnz == 32 * N * L
        assert np.all(net.bias == np.float32(sdgc.SDGC_BIAS[N]))
        assert np.all(net.val == np.float32(1 / 16))
    assert sdgc.SDGC_BIAS == {1024: -0.3, 4096: -0.35, 16384: -0.4, 65536: -0.45}


def test_f32_oracle_agrees_with_f64_definition_on_c1_sample():
    net = sdgc.gen_network(1024, 120)
    Y0 = sdgc.gen_inputs(1024, 150)
    a = oracle.layers_f32(net, Y0)
    b = oracle.layers_f64(net, Y0)
    assert np.array_equal((a != 0).any(1), (b != 0).any(1))
    np.testing.assert_allclose(a, b, atol=1e-4, rtol=1e-5)
    assert a.min() >= 0 and a.max() <= 32  # range invariant, north star


# ---------------------------------------------------------------- sum downsampling

def test_downsample_matches_segment_sums():
    """F = per-segment sums of the first s rows (Fig. 3a)."""
    rs = np.random.RandomState(0)
    rows = rs.randint(0, 33, size=(7, 64)).astype(np.float32)  # integers: sums are exact
    F = oracle.sum_downsample(rows, 16)
    assert F.shape == (16, 7)
    assert np.array_equal(F, rows.reshape(7, 16, 4).sum(-1).T.astype(np.float64))
    # ragged: N = 37, n = 5 -> segments of 7, last takes the remainder (reading R15)
    rows = rs.randint(0, 5, size=(3, 37)).astype(np.float32)
    F = oracle.sum_downsample(rows, 5)
    bounds = [0, 7, 14, 21, 28, 37]
    ref = np.stack([rows[:, bounds[g]:bounds[g + 1]].sum(1) for g in range(5)])
    assert np.array_equal(F, ref)
    # n = 0: no downsampling (medium nets), F = rows^T
    assert np.array_equal(oracle.sum_downsample(rows, 0), rows.T.astype(np.float64))


# ---------------------------------------------------------------- Alg. 1

def test_prune_fig3b_worked_example():
    g = read_golden("fig3b_prune.txt")
    eta, eps = float(g[0][0]), float(g[0][1])
    F = np.array([[float(x) for x in r] for r in g[1:5]])
    after_first = np.array([int(x) for x in g[5]])
    final = np.array([int(x) for x in g[6]])
    # first iteration only: prune with column 0 as the only possible base -> restrict to base col 0
    ci = oracle.prune(F, eta, eps)
    assert np.array_equal(ci, final)
    # the intermediate state: columns similar to col 0 are exactly {1, 3}
    sim0 = [q for q in range(1, 6) if (np.abs(F[:, q] - F[:, 0]) > eta).sum() < F.shape[0] * eps]
    assert [q for q in range(6) if after_first[q] == -1] == sim0 == [1, 3]


def _similar(F, a, b, eta, eps):
    return (np.abs(F[:, a] - F[:, b]) > eta).sum() < F.shape[0] * eps


@pytest.mark.parametrize("seed", range(6))
def test_prune_is_greedy_leader_clustering(seed):
    """Alg. 1 with Eq. (2) is characterised by: (a) no survivor is similar to an earlier survivor;
    (b) every pruned column is similar to some earlier survivor.  (a)+(b) determine the result."""
    rs = np.random.RandomState(seed)
    n, s = 5, 40
    centers = rs.randint(0, 6, size=(n, 7)).astype(np.float64)
    F = centers[:, rs.randint(0, 7, size=s)] + rs.choice([0, 0, 0.01, 0.5], size=(n, s))
    for eta, eps in ((0.03, 0.03), (0.2, 0.3), (0.6, 0.5)):
        ci = oracle.prune(F, eta, eps)
        surv = [q for q in range(s) if ci[q] != -1]
        assert surv[0] == 0
        for i, a in enumerate(surv):
            assert ci[a] == a
            for b in surv[:i]:
                assert not _similar(F, a, b, eta, eps)
        for q in range(s):
            if ci[q] == -1:
                assert any(_similar(F, q, a, eta, eps) for a in surv if a < q)


def test_prune_limits():
    F = np.random.RandomState(1).uniform(0, 10, size=(4, 9))
    assert np.array_equal(oracle.prune(F, 1e9, 0.03), np.array([0] + [-1] * 8))  # all similar
    assert np.array_equal(oracle.prune(F, -1.0, 0.03), np.arange(9))  # nothing similar
    # n*eps = 2.4: columns differing in <= 2 segments are pruned (Eq. 2 'diff < n eps')
    G = np.zeros((4, 3))
    G[:2, 1] = 5.0  # col 1 differs from col 0 in 2 segments -> pruned
    G[:3, 2] = 5.0  # col 2 differs from col 0 in 3 segments, from col 1 in 1 -> survives col 0
    assert np.array_equal(oracle.prune(G, 0.03, 0.6), np.array([0, -1, 2]))


# ---------------------------------------------------------------- Eq. (3)-(4), Alg. 2

@pytest.mark.parametrize("seed", range(4))
def test_map_residual_brute_force(seed):
    rs = np.random.RandomState(seed)
    R, N = 30, 12
    Y = rs.choice([0.0, 0.5, 32.0], size=(R, N)).astype(np.float32)
    Y[5] = Y[3]  # duplicates (distance 0)
    live = rs.rand(R) > 0.15
    live[[3, 8]] = True
    cent = np.array(sorted(rs.choice(np.nonzero(live)[0], size=4, replace=False)), np.int32)
    M, Yhat, ne = oracle.map_residual(Y, cent, live.astype(np.uint8))
    dist = (Y[:, None, :] != Y[cent][None, :, :]).sum(-1)  # L0 distances
    for r in range(R):
        if not live[r]:
            assert M[r] == -2 and ne[r] == 0
        elif r in cent:
            assert M[r] == -1 and ne[r] == 1 and np.array_equal(Yhat[r], Y[r])
        else:
            c = cent[np.argmin(dist[r])]  # argmin returns the first minimum (reading R6)
            assert M[r] == c
            assert np.array_equal(Yhat[r], Y[r] - Y[c])
            assert ne[r] == (dist[r].min() != 0)
    # Eq. (6) reverses Eq. (4) exactly on these values
    Yrec, cat = oracle.recover(M, ne, Yhat)
    for r in range(R):
        if live[r]:
            assert np.array_equal(Yrec[r], Y[r])
            assert cat[r] == (Y[r] != 0).any()
        else:
            assert not Yrec[r].any() and cat[r] == 0


def test_eq4_eq6_round_trip_within_one_ulp():
    rs = np.random.RandomState(9)
    Y = rs.uniform(0, 32, size=(20, 50)).astype(np.float32)
    M, Yhat, ne = oracle.map_residual(Y, np.array([0, 7], np.int32))
    Yrec, _ = oracle.recover(M, ne, Yhat)
    Yc = Y[np.where(M >= 0, M, np.arange(20))]
    ulp = np.spacing(np.maximum(np.abs(Y), np.abs(Yc)).astype(np.float32))  # 1 ulp of the operands
    assert np.all(np.abs(Yrec - Y) <= ulp)
    assert np.mean(Yrec == Y) > 0.5


# ---------------------------------------------------------------- Eq. (5), Alg. 3

def test_absorbing_zero_residual_fp32():
    """sigma((a + 0) + b) - sigma(a + b) == 0 exactly in fp32: a zero residual stays zero (R16)."""
    rs = np.random.RandomState(0)
    a = rs.uniform(-40, 40, size=10 ** 6).astype(np.float32)
    b = rs.uniform(-1, 1, size=10 ** 6).astype(np.float32)
    sig = lambda x: np.minimum(np.maximum(x, np.float32(0)), np.float32(32))
    v = sig((a + np.float32(0)) + b) - sig(a + b)
    assert not v.any()


def test_post_layer_fig5_example():
    g = read_golden("fig5_ne.txt")
    ne_before = [int(x) for x in g[0]]
    ne_after = np.array([x == "T" for x in g[1]])
    cent = [int(x) for x in g[2]]
    B, N = 16, 4
    # identity layer: output j reads input j with weight 1, bias 0, YMAX 32
    net = Network(N=N, L=1, ptr=np.arange(N + 1, dtype=np.int64), idx=np.arange(N, dtype=np.int32),
                  val=np.ones(N, np.float32), bias=np.zeros(N, np.float32), ymax=32.0, mode="test")
    Yhat = np.zeros((B, N), np.float32)
    M = np.full(B, cent[0], np.int32)
    Yhat[cent[0]] = 32.0  # saturated centroid
    Yhat[cent[1]] = 10.0
    Yhat[cent[2]] = 5.0
    Yhat[cent[3]] = 1.0
    M[cent] = -1
    ne = np.zeros(B, np.uint8)
    ne[ne_before] = 1
    for r in ne_before:
        if r in cent:
            continue
        if r == 8:
            M[r] = cent[0]
            Yhat[r] = [1.0, 2.0, 0.0, 0.5]  # pushes a saturated centroid further: residual vanishes
        else:
            M[r] = cent[1]
            Yhat[r] = [1.0, 0.0, 0.0, 0.0]
    out, ne2 = oracle.post_layer(net, 0, M, Yhat, ne)
    assert np.array_equal(ne2.astype(bool), ne_after)
    assert list(np.nonzero(ne2)[0]) == [0, 1, 2, 5, 6, 11, 12, 14, 15]


def _c1_small(N=1024, L=24, B=300, mode="radix"):
    return sdgc.gen_network(N, L, mode), sdgc.gen_inputs(N, B)


@pytest.mark.parametrize("t", [0, 2, 5, 9, 16])
def test_snicit_reconstructs_plain_result(t):
    """Eq. (4)-(6) telescoping: for any centroids and M, Eq. (6) returns Y(l) in real
    arithmetic.  In fp32: categories identical, activations within 1e-4 abs / 1e-5 rel."""
    net, Y0 = _c1_small()
    plain = oracle.layers_f32(net, Y0)
    res = oracle.snicit(net, Y0, t=t, s=32, n=16)
    assert np.array_equal(res["categories"], oracle.categories(plain))
    np.testing.assert_allclose(res["Y"], plain, atol=1e-4, rtol=1e-5)
    assert res["Y"].min() >= 0 and res["Y"].max() <= 32
    assert len(res["cent"]) >= 1


def test_snicit_reconstruction_invariant_every_layer():
    """At every post-convergence layer, Yhat_r + Yhat_M(r) equals the plain activation (within fp32
    tolerance) -- the per-layer form of the telescoping identity for Eq. (5)."""
    net, Y0 = _c1_small(N=1024, L=14, B=120)
    t = 3
    Yt = oracle.layers_f32(net, Y0, 0, t)
    live = (Yt != 0).any(1)
    sample = np.nonzero(live)[0][:32]
    ci = oracle.prune(oracle.sum_downsample(Yt[sample], 16), 0.03, 0.03)
    cent = np.sort(sample[ci != -1]).astype(np.int32)
    M, Yhat, ne = oracle.map_residual(Yt, cent, live.astype(np.uint8))
    Yplain = Yt
    for l in range(t, net.L):
        Yhat, ne = oracle.post_layer(net, l, M, Yhat, ne, out=Yhat.copy() * 0)
        Yplain = oracle.layers_f32(net, Yplain, l, l + 1)
        rec, _ = oracle.recover(M, ne, Yhat)
        np.testing.assert_allclose(rec[live], Yplain[live], atol=1e-4, rtol=1e-5)
        assert np.all(np.abs(Yhat[ne.astype(bool) & (M >= 0)]) <= 32)


def test_snicit_special_cases_bit_exact():
    net, Y0 = _c1_small(L=16, B=200)
    plain = oracle.layers_f32(net, Y0)
    # t >= L: no conversion -> the plain path exactly
    assert np.array_equal(oracle.snicit(net, Y0, t=net.L)["Y"], plain)
    # s = B, eta < 0 never prunes ... eta = 0 with n = 0 prunes exact duplicates only: every row maps
    # to an identical centroid, all residuals are zero -> bit-exact
    res = oracle.snicit(net, Y0, t=4, s=200, n=0, eta=0.0, eps=1e-6)
    assert np.array_equal(res["Y"], plain)
    assert not res["ne"][res["M"] >= 0].any()


def test_snicit_without_dead_row_drop_matches():
    net, Y0 = _c1_small(L=20, B=150)
    a = oracle.snicit(net, Y0, t=6, drop_dead=True)
    b = oracle.snicit(net, Y0, t=6, drop_dead=False)
    assert np.array_equal(a["categories"], b["categories"])
    np.testing.assert_allclose(a["Y"], b["Y"], atol=1e-4, rtol=1e-5)


def test_medium_net_snicit_vs_plain():
    """Config 5 stand-in: YMAX 1, per-neuron bias (some > 0 -> no dead-row drop),
    no downsampling, s = 128."""
    net = sdgc.gen_medium_network(256, 18)
    Y0 = sdgc.gen_medium_inputs(256, 400)
    plain = oracle.layers_f32(net, Y0)
    res = oracle.snicit(net, Y0, t=sdgc.medium_t(18), s=128, n=0)
    assert np.array_equal(res["categories"], oracle.categories(plain))
    np.testing.assert_allclose(res["Y"], plain, atol=1e-4, rtol=1e-5)
    assert plain.max() <= 1.0


def test_circulant_form_equals_csc():
    """The compact circulant network is the radix CSC network, and the oracle's circulant-form layer
    loop equals its CSC layer loop bit for bit (same definition, same fma order)."""
    for N, L in ((1024, 6), (4096, 4)):
        c = sdgc.gen_circulant(N, L)
        net = sdgc.gen_network(N, L, "radix")
        e = c.to_network()
        assert np.array_equal(e.ptr, net.ptr) and np.array_equal(e.idx, net.idx) and np.array_equal(e.val, net.val)
        assert c.nnz == net.nnz
        Y0 = sdgc.gen_inputs(N, 7) * np.float32(3.3)
        assert np.array_equal(oracle.layers_circulant_f32(c, Y0), oracle.layers_f32(net, Y0))


# ---------------------------------------------------------------- exact fast mode

def _same(a, b):
    """Equal under == (reading R19: +0 == -0) -- the comparison every parity test uses."""
    return a.shape == b.shape and bool(np.all(a == b))


@pytest.mark.parametrize("N,L,B", [(1024, 120, 2000)])
def test_fast_oracle_equals_plain_c1(N, L, B):
    """Fast mode == plain Eq. (1) on the whole C1 workload (SDGC 1024 x 120, B = 2000), and it skips most
    row-layers there (rows collapse to all-0 / all-32)."""
    net = sdgc.gen_network(N, L, "radix")
    Y0 = sdgc.gen_inputs(N, B)
    plain = oracle.layers_f32(net, Y0)
    fast, skipped = oracle.layers_f32_fast(net, Y0, return_skipped=True)
    assert _same(fast, plain)
    assert skipped > 0.5 * B * L


def test_fast_oracle_equals_plain_c2_rows_and_compact_form():
    """C2 (4096 x 480) on a row sample, through the CSC and the compact circulant forms."""
    cn = sdgc.gen_circulant(4096, 480)
    rs = np.random.RandomState(11)
    rows = np.sort(rs.choice(60000, 48, replace=False))
    Y0 = np.concatenate([sdgc.gen_inputs(4096, 1, row0=int(r)) for r in rows])
    plain = oracle.layers_circulant_f32(cn, Y0)
    assert _same(oracle.layers_f32_fast(cn, Y0), plain)
    assert _same(oracle.layers_f32_fast(cn.to_network(), Y0), plain)


def test_fast_oracle_degenerate_rows_and_non_fixed_layers():
    """All-zero, all-YMAX, constant and random rows; layers where the zero row is NOT a fixed point
    (positive biases) and where YMAX is not (negative weights): fast == plain, bit for bit under ==."""
    N, L = 64, 9
    net = tiny_random_net(N, L, 12, 5)
    rs = np.random.RandomState(2)
    Y0 = rs.uniform(0, 32, size=(40, N)).astype(np.float32)
    Y0[0::5] = 0.0
    Y0[1::5] = 32.0
    Y0[2::5] = -0.0
    Y0[3::5] = 7.25
    assert _same(oracle.layers_f32_fast(net, Y0), oracle.layers_f32(net, Y0))
    # SDGC layers with one positive-bias layer in the middle (zero rows wake up there)
    c = sdgc.gen_circulant(1024, 12)
    c.bias[5 * 1024:6 * 1024] = 0.25
    Y1 = sdgc.gen_inputs(1024, 300)
    Y1[::3] = 0.0
    assert _same(oracle.layers_f32_fast(c, Y1), oracle.layers_circulant_f32(c, Y1))
    out6 = oracle.layers_f32_fast(c, Y1, 0, 6)
    assert _same(out6, oracle.layers_circulant_f32(c, Y1, 0, 6))
    assert (out6[::3] == np.float32(0.25)).all()  # the zero rows were evaluated by the positive-bias layer


def test_fast_oracle_equals_plain_c3_rows():
    """C3 geometry (16384 x 1920, compact form) on a few rows: fast == plain."""
    cn = sdgc.gen_circulant(16384, 1920)
    Y0 = np.concatenate([sdgc.gen_inputs(16384, 1, row0=r) for r in (0, 1, 7, 59999)])
    assert _same(oracle.layers_f32_fast(cn, Y0), oracle.layers_circulant_f32(cn, Y0))
