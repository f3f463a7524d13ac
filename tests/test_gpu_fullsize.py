"""Full-size parity (round 2): the CUDA path at BASELINE.json's full sizes, in bench.py's launch
configuration, against the CPU oracle on EVERY row (C2, C3) or on a fixed quarter of the rows (C4).

The oracle side is the exact fast mode of Eq. 1 (oracle.layers_f32_fast: memoised all-0 / all-YMAX
fixed points), which tests/test_oracle_pins.py pins bit-identical to the plain mode
on C1, C2 rows, C3 rows and degenerate nets; a sample of rows is also checked against the plain oracle
here.  Bars (north_star): the category set bit-exact; activations within 1e-4 abs or 1e-5 rel.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork, pack_rows  # noqa: E402
from workload import sdgc  # noqa: E402

pytestmark = pytest.mark.gpu

ATOL, RTOL = 1e-4, 1e-5
CHUNK = 4000


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_jiangh0h23_b200 import build
    build.build()


def _inputs_device(N, B):
    """The seeded SDGC inputs of rows [0, B) generated chunk-wise straight into one device tensor."""
    y0 = torch.empty((B, N), dtype=torch.float32, device="cuda")
    for a in range(0, B, CHUNK):
        b = min(B, a + CHUNK)
        y0[a:b].copy_(torch.from_numpy(sdgc.gen_inputs(N, b - a, row0=a)))
    return y0


def _check_rows(net, Yd, rows, label):
    """Oracle (fast mode) on `rows` (ascending ids) vs the device activations Yd[rows]; returns the
    oracle's category ids among `rows`."""
    cats = []
    N = net.N
    for a in range(0, len(rows), CHUNK):
        rr = rows[a:a + CHUNK]
        if len(rr) and rr[-1] - rr[0] == len(rr) - 1:  # contiguous block
            Y0 = sdgc.gen_inputs(N, len(rr), row0=int(rr[0]))
            got = Yd[int(rr[0]):int(rr[-1]) + 1].cpu().numpy()
        else:
            Y0 = np.concatenate([sdgc.gen_inputs(N, 1, row0=int(r)) for r in rr])
            got = Yd[torch.from_numpy(np.asarray(rr, np.int64)).cuda()].cpu().numpy()
        ref = oracle.layers_f32_fast(net, Y0)
        np.testing.assert_allclose(got, ref, atol=ATOL, rtol=RTOL, err_msg=f"{label} rows {rr[0]}..{rr[-1]}")
        cats.append(np.asarray(rr)[(ref != 0).any(1)])
    return np.concatenate(cats) if cats else np.zeros(0, np.int64)


def test_full_c2_every_row():
    """C2 (SDGC 4096 x 480, B = 60000, t = 30, s = 32, n = 16) through the CSC loader: the whole category
    set and all 60000 x 4096 activations against the oracle; 2000 rows also against the plain oracle."""
    c = sdgc.CONFIGS["C2"]
    N, L, B = c["N"], c["L"], c["B"]
    net = sdgc.gen_network(N, L, "radix")
    y0 = _inputs_device(N, B)
    out = torch.empty_like(y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(y0, t=30, s=32, y_out=out)
        cats = g.categories()
        st = g.stats()
    del y0
    ref_cats = _check_rows(net, out, np.arange(B), "C2")
    assert np.array_equal(cats, ref_cats)
    assert st["n_categories"] == len(cats)
    # plain oracle (no memoisation) on 2000 spread rows
    rs = np.random.RandomState(3)
    sample = np.sort(rs.choice(B, 2000, replace=False))
    Y0s = np.concatenate([sdgc.gen_inputs(N, 1, row0=int(r)) for r in sample])
    plain = oracle.layers_f32(net, Y0s)
    np.testing.assert_allclose(out[torch.from_numpy(sample).cuda()].cpu().numpy(), plain, atol=ATOL, rtol=RTOL)


def test_full_c3_every_row():
    """C3 (SDGC 16384 x 1920, B = 60000, t = 30) through the compact circulant loader, bench.py's
    configuration: the whole category set and every row's activations against the oracle (compact
    form); 8 rows also against the plain oracle."""
    c = sdgc.CONFIGS["C3"]
    N, L, B = c["N"], c["L"], c["B"]
    cn = sdgc.gen_circulant(N, L)
    y0 = _inputs_device(N, B)
    out = torch.empty_like(y0)
    with SnicitNetwork.circulant(cn.N, cn.L, cn.nu, cn.w, cn.bias, cn.ymax) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(y0, t=30, s=32, y_out=out)
        cats = g.categories()
        st = g.stats()
    del y0
    assert float(out.min()) >= 0.0 and float(out.max()) <= 32.0
    ref_cats = _check_rows(cn, out, np.arange(B), "C3")
    assert np.array_equal(cats, ref_cats)
    assert st["n_categories"] == len(cats)
    sample = np.array([0, 1, 2, 12345, 30000, 45678, 59998, 59999])
    Y0s = np.concatenate([sdgc.gen_inputs(N, 1, row0=int(r)) for r in sample])
    np.testing.assert_allclose(out[torch.from_numpy(sample).cuda()].cpu().numpy(),
                               oracle.layers_circulant_f32(cn, Y0s), atol=ATOL, rtol=RTOL)


@pytest.mark.parametrize("pf,step", [(1, 4), (0, 16)])
def test_c4_quarter_rows_packed(pf, step):
    """C4 (SDGC 65536 x 1920, B = 60000, t = 30) through the compact loader and the packed-input call, with
    the default pre phase (pf = 1: a row split over an 8-CTA cluster, R26/R30/R31) and the per-layer
    kernels (pf = 0): every `step`-th row against the oracle, and at every size the category set = the
    non-zero rows of the returned activations."""
    c = sdgc.CONFIGS["C4"]
    N, L, B = c["N"], c["L"], c["B"]
    cn = sdgc.gen_circulant(N, L)
    bits = np.concatenate([pack_rows(sdgc.gen_inputs(N, 2000, row0=a)) for a in range(0, B, 2000)])
    with SnicitNetwork.circulant(cn.N, cn.L, cn.nu, cn.w, cn.bias, cn.ymax) as g:
        g.set_stream(torch.cuda.current_stream())
        out = torch.empty((B, N), dtype=torch.float32, device="cuda")
        g.infer_packed(torch.from_numpy(bits.view(np.int32)).cuda(), t=30, s=32, y_out=out, pre_fused=pf)
        assert g.stats()["pre_fused"] == (2 if pf else 0)
        cats = g.categories()
        nzrows = torch.nonzero((out != 0).any(1)).flatten().cpu().numpy()
        rows = np.arange(0, B, step)
        ref_cats = _check_rows(cn, out, rows, "C4")
        del out
    assert np.array_equal(cats, nzrows)
    assert np.array_equal(np.intersect1d(cats, rows), ref_cats)


def test_full_c2_perm_every_row():
    """C2 with "perm" weights (general CSC: the row-interleaved kernel of kernels_gen.cu, G = 16 quads under
    the load-time schedule; bench.py's general_csc line) at B = 60000, t = 30: the whole category set and
    every activation against the oracle (fast mode), 1000 rows against the plain oracle."""
    c = sdgc.CONFIGS["C2"]
    N, L, B = c["N"], c["L"], c["B"]
    net = sdgc.gen_network(N, L, "perm")
    y0 = _inputs_device(N, B)
    out = torch.empty_like(y0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        g.infer(y0, t=30, s=32, y_out=out)
        cats = g.categories()
        st = g.stats()
    del y0
    assert st["circ_layers"] == 0
    ref_cats = _check_rows(net, out, np.arange(B), "C2 perm")
    assert np.array_equal(cats, ref_cats)
    rs = np.random.RandomState(5)
    sample = np.sort(rs.choice(B, 1000, replace=False))
    Y0s = np.concatenate([sdgc.gen_inputs(N, 1, row0=int(r)) for r in sample])
    plain = oracle.layers_f32(net, Y0s)
    np.testing.assert_allclose(out[torch.from_numpy(sample).cuda()].cpu().numpy(), plain, atol=ATOL, rtol=RTOL)


def test_full_c5_every_row():
    """Config 5 (medium MLP 256 x 18, per-entry weights, B = 60000; bench.py's C5 line: t = 8, s = 128,
    n = N): the GPU SNICIT path (general-CSC kernel G = 2 in the pre phase and, per layer, in the post
    phase; Alg. 1 from precomputed pair counts) equals the oracle's SNICIT pipeline bit for bit and the
    plain oracle within tolerance on every row; categories exact; the uncompressed path is bit-exact."""
    c = sdgc.CONFIGS["C5"]
    N, L, B = c["N"], c["L"], c["B"]
    net = sdgc.gen_medium_network(N, L)
    Y0 = sdgc.gen_medium_inputs(N, B)
    t = sdgc.medium_t(L)
    plain = oracle.layers_f32(net, Y0)
    ref = oracle.snicit(net, Y0, t=t, s=128, n=0)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        y0 = torch.from_numpy(Y0).cuda()
        out = torch.empty_like(y0)
        g.infer(y0, t=t, s=128, n_segments=0, y_out=out)
        cats = g.categories()
        Y = out.cpu().numpy()
        assert np.array_equal(Y, ref["Y"])
        np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)
        assert np.array_equal(cats, oracle.categories(plain))
        g.infer(y0, t=L, s=128, n_segments=0, y_out=out)
        assert np.array_equal(out.cpu().numpy(), plain)
