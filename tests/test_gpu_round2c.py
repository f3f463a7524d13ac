"""Round 2 (r02c) GPU parity: the general-CSC row-interleaved kernel (kernels_gen.cu) against
the oracle, bit-exact (Eq. 1 P:435-438 evaluated in stored order, R12), over both tile shapes (RL = 32
lanes over rows, RL = 8 quads of outputs), ragged tiles (row counts not a multiple of RL), ragged and
padded columns (K not a multiple of 4), non-uniform weights and biases, and the whole SNICIT path on
general layers (PLAIN / CENTROID / RESIDUAL epilogues)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from paper_conf_icpp_jiangh0h23_b200 import KERNEL_ELL, SnicitNetwork  # noqa: E402
from paper_conf_icpp_jiangh0h23_b200.api import gen_schedule  # noqa: E402
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


def random_k_net(N, L, K, seed, uniform=False, ymax=32.0):
    """K random distinct inputs per column in random (not sorted) chain order, per-entry weights."""
    rs = np.random.RandomState(seed)
    ptr, idx, val = [], [], []
    for l in range(L):
        ptr.extend((l * N * K + np.arange(N + 1) * K).tolist())
        for j in range(N):
            idx.extend(rs.choice(N, size=K, replace=False).tolist())
        val.extend((np.full(N * K, 0.0625) if uniform else rs.uniform(-0.3, 0.5, size=N * K)).tolist())
    bias = rs.uniform(-0.4, 0.2, size=L * N)
    return Network(N=N, L=L, ptr=np.array(ptr, np.int64), idx=np.array(idx, np.int32),
                   val=np.array(val, np.float32), bias=bias.astype(np.float32), ymax=ymax, mode="random_k")


def layer_cols(net, l):
    N = net.N
    p = net.ptr[l * (N + 1):(l + 1) * (N + 1)]
    return [net.idx[p[j]:p[j + 1]] for j in range(N)]


# (more than 256 rows: fewer go to the thread-per-output kernel, kernels_layer.cu; ragged w.r.t. every tile)
@pytest.mark.parametrize("N,K,rows,uniform", [(64, 7, 257, False), (256, 26, 289, False), (512, 32, 321, True),
                                               (1024, 30, 287, False), (2048, 32, 265, True), (4096, 32, 263, False)])
def test_gen_layer_bit_exact(N, K, rows, uniform):
    net = random_k_net(N, 2, K, seed=N + K, uniform=uniform)
    rl = gen_schedule(np.stack(layer_cols(net, 0)).astype(np.int32))[0]
    assert rl == (2 if N <= 384 else 4 if N <= 1536 else 16)
    rs = np.random.RandomState(rows)
    Y0 = rs.uniform(0, 32, size=(rows, N)).astype(np.float32)
    Y0[rs.uniform(size=Y0.shape) < 0.3] = 0.0
    with SnicitNetwork.from_network(net) as g:
        yin = torch.from_numpy(Y0).cuda()
        for l in range(net.L):
            ref = oracle.layers_f32(net, Y0, l, l + 1)
            out = torch.full_like(yin, float("nan"))
            g.debug_layer(l, yin, out, kernel=KERNEL_ELL)
            assert np.array_equal(out.cpu().numpy(), ref), f"layer {l}"


@pytest.mark.parametrize("N,mode,B,t", [(1024, "perm", 700, 6), (4096, "random", 300, 4), (256, "medium", 2500, 8)])
def test_gen_snicit_path(N, mode, B, t):
    """The whole path on general layers: pre phase (PLAIN with constant-row ranges), conversion, post phase
    (CENTROID / RESIDUAL epilogues), recovery: equal to the oracle's SNICIT pipeline bit for bit and to the
    plain oracle within tolerance; categories exact."""
    if mode == "medium":
        net = sdgc.gen_medium_network(256, 18)
        Y0 = sdgc.gen_medium_inputs(256, B)
        s, n = 128, 0
    else:
        net = sdgc.gen_network(N, 24, mode)
        Y0 = sdgc.gen_inputs(N, B)
        s, n = 32, 16
    plain = oracle.layers_f32(net, Y0)
    ref = oracle.snicit(net, Y0, t=t, s=s, n=n)
    with SnicitNetwork.from_network(net) as g:
        g.set_stream(torch.cuda.current_stream())
        y0 = torch.from_numpy(Y0).cuda()
        out = torch.empty_like(y0)
        for kern in (0, KERNEL_ELL):
            g.infer(y0, t=t, s=s, n_segments=n, y_out=out, kernel=kern)
            cats = g.categories()
            Y = out.cpu().numpy()
            assert np.array_equal(cats, oracle.categories(plain))
            assert np.array_equal(Y, ref["Y"])
            np.testing.assert_allclose(Y, plain, atol=ATOL, rtol=RTOL)
        g.infer(y0, t=net.L, s=s, n_segments=n, y_out=out)  # uncompressed: every layer through the kernel
        assert np.array_equal(out.cpu().numpy(), plain)
