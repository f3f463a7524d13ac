"""The C-ABI library (no GPU needed): it loads, exports every symbol include/snicit.h declares, and
its host-side argument validation reports bad input with the documented status codes."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_icpp_jiangh0h23_b200 as pkg
from paper_conf_icpp_jiangh0h23_b200 import _lib
from paper_conf_icpp_jiangh0h23_b200 import build as pkg_build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    pkg_build.build()
    return _lib.load_library()


def header_functions():
    src = open(os.path.join(ROOT, "include", "snicit.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(snicit_[a-z_]+)\s*\(", src)))


def test_header_symbols_exported(lib):
    names = header_functions()
    assert "snicit_infer" in names and "snicit_load_network" in names and "snicit_categories" in names
    for n in names:
        assert hasattr(lib, n), f"{n} declared in include/snicit.h but not exported"
    assert sorted(_lib.EXPORTED) == names


def test_abi_version_and_defaults(lib):
    assert lib.snicit_abi_version() == 6
    o = _lib.default_options()
    # SDGC defaults, P:1038 / P:1138
    assert o.n_segments == 16 and abs(o.eta - 0.03) < 1e-7 and abs(o.eps - 0.03) < 1e-7
    assert o.prune_eps == 0.0 and o.drop_dead_rows == 1 and o.kernel == 0 and o.ne_interval == 64
    assert o.post_const == 1 and o.pre_fused == 1 and o.pre_const == 1
    assert ctypes.sizeof(_lib.Options) == 60 and ctypes.sizeof(_lib.Stats) == 200


def _load(lib, N, L, ptr, idx, val, bias, ymax=32.0, fmt=0):
    h = ctypes.c_void_p()
    ptr = np.ascontiguousarray(ptr, np.int64)
    idx = np.ascontiguousarray(idx, np.int32)
    val = np.ascontiguousarray(val, np.float32)
    bias = np.ascontiguousarray(bias, np.float32)
    st = lib.snicit_load_network(N, L, fmt, ptr.ctypes.data, idx.ctypes.data, val.ctypes.data, bias.ctypes.data,
                                 ymax, 0, ctypes.byref(h))
    if st == 0:
        lib.snicit_free_network(h)
    return st


def test_validation_codes(lib):
    N = 8
    ptr = np.arange(N + 1) * 2
    idx = np.array([(j + d) % N for j in range(N) for d in (0, 1)])
    val = np.full(2 * N, 0.5)
    bias = np.zeros(N)
    bad = idx.copy()
    bad[3] = N  # out of range
    assert _load(lib, N, 1, ptr, bad, val, bias) == -2
    dup = idx.copy()
    dup[1] = dup[0]  # duplicate input in column 0
    assert _load(lib, N, 1, ptr, dup, val, bias) == -2
    nonmono = ptr.copy()
    nonmono[2], nonmono[3] = nonmono[3], nonmono[2]
    assert _load(lib, N, 1, nonmono, idx, val, bias) == -2
    nan = val.copy()
    nan[0] = np.nan
    assert _load(lib, N, 1, ptr, idx, nan, bias) == -1
    assert _load(lib, N, 1, ptr, idx, val, bias, ymax=-1.0) == -1
    assert _load(lib, 6, 1, np.arange(7) * 0, idx[:0], val[:0], np.zeros(6)) == -6  # N % 4 != 0
    # a valid network: without a GPU the library reports E_CUDA (never a CPU fallback)
    st = _load(lib, N, 1, ptr, idx, val, bias)
    try:
        import torch
        has_gpu = torch.cuda.is_available()
    except Exception:
        has_gpu = False
    assert st == (0 if has_gpu else -4)
    assert lib.snicit_last_error() is not None


def test_null_handle_errors(lib):
    n = ctypes.c_int64(0)
    assert lib.snicit_categories(None, None, ctypes.byref(n), 0) == -1
    assert lib.snicit_infer(None, None, 0, 0, 0, 0, 1, None, None, 0) == -1
    assert lib.snicit_infer_packed(None, None, 0, 0, 1.0, 0, 0, 1, None, None, 0) == -1
    lib.snicit_free_network(None)  # no-op


def test_package_exports():
    assert callable(pkg.SnicitNetwork) and callable(pkg.shard_rows)
    assert pkg.shard_rows(10, 3, 0) == (0, 4) and pkg.shard_rows(10, 3, 2) == (7, 10)


@pytest.mark.parametrize("b0,kmax", [(-0.3, 32), (-0.4, 32), (-0.45, 12), (0.05, 8), (-40.0, 4)])
def test_range_tables_match_reference(b0, kmax):
    """R30 horizon tables computed by the library (composition: hi[k] = least v with out(v) >= hi[k-1])
    equal an independent direct iteration of out^k (tests/range_ref.py), bit for bit; hi non-increasing,
    lo non-decreasing, never overlapping; inactive tables are +inf / -1."""
    from paper_conf_icpp_jiangh0h23_b200 import range_tables
    from range_ref import range_thresholds
    w0, ymax = 1.0 / 16.0, 32.0
    hi, lo, active = range_tables(w0, b0, ymax, kmax)
    rhi, rlo = range_thresholds(w0, b0, ymax, kmax)
    assert active
    assert np.array_equal(hi, np.array(rhi, np.float32)) and np.array_equal(lo, np.array(rlo, np.float32))
    assert np.all(hi[1:] <= hi[:-1]) and np.all(lo[1:] >= lo[:-1]) and np.all(lo < hi)
    if b0 > 0:
        assert np.all(lo == -1.0)  # out(0) = b0 > 0: no row is ever proven zero
    if b0 == -0.3:  # out(v) = 2v - 0.3: one layer saturates from (32 + 0.3)/2 and zeroes up to 0.15
        assert abs(hi[0] - 16.15) < 1e-5 and abs(lo[0] - 0.15) < 1e-6
        assert abs(hi[-1] - 0.3) < 1e-5 and abs(lo[-1] - 0.3) < 1e-5  # both close in on v* = -b0
    if b0 == -40.0:  # out(v) = 2v - 40 < 32 on [0, 32]: no row reaches YMAX; zero after k layers from
        assert np.all(np.isinf(hi)) and list(lo) == [20.0, 30.0, 32.0, 32.0]  # v <= 40 - 40/2^k (capped)


def test_range_tables_rejects_bad_args():
    from paper_conf_icpp_jiangh0h23_b200 import range_tables
    with pytest.raises(Exception):
        range_tables(0.0625, -0.3, 32.0, 33)
    assert not range_tables(-0.0625, -0.3, 32.0, 4)[2]  # w0 < 0: outputs not monotone, tables off


def _quad_cost(cols: np.ndarray) -> float:
    """Mean shared-memory wavefronts per tap when outputs 4i..4i+3 share a warp instruction and input k
    lives in bank group k % 4 (the RL = 8 tile), identical inputs broadcast: the unscheduled baseline."""
    N, K = cols.shape
    tot = 0
    for g in range(N // 4):
        for n in range(K):
            ks = set(int(k) for k in cols[4 * g:4 * g + 4, n])
            m = [0, 0, 0, 0]
            for k in ks:
                m[k % 4] += 1
            tot += max(m)
    return tot / (N // 4 * K)


def _layer_cols(net, l):
    N = net.N
    p = net.ptr[l * (N + 1):(l + 1) * (N + 1)]
    return np.stack([net.idx[p[j]:p[j + 1]] for j in range(N)]).astype(np.int32)


def test_gen_schedule_quads(lib):
    """General-CSC kernel schedule: the tile shape follows N, whole-line reads
    (G = 2, 4) never conflict, shift-structured layers get conflict-free quads (radix: inputs of the outputs
    of a quad differ mod 4 at every tap), a random permutation of them (perm) nearly so, and unstructured
    random columns beat the unscheduled quads."""
    from paper_conf_icpp_jiangh0h23_b200.api import gen_schedule
    from workload import sdgc
    assert gen_schedule(np.zeros((256, 4), np.int32))[0] == 2
    assert gen_schedule(np.zeros((1024, 4), np.int32)) == (4, 1.0)
    for N, mode in [(2048, "radix"), (4096, "radix"), (4096, "perm"), (2048, "random")]:
        net = sdgc.gen_network(N, 3, mode)
        for l in range(3):
            cols = _layer_cols(net, l)
            rl, cost = gen_schedule(cols)
            assert rl == 16, (N, rl)
            base = _quad_cost(cols)
            if mode == "radix":
                assert cost == 1.0
            elif mode == "perm":
                assert cost < 1.25 and cost < base - 0.5, (cost, base)
            else:
                assert cost < base - 0.2, (cost, base)
    rl, cost = gen_schedule(_layer_cols(sdgc.gen_medium_network(256, 2), 0))
    assert rl == 2 and cost == 1.0
    with pytest.raises(Exception):
        gen_schedule(np.full((64, 3), 64, np.int32))  # index out of range
