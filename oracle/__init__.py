"""SNICIT CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_icpp_jiangh0h23_b200``) never imports it and shares no code with it.

A thin ctypes binding over ``oracle/liboracle.so`` (plain C, ``oracle.c``; every function
cites the PAPER.md passage it follows).  Argument marshalling only.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain C11, OpenMP, no FP contraction)."""
    src = os.path.join(_HERE, "oracle.c")
    if (not force and os.path.exists(LIB_PATH)
            and os.path.getmtime(LIB_PATH) >= max(os.path.getmtime(src),
                                                  os.path.getmtime(os.path.join(_HERE, "oracle.h")))):
        return LIB_PATH
    cmd = ["gcc", "-O2", "-std=gnu11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC",
           "-shared", "-o", LIB_PATH + ".tmp", src, "-lm"]
    subprocess.check_call(cmd, cwd=_HERE)
    os.replace(LIB_PATH + ".tmp", LIB_PATH)
    return LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB_PATH)
        P = ctypes.c_void_p
        i32, i64, f32 = ctypes.c_int32, ctypes.c_int64, ctypes.c_float
        L.oracle_version.restype = i32
        L.oracle_layers_f32.argtypes = [i32, P, P, P, P, f32, i32, i32, i64, P, P, i32]
        L.oracle_layers_f64.argtypes = [i32, P, P, P, P, f32, i32, i32, i64, P, P, i32]
        L.oracle_layers_circulant_f32.argtypes = [i32, i32, P, P, P, f32, i32, i32, i64, P, P, i32]
        L.oracle_layers_f32_fast.argtypes = [i32, P, P, P, P, f32, i32, i32, i64, P, P, i32]
        L.oracle_layers_f32_fast.restype = i64
        L.oracle_layers_circulant_f32_fast.argtypes = [i32, i32, P, P, P, f32, i32, i32, i64, P, P, i32]
        L.oracle_layers_circulant_f32_fast.restype = i64
        L.oracle_sum_downsample.argtypes = [i32, i32, i32, P, P]
        L.oracle_prune.argtypes = [i32, i32, P, f32, f32, P]
        L.oracle_prune.restype = i32
        L.oracle_map_residual.argtypes = [i32, i64, P, P, i32, P, P, P, P]
        L.oracle_post_layer.argtypes = [i32, P, P, P, P, f32, i32, i64, P, P, P, P, f32, i32]
        L.oracle_recover.argtypes = [i32, i64, P, P, P, P, P]
        L.oracle_snicit.argtypes = [i32, i32, P, P, P, P, f32, i64, P, i32, i32, i32, f32, f32, f32,
                                    i32, P, P, P, P, P, P, P, P, i32]
        L.oracle_snicit.restype = i32
        _lib = L
    return _lib


def _p(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _net_arrays(net):
    return (np.ascontiguousarray(net.ptr, dtype=np.int64), np.ascontiguousarray(net.idx, dtype=np.int32),
            np.ascontiguousarray(net.val, dtype=np.float32), np.ascontiguousarray(net.bias, dtype=np.float32))


def layers_f32(net, Y: np.ndarray, l0: int = 0, l1: Optional[int] = None, nthreads: int = 0) -> np.ndarray:
    """Plain Eq. (1) in fp32 over layers [l0, l1)."""
    l1 = net.L if l1 is None else l1
    Y = np.ascontiguousarray(Y, dtype=np.float32)
    out = np.empty_like(Y)
    ptr, idx, val, bias = _net_arrays(net)
    lib().oracle_layers_f32(net.N, _p(ptr), _p(idx), _p(val), _p(bias), net.ymax, l0, l1,
                            Y.shape[0], _p(Y), _p(out), nthreads)
    return out


def layers_f64(net, Y: np.ndarray, l0: int = 0, l1: Optional[int] = None, nthreads: int = 0) -> np.ndarray:
    """Plain Eq. (1) in fp64 (the definition at higher precision)."""
    l1 = net.L if l1 is None else l1
    Y = np.ascontiguousarray(Y, dtype=np.float64)
    out = np.empty_like(Y)
    ptr, idx, val, bias = _net_arrays(net)
    lib().oracle_layers_f64(net.N, _p(ptr), _p(idx), _p(val), _p(bias), net.ymax, l0, l1,
                            Y.shape[0], _p(Y), _p(out), nthreads)
    return out


def layers_circulant_f32(cnet, Y: np.ndarray, l0: int = 0, l1: Optional[int] = None, nthreads: int = 0) -> np.ndarray:
    """Plain Eq. (1) in fp32 for a network in compact circulant form (workload.sdgc.CirculantNetwork)."""
    l1 = cnet.L if l1 is None else l1
    Y = np.ascontiguousarray(Y, dtype=np.float32)
    out = np.empty_like(Y)
    nu = np.ascontiguousarray(cnet.nu, dtype=np.int32)
    w = np.ascontiguousarray(cnet.w, dtype=np.float32)
    b = np.ascontiguousarray(cnet.bias, dtype=np.float32)
    lib().oracle_layers_circulant_f32(cnet.N, w.shape[1], _p(nu), _p(w), _p(b), cnet.ymax, l0, l1, Y.shape[0],
                                      _p(Y), _p(out), nthreads)
    return out


def layers_f32_fast(net, Y: np.ndarray, l0: int = 0, l1: Optional[int] = None, nthreads: int = 0,
                    return_skipped: bool = False):
    """Exact fast mode of Eq. (1) (oracle.h): fixed-point rows (all-zero / all-YMAX) whose image under a
    layer is themselves are not re-evaluated.  Identical to layers_f32 (pinned).  Accepts a CSC Network
    or a compact CirculantNetwork."""
    l1 = net.L if l1 is None else l1
    Y = np.ascontiguousarray(Y, dtype=np.float32)
    out = np.empty_like(Y)
    if hasattr(net, "nu"):
        nu = np.ascontiguousarray(net.nu, dtype=np.int32)
        w = np.ascontiguousarray(net.w, dtype=np.float32)
        b = np.ascontiguousarray(net.bias, dtype=np.float32)
        sk = lib().oracle_layers_circulant_f32_fast(net.N, w.shape[1], _p(nu), _p(w), _p(b), net.ymax, l0, l1,
                                                    Y.shape[0], _p(Y), _p(out), nthreads)
    else:
        ptr, idx, val, bias = _net_arrays(net)
        sk = lib().oracle_layers_f32_fast(net.N, _p(ptr), _p(idx), _p(val), _p(bias), net.ymax, l0, l1,
                                          Y.shape[0], _p(Y), _p(out), nthreads)
    return (out, int(sk)) if return_skipped else out


def categories(Y: np.ndarray) -> np.ndarray:
    """Reading R13: ascending ids of rows with any non-zero."""
    return np.nonzero((Y != 0).any(axis=1))[0].astype(np.int64)


def sum_downsample(rows: np.ndarray, n: int) -> np.ndarray:
    rows = np.ascontiguousarray(rows, dtype=np.float32)
    s, N = rows.shape
    nn = N if n <= 0 else n
    F = np.empty((nn, s), dtype=np.float64)
    lib().oracle_sum_downsample(N, n, s, _p(rows), _p(F))
    return F


def prune(F: np.ndarray, eta: float, eps: float, col_idx: Optional[np.ndarray] = None) -> np.ndarray:
    F = np.ascontiguousarray(F, dtype=np.float64)
    n, s = F.shape
    ci = np.arange(s, dtype=np.int32) if col_idx is None else np.ascontiguousarray(col_idx, dtype=np.int32).copy()
    lib().oracle_prune(n, s, _p(F), eta, eps, _p(ci))
    return ci


def map_residual(Y: np.ndarray, cent: np.ndarray, live: Optional[np.ndarray] = None):
    Y = np.ascontiguousarray(Y, dtype=np.float32)
    R, N = Y.shape
    cent = np.ascontiguousarray(cent, dtype=np.int32)
    lv = None if live is None else np.ascontiguousarray(live, dtype=np.uint8)
    M = np.empty(R, dtype=np.int32)
    Yhat = np.zeros_like(Y)
    ne = np.empty(R, dtype=np.uint8)
    lib().oracle_map_residual(N, R, _p(Y), _p(lv), len(cent), _p(cent), _p(M), _p(Yhat), _p(ne))
    return M, Yhat, ne


def post_layer(net, l: int, M: np.ndarray, Yhat: np.ndarray, ne: np.ndarray, prune_eps: float = 0.0,
               out: Optional[np.ndarray] = None, nthreads: int = 0):
    Yhat = np.ascontiguousarray(Yhat, dtype=np.float32)
    R, N = Yhat.shape
    M = np.ascontiguousarray(M, dtype=np.int32)
    ne2 = np.ascontiguousarray(ne, dtype=np.uint8).copy()
    if out is None:
        out = np.zeros_like(Yhat)
    ptr, idx, val, bias = _net_arrays(net)
    lib().oracle_post_layer(N, _p(ptr), _p(idx), _p(val), _p(bias), net.ymax, l, R, _p(M), _p(Yhat),
                            _p(ne2), _p(out), prune_eps, nthreads)
    return out, ne2


def recover(M: np.ndarray, ne: np.ndarray, Yhat: np.ndarray):
    Yhat = np.ascontiguousarray(Yhat, dtype=np.float32)
    R, N = Yhat.shape
    out = np.empty_like(Yhat)
    cat = np.empty(R, dtype=np.uint8)
    lib().oracle_recover(N, R, _p(np.ascontiguousarray(M, dtype=np.int32)),
                         _p(np.ascontiguousarray(ne, dtype=np.uint8)), _p(Yhat), _p(out), _p(cat))
    return out, cat


def snicit(net, Y0: np.ndarray, t: int, s: int = 32, n: int = 16, eta: float = 0.03, eps: float = 0.03,
           prune_eps: float = 0.0, drop_dead: bool = True, nthreads: int = 0) -> dict:
    """The whole SNICIT pipeline in the paper's order (Fig. 2)."""
    Y0 = np.ascontiguousarray(Y0, dtype=np.float32)
    B, N = Y0.shape
    Y = np.empty_like(Y0)
    cat = np.empty(B, dtype=np.uint8)
    M = np.empty(B, dtype=np.int32)
    cent = np.empty(max(s, 1), dtype=np.int32)
    ncent = np.zeros(1, dtype=np.int32)
    nn = N if n <= 0 else n
    F = np.zeros(nn * max(s, 1), dtype=np.float64)
    live = np.empty(B, dtype=np.uint8)
    ne = np.empty(B, dtype=np.uint8)
    ptr, idx, val, bias = _net_arrays(net)
    rc = lib().oracle_snicit(N, net.L, _p(ptr), _p(idx), _p(val), _p(bias), net.ymax, B, _p(Y0), t, s, n,
                             eta, eps, prune_eps, int(drop_dead), _p(Y), _p(cat), _p(M), _p(cent), _p(ncent),
                             _p(F), _p(live), _p(ne), nthreads)
    if rc != 0:
        raise ValueError("oracle_snicit: bad arguments")
    C = int(ncent[0])
    ss = int(min(s, int(live.sum()))) if t < net.L else 0
    return dict(Y=Y, cat=cat, categories=np.nonzero(cat)[0].astype(np.int64), M=M, cent=cent[:C].copy(),
                F=F[:nn * ss].reshape(nn, ss).copy(), live_t=live.astype(bool),
                ne=ne.astype(bool))
