"""ctypes binding of libsnicit.so (include/snicit.h).  Argument marshalling only.

Every computation of the SNICIT path runs in the library's CUDA kernels.  There is no CPU
fallback: if the shared library is missing or no sm_100 device is present, calls raise.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libsnicit.so")

SNICIT_OK = 0
STATUS_NAMES = {0: "OK", -1: "E_INVALID_ARG", -2: "E_BAD_SPARSE", -3: "E_OOM", -4: "E_CUDA", -5: "E_STATE",
                -6: "E_UNSUPPORTED"}
CSC, CSR = 0, 1
KERNEL_AUTO, KERNEL_ELL, KERNEL_CIRC, KERNEL_CIRC_SMEM = 0, 1, 2, 3

EXPORTED = ["snicit_default_options", "snicit_load_network", "snicit_set_stream", "snicit_infer",
            "snicit_categories", "snicit_stats", "snicit_debug_clustering", "snicit_debug_layer",
            "snicit_layer_is_circulant", "snicit_free_network", "snicit_last_error", "snicit_abi_version",
            "snicit_layer_profile", "snicit_load_network_circulant", "snicit_infer_packed",
            "snicit_categories_device", "snicit_dynamics", "snicit_debug_range_tables",
            "snicit_debug_gen_schedule"]


class Options(ctypes.Structure):
    _fields_ = [("n_segments", ctypes.c_int32), ("eta", ctypes.c_float), ("eps", ctypes.c_float),
                ("prune_eps", ctypes.c_float), ("drop_dead_rows", ctypes.c_int32), ("kernel", ctypes.c_int32),
                ("timing", ctypes.c_int32), ("ne_interval", ctypes.c_int32), ("post_mode", ctypes.c_int32),
                ("post_cluster", ctypes.c_int32), ("post_const", ctypes.c_int32),
                ("pre_fused", ctypes.c_int32), ("pre_const", ctypes.c_int32), ("res_sparse", ctypes.c_int32),
                ("dyn_t", ctypes.c_int32)]


class Stats(ctypes.Structure):
    _fields_ = [("t_pre_ms", ctypes.c_double), ("t_convert_ms", ctypes.c_double), ("t_post_ms", ctypes.c_double),
                ("t_recover_ms", ctypes.c_double), ("t_total_ms", ctypes.c_double), ("batch", ctypes.c_int64),
                ("live_at_t", ctypes.c_int64), ("residual_at_t", ctypes.c_int64),
                ("residual_final", ctypes.c_int64), ("n_categories", ctypes.c_int64),
                ("n_centroids", ctypes.c_int32), ("n_sampled", ctypes.c_int32), ("threshold_layer", ctypes.c_int32),
                ("circ_layers", ctypes.c_int32), ("kernel_launches", ctypes.c_int64),
                ("const_centroids", ctypes.c_int32), ("pre_fused", ctypes.c_int32),
                ("pre_const_rows", ctypes.c_int32), ("pre_full_rows", ctypes.c_int64),
                ("res_nnz_at_t", ctypes.c_int64), ("res_full_rl", ctypes.c_int64), ("res_sparse_rl", ctypes.c_int64),
                ("res_sparse_out", ctypes.c_int64), ("res_scalar_rl", ctypes.c_int64), ("map_rows", ctypes.c_int64),
                ("t_map_ms", ctypes.c_double),
                ("t_residual_ms", ctypes.c_double), ("pre_popc_rows", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class SnicitError(RuntimeError):
    pass


_lib = None


def load_library(path: str = LIB_PATH):
    """Load libsnicit.so and declare the C signatures (raises if the library was not built).
    SNICIT_LIB overrides the path (A/B builds in experiments)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("SNICIT_LIB") or path
    if not os.path.exists(path):
        raise SnicitError(f"{path} not found: run __graft_entry__.build() (nvcc, sm_100a)")
    L = ctypes.CDLL(path)
    P, i32, i64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_float
    L.snicit_default_options.argtypes = [ctypes.POINTER(Options)]
    L.snicit_default_options.restype = None
    L.snicit_load_network.argtypes = [i32, i32, i32, P, P, P, P, f32, i32, ctypes.POINTER(P)]
    L.snicit_load_network.restype = i32
    L.snicit_load_network_circulant.argtypes = [i32, i32, P, i32, P, P, f32, i32, ctypes.POINTER(P)]
    L.snicit_load_network_circulant.restype = i32
    L.snicit_set_stream.argtypes = [P, P]
    L.snicit_set_stream.restype = i32
    L.snicit_infer.argtypes = [P, P, i64, i32, i64, i32, i32, ctypes.POINTER(Options), P, i32]
    L.snicit_infer.restype = i32
    L.snicit_infer_packed.argtypes = [P, P, i64, i32, f32, i64, i32, i32, ctypes.POINTER(Options), P, i32]
    L.snicit_infer_packed.restype = i32
    L.snicit_categories.argtypes = [P, P, ctypes.POINTER(i64), i32]
    L.snicit_categories.restype = i32
    L.snicit_categories_device.argtypes = [P, P, i64]
    L.snicit_categories_device.restype = i32
    L.snicit_stats.argtypes = [P, ctypes.POINTER(Stats)]
    L.snicit_stats.restype = i32
    L.snicit_dynamics.argtypes = [P, i32, P, P, P, P, P]
    L.snicit_dynamics.restype = i32
    L.snicit_layer_profile.argtypes = [P, i32, P, P, P, P]
    L.snicit_layer_profile.restype = i32
    L.snicit_debug_clustering.argtypes = [P, P, P, P, P, P, P, P]
    L.snicit_debug_clustering.restype = i32
    L.snicit_debug_layer.argtypes = [P, i32, P, P, i64, i32]
    L.snicit_debug_layer.restype = i32
    L.snicit_debug_range_tables.argtypes = [f32, f32, f32, i32, P, P]
    L.snicit_debug_range_tables.restype = i32
    L.snicit_debug_gen_schedule.argtypes = [i32, i32, P, P, P]
    L.snicit_debug_gen_schedule.restype = i32
    L.snicit_layer_is_circulant.argtypes = [P, i32]
    L.snicit_layer_is_circulant.restype = i32
    L.snicit_free_network.argtypes = [P]
    L.snicit_free_network.restype = None
    L.snicit_last_error.argtypes = []
    L.snicit_last_error.restype = ctypes.c_char_p
    L.snicit_abi_version.argtypes = []
    L.snicit_abi_version.restype = i32
    _lib = L
    return L


def check(status: int, what: str):
    if status != SNICIT_OK:
        msg = _lib.snicit_last_error().decode(errors="replace") if _lib is not None else ""
        raise SnicitError(f"{what} failed: {STATUS_NAMES.get(status, status)}: {msg}")


def default_options(**kw) -> Options:
    o = Options()
    load_library().snicit_default_options(ctypes.byref(o))
    for k, v in kw.items():
        if not hasattr(o, k):
            raise KeyError(k)
        setattr(o, k, v)
    return o


def _ptr(a) -> Optional[int]:
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    if hasattr(a, "data_ptr"):  # torch tensor
        return a.data_ptr()
    return int(a)
