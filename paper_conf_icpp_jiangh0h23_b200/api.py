"""Python front end of the SNICIT C ABI (same names as include/snicit.h, argument marshalling only).

Device memory, streams and process groups come from PyTorch; all compute is in libsnicit.so.
"""
from __future__ import annotations

import ctypes
from typing import Optional

import numpy as np

from . import _lib
from ._lib import Options, SnicitError, Stats, check, default_options, load_library


def range_tables(w0: float, b0: float, ymax: float, kmax: int = 32):
    """snicit_debug_range_tables (R30): (hi, lo, active) horizon tables of the constant-row map
    out(v) = sigma(chain(v) + b0), k = 1..kmax.  Host computation inside the library (no GPU needed)."""
    L = load_library()
    hi = np.empty(kmax, np.float32)
    lo = np.empty(kmax, np.float32)
    r = L.snicit_debug_range_tables(float(w0), float(b0), float(ymax), int(kmax), hi.ctypes.data, lo.ctypes.data)
    if r < 0:
        check(r, "snicit_debug_range_tables")
    return hi, lo, bool(r)


def gen_schedule(cols: np.ndarray):
    """snicit_debug_gen_schedule (general-CSC kernel): (rows_per_tile, cost) of the
    load-time quad schedule for one layer given as an N x K array of input indices (chain order per
    output).  cost = mean shared-memory wavefronts per tap (1.0 = conflict-free).  Host only."""
    L = load_library()
    c = np.ascontiguousarray(cols, dtype=np.int32)
    if c.ndim != 2:
        raise ValueError("cols must be N x K")
    rl = ctypes.c_int32(0)
    cost = ctypes.c_double(0.0)
    check(L.snicit_debug_gen_schedule(int(c.shape[0]), int(c.shape[1]), c.ctypes.data, ctypes.byref(rl),
                                      ctypes.byref(cost)), "snicit_debug_gen_schedule")
    return int(rl.value), float(cost.value)


def _is_cuda_tensor(x) -> bool:
    return hasattr(x, "is_cuda") and bool(x.is_cuda)


def pack_rows(Y: np.ndarray, one: float = 1.0) -> np.ndarray:
    """Binary B x N rows (every value 0 or `one`) -> the packed bitmap of snicit_infer_packed:
    B x ceil(N/32) uint32, bit j % 32 (LSB first) of word j / 32 set where Y[r, j] == one.
    Layout marshalling only (no SNICIT arithmetic)."""
    Y = np.asarray(Y)
    nz = Y != 0
    if not np.all(Y[nz] == np.float32(one)):
        raise ValueError("pack_rows: rows must be binary (0 or `one`)")
    B, N = Y.shape
    W = (N + 31) // 32
    padded = np.zeros((B, W * 32), dtype=bool)
    padded[:, :N] = nz
    by = np.packbits(padded.reshape(B, W * 4, 8), axis=2, bitorder="little").reshape(B, W * 4)
    return np.ascontiguousarray(by).view("<u4").reshape(B, W)


def _check_device(x, device: int, what: str) -> None:
    if _is_cuda_tensor(x) and int(x.device.index) != int(device):
        raise ValueError(f"{what} is on cuda:{x.device.index}, the network on cuda:{device}")


def _out_arg(y_out, B: int, N: int, device: int):
    """(on_device, pointer) of a caller-owned B x N fp32 C-contiguous output (None -> not materialised).
    The library writes B*N*4 bytes there, so shape, dtype and layout are checked first."""
    if y_out is None:
        return 0, None
    if _is_cuda_tensor(y_out):
        import torch
        if y_out.dtype != torch.float32 or tuple(y_out.shape) != (B, N) or not y_out.is_contiguous():
            raise ValueError(f"y_out must be a contiguous float32 tensor of shape ({B}, {N})")
        _check_device(y_out, device, "y_out")
        return 1, y_out.data_ptr()
    ya = y_out.numpy() if hasattr(y_out, "numpy") else y_out
    if not (isinstance(ya, np.ndarray) and ya.dtype == np.float32 and ya.shape == (B, N) and ya.flags.c_contiguous
            and ya.flags.writeable):
        raise ValueError(f"host y_out must be a writeable C-contiguous float32 array of shape ({B}, {N})")
    return 0, ya.ctypes.data


class SnicitNetwork:
    """Owns one `snicit_network*` (device copy of W, b + workspace) on `device`.

    `ptr` (int64, L*(N+1) absolute offsets), `idx` (int32), `val` (float32), `bias` (float32, L*N):
    CSC over output neurons with the accumulation order stored (include/snicit.h).
    """

    def __init__(self, N: int, L: int, ptr, idx, val, bias, ymax: float, device: int = 0, fmt: int = _lib.CSC):
        self._lib = load_library()
        self.N, self.L, self.ymax, self.device = int(N), int(L), float(ymax), int(device)
        ptr = np.ascontiguousarray(ptr, dtype=np.int64)
        idx = np.ascontiguousarray(idx, dtype=np.int32)
        val = np.ascontiguousarray(val, dtype=np.float32)
        bias = np.ascontiguousarray(bias, dtype=np.float32)
        if ptr.size != self.L * (self.N + 1) or bias.size != self.L * self.N:
            raise ValueError("ptr must have L*(N+1) entries and bias L*N")
        h = ctypes.c_void_p()
        st = self._lib.snicit_load_network(self.N, self.L, fmt, ptr.ctypes.data, idx.ctypes.data if idx.size else None,
                                           val.ctypes.data if val.size else None, bias.ctypes.data, self.ymax,
                                           self.device, ctypes.byref(h))
        check(st, "snicit_load_network")
        self._h = h
        self._last_batch = 0
        self._last_ns = (0, 1)
        self._stream = None

    @classmethod
    def circulant(cls, N: int, L: int, nu, w, bias, ymax: float, device: int = 0):
        """Compact shift-invariant form (snicit_load_network_circulant): column j of layer l reads
        (j + n*nu[l]) mod N with weight w[l, n], n = 0..K-1."""
        self = cls.__new__(cls)
        self._lib = load_library()
        self.N, self.L, self.ymax, self.device = int(N), int(L), float(ymax), int(device)
        nu = np.ascontiguousarray(nu, dtype=np.int32)
        w = np.ascontiguousarray(w, dtype=np.float32).reshape(L, -1)
        bias = np.ascontiguousarray(bias, dtype=np.float32)
        if nu.size != L or bias.size != L * N:
            raise ValueError("nu must have L entries and bias L*N")
        h = ctypes.c_void_p()
        check(self._lib.snicit_load_network_circulant(self.N, self.L, nu.ctypes.data, int(w.shape[1]),
                                                      w.ctypes.data, bias.ctypes.data, self.ymax, self.device,
                                                      ctypes.byref(h)), "snicit_load_network_circulant")
        self._h = h
        self._last_batch = 0
        self._last_ns = (0, 1)
        self._stream = None
        return self

    @classmethod
    def from_network(cls, net, device: int = 0):
        """From a workload.sdgc.Network-like object (N, L, ptr, idx, val, bias, ymax)."""
        return cls(net.N, net.L, net.ptr, net.idx, net.val, net.bias, net.ymax, device=device)

    # ------------------------------------------------------------------ lifecycle
    def close(self):
        if getattr(self, "_h", None):
            self._lib.snicit_free_network(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ------------------------------------------------------------------ calls
    def set_stream(self, stream) -> None:
        """stream: a torch.cuda.Stream, a raw cudaStream_t int, or None (legacy default stream)."""
        raw = None
        if stream is not None:
            raw = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
        self._stream = stream
        check(self._lib.snicit_set_stream(self._h, raw), "snicit_set_stream")

    def infer(self, y0, t: int, s: int = 32, options: Optional[Options] = None, y_out=None,
              row_offset: int = 0, **opt_kw):
        """Run SNICIT on y0 (B x N fp32: CUDA tensor, CPU tensor or numpy array).

        y_out: None (not materialised), or a B x N fp32 CUDA tensor / CPU tensor / numpy array to fill.
        Returns y_out.
        """
        if options is None:
            options = default_options(**opt_kw)
        elif opt_kw:
            raise ValueError("pass either options or keyword options")
        if _is_cuda_tensor(y0):
            import torch
            if y0.dtype != torch.float32 or not y0.is_contiguous() or y0.dim() != 2:
                raise ValueError("device y0 must be a contiguous 2-D float32 tensor")
            _check_device(y0, self.device, "y0")
            B = int(y0.shape[0])
            y0_dev, y0p = 1, y0.data_ptr()
        else:
            arr = y0.numpy() if hasattr(y0, "numpy") else y0
            if not (isinstance(arr, np.ndarray) and arr.dtype == np.float32 and arr.flags.c_contiguous
                    and arr.ndim == 2):
                raise ValueError("host y0 must be a C-contiguous 2-D float32 array")
            B = int(arr.shape[0])
            y0_dev, y0p = 0, arr.ctypes.data
        if int(y0.shape[1]) != self.N:
            raise ValueError(f"y0 must be B x {self.N}")
        yo_dev, yop = _out_arg(y_out, B, self.N, self.device)
        st = self._lib.snicit_infer(self._h, y0p, B, y0_dev, int(row_offset), int(t), int(s), ctypes.byref(options),
                                    yop, yo_dev)
        check(st, "snicit_infer")
        self._last_batch = B
        self._last_ns = (self.N if options.n_segments == 0 else int(options.n_segments), int(s))
        return y_out

    def infer_packed(self, bits, t: int, s: int = 32, options: Optional[Options] = None, y_out=None,
                     row_offset: int = 0, one: float = 1.0, **opt_kw):
        """snicit_infer_packed: binary inputs as the packed bitmap of `pack_rows` (B x ceil(N/32)
        uint32: numpy array, CPU tensor or CUDA tensor of int32/uint32).  Same results as infer()."""
        if options is None:
            options = default_options(**opt_kw)
        elif opt_kw:
            raise ValueError("pass either options or keyword options")
        W = (self.N + 31) // 32
        if _is_cuda_tensor(bits):
            if bits.element_size() != 4 or not bits.is_contiguous() or bits.dim() != 2:
                raise ValueError("device bits must be a contiguous 2-D tensor of 32-bit words")
            _check_device(bits, self.device, "bits")
            B, dev, bp = int(bits.shape[0]), 1, bits.data_ptr()
        else:
            arr = bits.numpy() if hasattr(bits, "numpy") else bits
            if not (isinstance(arr, np.ndarray) and arr.dtype.itemsize == 4 and arr.flags.c_contiguous
                    and arr.ndim == 2):
                raise ValueError("host bits must be a C-contiguous 2-D 32-bit array")
            B, dev, bp = int(arr.shape[0]), 0, arr.ctypes.data
        if int(bits.shape[1]) != W:
            raise ValueError(f"bits must be B x {W}")
        yo_dev, yop = _out_arg(y_out, B, self.N, self.device)
        check(self._lib.snicit_infer_packed(self._h, bp, B, dev, float(one), int(row_offset), int(t), int(s),
                                            ctypes.byref(options), yop, yo_dev), "snicit_infer_packed")
        self._last_batch = B
        self._last_ns = (self.N if options.n_segments == 0 else int(options.n_segments), int(s))
        return y_out

    def categories(self) -> np.ndarray:
        """Ascending global row ids of the category set (R13) of the last infer."""
        n = ctypes.c_int64(0)
        check(self._lib.snicit_categories(self._h, None, ctypes.byref(n), 0), "snicit_categories")
        out = np.empty(n.value, dtype=np.int64)
        if n.value:
            check(self._lib.snicit_categories(self._h, out.ctypes.data, ctypes.byref(n), 0), "snicit_categories")
        return out[:n.value]

    def categories_device(self, out) -> None:
        """snicit_categories_device: out (CUDA int64 tensor of 1 + capacity) <- [count, ids...], queued on
        the handle's stream (no host synchronisation)."""
        import torch
        if not (_is_cuda_tensor(out) and out.dtype == torch.int64 and out.is_contiguous() and out.dim() == 1
                and out.numel() >= 1):
            raise ValueError("out must be a contiguous 1-D int64 CUDA tensor of 1 + capacity entries")
        _check_device(out, self.device, "out")
        check(self._lib.snicit_categories_device(self._h, out.data_ptr(), int(out.numel()) - 1),
              "snicit_categories_device")

    def num_categories(self) -> int:
        n = ctypes.c_int64(0)
        check(self._lib.snicit_categories(self._h, None, ctypes.byref(n), 0), "snicit_categories")
        return int(n.value)

    def stats(self) -> dict:
        s = Stats()
        check(self._lib.snicit_stats(self._h, ctypes.byref(s)), "snicit_stats")
        return s.as_dict()

    def layer_profile(self, max_layers: int = 4096) -> dict:
        """Per pre-convergence layer kernel: CUDA-event ms, active rows, algorithmic bytes
        (needs options.timing == 2 on the last infer)."""
        ms = np.zeros(max_layers, np.float64)
        rows = np.zeros(max_layers, np.int64)
        by = np.zeros(max_layers, np.float64)
        n = ctypes.c_int32(0)
        check(self._lib.snicit_layer_profile(self._h, max_layers, ms.ctypes.data, rows.ctypes.data, by.ctypes.data,
                                             ctypes.byref(n)), "snicit_layer_profile")
        k = n.value
        return dict(ms=ms[:k].copy(), rows=rows[:k].copy(), bytes=by[:k].copy())

    def dynamics(self) -> dict:
        """Per-layer dynamics of the last infer run with options.timing >= 1 (snicit_dynamics): arrays over
        layers 0..L-1, -1 where not recorded."""
        L = self.L
        arrs = {k: np.full(L, -1, np.int64) for k in ("pre_full", "pre_live", "res_alive", "res_scalar")}
        n = ctypes.c_int32(0)
        check(self._lib.snicit_dynamics(self._h, L, arrs["pre_full"].ctypes.data, arrs["pre_live"].ctypes.data,
                                        arrs["res_alive"].ctypes.data, arrs["res_scalar"].ctypes.data,
                                        ctypes.byref(n)), "snicit_dynamics")
        return arrs

    def write_dynamics_jsonl(self, path: str, extra: Optional[dict] = None) -> int:
        """One JSON object per layer (SURVEY 5 per-layer log): layer, phase, live / full / residue counts,
        plus the run's clustering stats on the first line.  Returns the number of lines written."""
        import json
        d = self.dynamics()
        st = self.stats()
        t = int(st["threshold_layer"])
        with open(path, "w") as f:
            head = {"run": {k: st[k] for k in ("batch", "threshold_layer", "live_at_t", "n_centroids", "n_sampled",
                                               "residual_at_t", "residual_final", "res_nnz_at_t", "n_categories")}}
            if extra:
                head["run"].update(extra)
            f.write(json.dumps(head) + "\n")
            for l in range(self.L):
                rec = {"layer": l, "phase": "pre" if l < t else "post"}
                if l < t:
                    rec.update(pre_full=int(d["pre_full"][l]), pre_live=int(d["pre_live"][l]))
                else:
                    rec.update(centroids=int(st["n_centroids"]), res_alive=int(d["res_alive"][l]),
                               res_scalar=int(d["res_scalar"][l]))
                f.write(json.dumps(rec) + "\n")
        return self.L + 1

    def debug_clustering(self, n_segments: Optional[int] = None, s: Optional[int] = None) -> dict:
        """Clustering state of the last infer.  The buffers are sized from that infer's n and s (the
        arguments are accepted for compatibility and must match them if given)."""
        B = self._last_batch
        n_last, s_last = self._last_ns
        if (n_segments is not None and (self.N if n_segments == 0 else n_segments) != n_last) or \
                (s is not None and s != s_last):
            raise ValueError(f"last infer used n={n_last}, s={s_last}")
        n, s = n_last, s_last
        cent = np.empty(max(s, 1), np.int32)
        ncent = ctypes.c_int32(0)
        M = np.empty(max(B, 1), np.int32)
        ne = np.empty(max(B, 1), np.uint8)
        F = np.empty(n * max(s, 1), np.float64)
        ns = ctypes.c_int32(0)
        live = np.empty(max(B, 1), np.uint8)
        check(self._lib.snicit_debug_clustering(self._h, cent.ctypes.data, ctypes.byref(ncent), M.ctypes.data,
                                                ne.ctypes.data, F.ctypes.data, ctypes.byref(ns), live.ctypes.data),
              "snicit_debug_clustering")
        return dict(cent=cent[:ncent.value].copy(), M=M[:B].copy(), ne_t=ne[:B].astype(bool),
                    F=F[:n * ns.value].reshape(n, ns.value).copy(), n_sampled=ns.value, live_t=live[:B].astype(bool))

    def debug_layer(self, layer: int, yin, yout, kernel: int = _lib.KERNEL_AUTO) -> None:
        """One plain layer on CUDA tensors (rows x N)."""
        assert _is_cuda_tensor(yin) and _is_cuda_tensor(yout)
        check(self._lib.snicit_debug_layer(self._h, int(layer), yin.data_ptr(), yout.data_ptr(), int(yin.shape[0]),
                                           int(kernel)), "snicit_debug_layer")

    def layer_is_circulant(self, layer: int) -> bool:
        r = self._lib.snicit_layer_is_circulant(self._h, int(layer))
        if r < 0:
            raise SnicitError("bad layer")
        return bool(r)


__all__ = ["SnicitNetwork", "Options", "Stats", "SnicitError", "default_options"]
