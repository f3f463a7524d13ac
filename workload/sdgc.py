"""Seeded synthetic SDGC-like workloads (networks and inputs).

The SDGC datasets are not available offline, so every input is synthetic with
the shapes, constants and structure the paper describes:

* networks: "generated based on Radix-Net ... Each neuron in all architectures
  has 32 edge connections with neurons in adjacent layers ... the biases are set
  as constants" (Sec. 2.1); per-net bias from Table 1
  (PAPER.md:251-290): -0.3 / -0.35 / -0.4 / -0.45 for N = 1024 / 4096 / 16384 /
  65536; weights 1/16 and YMAX = 32 (BASELINE.json north_star; sigma, Table 2
  PAPER.md:410);
* inputs: "stacks of feature vectors derived from ... MNIST. Each 28x28 pixel
  image is resized ... to 32x32 (1024 neurons), 64x64 (4096), 128x128 (16384),
  256x256 (65536), and then flattened"; binary values.

Layout convention: activations are ``B x N`` row-major
(one row per sample, the paper's column); ``W`` of a layer is stored as CSC over
the *output* neuron ``j`` (``ptr[j]..ptr[j+1]`` lists the inputs ``k`` feeding
``j``), i.e. the paper's row ``j`` of ``W(i+1)``.  The stored order of a column's
entries is the accumulation order (reading R12).

This module holds NO SNICIT arithmetic: it only draws numbers.  The recipe is
documented in DESIGN.md "Input recipe".
"""
from __future__ import annotations

import dataclasses
import math
from typing import Dict, Optional

import numpy as np

from . import rng

BASE_SEED = 20230807  # ICPP'23 date, SURVEY.md 8(d)

SDGC_BIAS = {1024: -0.3, 4096: -0.35, 16384: -0.4, 65536: -0.45}  # Table 1
SDGC_WEIGHT = 1.0 / 16.0
SDGC_YMAX = 32.0
SDGC_K = 32  # connections per neuron


@dataclasses.dataclass
class Network:
    """A sparse DNN: L layers of CSC (per output neuron) with explicit stored order."""

    N: int
    L: int
    ptr: np.ndarray  # int64 [L*(N+1)], absolute offsets into idx/val
    idx: np.ndarray  # int32 [nnz_total]
    val: np.ndarray  # float32 [nnz_total]
    bias: np.ndarray  # float32 [L*N]
    ymax: float
    mode: str = "radix"
    strides: Optional[list] = None

    @property
    def nnz(self) -> int:
        return int(self.ptr[-1])

    def layer(self, l: int):
        """(ptr relative to the layer, idx, val, bias) of layer l (0-based)."""
        p = self.ptr[l * (self.N + 1):(l + 1) * (self.N + 1)]
        a, b = int(p[0]), int(p[-1])
        return p - a, self.idx[a:b], self.val[a:b], self.bias[l * self.N:(l + 1) * self.N]


def radix_strides(N: int) -> list:
    """Stride cycle nu_l for the RadiX-like layers: {1, 32, 1024, ...} within [1, N/32], plus N/32."""
    top = N // SDGC_K
    s = []
    v = 1
    while v <= top:
        s.append(v)
        v *= 32
    if top not in s:
        s.append(top)
    return s


def _assemble(N, L, cols_per_layer, vals_per_layer, bias, ymax, mode, strides=None) -> Network:
    ptrs, idxs, vals = [], [], []
    off = 0
    for l in range(L):
        cols = cols_per_layer[l]  # list/array of per-column index arrays, or 2-D [N, K]
        v = vals_per_layer[l]
        if isinstance(cols, np.ndarray) and cols.ndim == 2:
            K = cols.shape[1]
            p = off + np.arange(N + 1, dtype=np.int64) * K
            idxs.append(cols.reshape(-1).astype(np.int32))
            vals.append(np.asarray(v, dtype=np.float32).reshape(-1))
        else:
            lens = np.array([len(c) for c in cols], dtype=np.int64)
            p = off + np.concatenate([[0], np.cumsum(lens)])
            idxs.append(np.concatenate(cols).astype(np.int32))
            vals.append(np.concatenate(v).astype(np.float32))
        ptrs.append(p)
        off = int(p[-1])
    return Network(N=N, L=L, ptr=np.concatenate(ptrs).astype(np.int64),
                   idx=np.concatenate(idxs), val=np.concatenate(vals),
                   bias=np.asarray(bias, dtype=np.float32).reshape(L * N), ymax=float(ymax),
                   mode=mode, strides=strides)


def gen_network(N: int, L: int, mode: str = "radix", seed: int = BASE_SEED, K: int = SDGC_K,
                bias: Optional[float] = None, weight: float = SDGC_WEIGHT,
                ymax: float = SDGC_YMAX) -> Network:
    """SDGC-like network.

    mode="radix": column j of layer l holds inputs (j + n*nu_l) mod N, n = 0..K-1 (stored in n
      order), nu_l cycling through radix_strides(N) -- a sum of K cyclic permutations.
    mode="perm":  same, then a seeded random permutation pi_l of the output neurons:
      column pi_l(j) holds the inputs of radix column j.  In- and out-degree stay K.
    mode="random": K distinct uniformly random inputs per column, stored ascending (no structure;
      in-degree varies).
    """
    if bias is None:
        bias = SDGC_BIAS.get(N, -0.3)
    strides = radix_strides(N) if mode in ("radix", "perm") else None
    cols, vals = [], []
    for l in range(L):
        if mode in ("radix", "perm"):
            nu = strides[l % len(strides)]
            assert K * nu <= N, "inputs of a column must be distinct"
            j = np.arange(N, dtype=np.int64)[:, None]
            c = (j + np.arange(K, dtype=np.int64)[None, :] * nu) % N
            if mode == "perm":
                pi = rng.permutation(seed, "perm", N, sub=l)
                cc = np.empty_like(c)
                cc[pi] = c  # column pi(j) <- radix column j
                c = cc
            cols.append(c)
            vals.append(np.full((N, K), weight, dtype=np.float32))
        elif mode == "random":
            keys = rng.u64(seed, "random_idx", np.arange(N * N, dtype=np.uint64), sub=l).reshape(N, N)
            c = np.sort(np.argsort(keys, axis=1, kind="stable")[:, :K], axis=1)
            cols.append(c)
            vals.append(np.full((N, K), weight, dtype=np.float32))
        else:
            raise ValueError(mode)
    b = np.full(L * N, bias, dtype=np.float32)
    return _assemble(N, L, cols, vals, b, ymax, mode, strides)


@dataclasses.dataclass
class CirculantNetwork:
    """Compact form of a radix network: column j of layer l reads (j + n*nu[l]) mod N, n = 0..K-1, in
    that order, with weight w[l, n] (exactly what gen_network(mode="radix") stores as CSC)."""

    N: int
    L: int
    nu: np.ndarray    # int32 [L]
    w: np.ndarray     # float32 [L, K]
    bias: np.ndarray  # float32 [L*N]
    ymax: float

    @property
    def nnz(self) -> int:
        return int(self.L) * int(self.N) * int(self.w.shape[1])

    def to_network(self) -> Network:
        K = self.w.shape[1]
        cols, vals = [], []
        for l in range(self.L):
            j = np.arange(self.N, dtype=np.int64)[:, None]
            cols.append((j + np.arange(K, dtype=np.int64)[None, :] * int(self.nu[l])) % self.N)
            vals.append(np.broadcast_to(self.w[l][None, :], (self.N, K)).astype(np.float32))
        return _assemble(self.N, self.L, cols, vals, self.bias, self.ymax, "radix",
                         radix_strides(self.N))


def gen_circulant(N: int, L: int, K: int = SDGC_K, bias: Optional[float] = None, weight: float = SDGC_WEIGHT,
                  ymax: float = SDGC_YMAX) -> CirculantNetwork:
    """The radix network of gen_network(N, L, "radix") in compact form (no L*N*K index arrays)."""
    if bias is None:
        bias = SDGC_BIAS.get(N, -0.3)
    strides = radix_strides(N)
    nu = np.array([strides[l % len(strides)] for l in range(L)], dtype=np.int32)
    w = np.full((L, K), weight, dtype=np.float32)
    return CirculantNetwork(N=N, L=L, nu=nu, w=w, bias=np.full(L * N, bias, dtype=np.float32), ymax=float(ymax))


def gen_medium_network(N: int = 256, L: int = 18, K: int = 26, seed: int = BASE_SEED) -> Network:
    """Config 5 stand-in: pruned MNIST/CIFAR-shaped sparse MLP, random init.

    K random inputs per column (~90% sparsity at N=256), Kaiming-uniform values over the K real
    inputs, bias U(-0.1, 0.1) per neuron, YMAX = 1.
    """
    cols, vals = [], []
    bound = math.sqrt(6.0 / K)
    for l in range(L):
        keys = rng.u64(seed, "random_idx", np.arange(N * N, dtype=np.uint64), sub=1000 + l).reshape(N, N)
        c = np.sort(np.argsort(keys, axis=1, kind="stable")[:, :K], axis=1)
        u = rng.uniform(seed, "random_val", np.arange(N * K, dtype=np.uint64), sub=l).reshape(N, K)
        cols.append(c)
        vals.append(((2.0 * u - 1.0) * bound).astype(np.float32))
    ub = rng.uniform(seed, "bias", np.arange(L * N, dtype=np.uint64))
    b = ((2.0 * ub - 1.0) * 0.1).astype(np.float32)
    return _assemble(N, L, cols, vals, b, 1.0, "medium")


# ---------------------------------------------------------------- inputs

_TEMPLATE_CACHE: Dict[tuple, np.ndarray] = {}


def _templates(seed: int, radius: float) -> np.ndarray:
    """10 digit-like class templates on a 28x28 canvas: 3 quadratic Bezier strokes each,
    control points inside the centre 20x20 box (MNIST digits occupy the centre 20x20)."""
    key = (seed, radius)
    if key in _TEMPLATE_CACHE:
        return _TEMPLATE_CACHE[key]
    yy, xx = np.mgrid[0:28, 0:28]
    pix = np.stack([xx.ravel() + 0.5, yy.ravel() + 0.5], axis=1)  # [784, 2]
    tt = np.linspace(0.0, 1.0, 96)[:, None]
    out = np.zeros((10, 784), dtype=bool)
    for c in range(10):
        u = rng.uniform(seed, "template", np.arange(18, dtype=np.uint64), sub=c).reshape(3, 3, 2)
        for s in range(3):
            P = 4.0 + 20.0 * u[s]  # 3 control points in [4, 24)^2
            curve = (1 - tt) ** 2 * P[0] + 2 * (1 - tt) * tt * P[1] + tt ** 2 * P[2]  # [96, 2]
            d2 = ((pix[:, None, :] - curve[None, :, :]) ** 2).sum(-1).min(1)
            out[c] |= d2 <= radius * radius
    _TEMPLATE_CACHE[key] = out
    return out


def gen_images(B: int, seed: int = BASE_SEED, radius: float = 2.6, row0: int = 0) -> np.ndarray:
    """B binary 28x28 images (uint8 [B, 784]) for global rows row0 .. row0+B-1.

    Class uniform over 10 (rows arrive shuffled, as PAPER.md:528-529 assumes), shift dx, dy in
    [-2, 2], 5% on-pixel dropout.  Row r's image depends only on (seed, r).
    """
    T = _templates(seed, radius).reshape(10, 28, 28)
    rows = np.arange(row0, row0 + B, dtype=np.uint64)
    cls = rng.randint(seed, "class", rows, 10)
    sh = rng.randint(seed, "shift", rows, 25)
    dx, dy = sh % 5 - 2, sh // 5 - 2
    # 250 shifted templates (class x shift), zero fill
    sht = np.zeros((10, 25, 28, 28), dtype=bool)
    for k in range(25):
        ddx, ddy = k % 5 - 2, k // 5 - 2
        src = T[:, max(0, -ddy):28 - max(0, ddy), max(0, -ddx):28 - max(0, ddx)]
        sht[:, k, max(0, ddy):28 - max(0, -ddy), max(0, ddx):28 - max(0, -ddx)] = src
    img = sht.reshape(250, 784)[cls * 25 + sh]
    drop = rng.uniform(seed, "dropout", rows[:, None] * np.uint64(784) + np.arange(784, dtype=np.uint64)[None, :]) < 0.05
    img = img & ~drop
    return img.astype(np.uint8)


def upscale_index(N: int) -> np.ndarray:
    """Nearest-neighbour map from an S x S (S = sqrt N) output pixel to a 28x28 source pixel."""
    S = int(round(math.isqrt(N)))
    assert S * S == N, "N must be a square (1024, 4096, 16384, 65536)"
    src = (np.arange(S) * 28) // S
    return (src[:, None] * 28 + src[None, :]).reshape(-1)


def gen_inputs(N: int, B: int, seed: int = BASE_SEED, radius: float = 2.6, row0: int = 0,
               out: Optional[np.ndarray] = None) -> np.ndarray:
    """MNIST-like binary inputs Y0, float32 [B, N] row-major, values in {0, 1}."""
    img = gen_images(B, seed, radius, row0)
    m = upscale_index(N)
    if out is None:
        out = np.empty((B, N), dtype=np.float32)
    CH = 4096
    for a in range(0, B, CH):
        out[a:a + CH] = img[a:a + CH][:, m]
    return out


def gen_medium_inputs(N: int, B: int, seed: int = BASE_SEED, row0: int = 0) -> np.ndarray:
    """Config 5 inputs: Y0 = clip(X . W0, 0, 1) for MNIST-like 784-vectors X through a seeded dense
    784 x N layer (input synthesis only; untimed)."""
    X = gen_images(B, seed, 2.6, row0).astype(np.float32)
    W0 = ((rng.uniform(seed, "dense_in", np.arange(784 * N, dtype=np.uint64)).reshape(784, N) * 2 - 1)
          * math.sqrt(6.0 / 784)).astype(np.float32)
    return np.clip(X @ W0, 0.0, 1.0).astype(np.float32)


# ---------------------------------------------------------------- configs (BASELINE.json)

CONFIGS = {
    # name: (N, L, B, description)
    "C1": dict(N=1024, L=120, B=2000, desc="SDGC 1024 neurons x 120 layers, batch 2,000"),
    "C2": dict(N=4096, L=480, B=60000, desc="SDGC 4096 neurons x 480 layers, batch 60,000, 1 B200"),
    "C3": dict(N=16384, L=1920, B=60000, desc="SDGC 16384 neurons x 1920 layers, batch 60,000"),
    "C4": dict(N=65536, L=1920, B=60000, desc="SDGC 65536 neurons x 1920 layers, batch 60,000"),
    "C5": dict(N=256, L=18, B=60000, desc="medium sparse MLP 256 x 18, batch 60,000"),
}

# SNICIT parameters for SDGC: s=32, t=30, n=16, eps=eta=0.03
SNICIT_SDGC = dict(t=30, s=32, n=16, eta=0.03, eps=0.03)
# medium nets: t = largest even <= l/2, s = 128, no downsampling
SNICIT_MEDIUM = dict(s=128, n=0, eta=0.03, eps=0.03)


def medium_t(L: int) -> int:
    t = L // 2
    return t - (t % 2)


def connections(net: Network) -> int:
    """Sum of nnz over layers -- Table 1's 'Connections' column."""
    return net.nnz
