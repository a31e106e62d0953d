"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This module holds NO stencil arithmetic: it only draws grids and weight arrays.  It is the
one piece of code both sides of the parity check may use (task rule ③).  The recipe is
DESIGN.md §"Input recipe" and SURVEY.md §8(d):

* Grid values: the standard SplitMix64 stream indexed by the linear index ``i`` into the
  WHOLE padded array (halo included), ``x_i = 0.5 + (z >> 11) * 2**-53`` in [0.5, 1.5).
* "rsym" weights: one draw per symmetry class of the offset (class id = lexicographic
  rank of the sorted |offset| tuple), ``w = 0.1 + 0.9 * u``, normalised so sum(W) = 1.
  This is the "radially symmetric" weight matrix of PAPER.md P:88-92 (Fig. 2): points at
  the same distance pattern share a weight.
* Presets (textbook weights; the paper does not print its weights, P:390 / Table II).

All arrays are float64 numpy arrays in C order; 2D shapes are (N0+2h, N1+2h), 3D shapes
(N0+2h, N1+2h, N2+2h), slowest axis first.
"""
from __future__ import annotations

import itertools
import math

import numpy as np

__all__ = [
    "splitmix64", "uniform_from_index", "grid", "rsym_weights", "star_weights", "preset",
    "CONFIGS", "config", "integer_pyramid_weights", "integer_grid", "asym_weights",
    "constant_grid", "sine_grid", "plane_wave_grid", "dyadic_box_weights", "grid_torch",
]

_GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(seed: int, idx: np.ndarray) -> np.ndarray:
    """z = seed + (i+1)*gamma; standard SplitMix64 finaliser (all arithmetic mod 2**64)."""
    idx = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed % (1 << 64)) + (idx + np.uint64(1)) * _GAMMA
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform_from_index(seed: int, idx: np.ndarray) -> np.ndarray:
    """Doubles in [0.5, 1.5): 0.5 + (z >> 11) * 2**-53 (exact in binary64)."""
    z = splitmix64(seed, idx)
    return 0.5 + (z >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def grid(padded_shape, seed: int, chunk: int = 1 << 24) -> np.ndarray:
    """Whole padded grid (halo included) from the SplitMix64 stream, chunked to bound memory."""
    n = int(np.prod(padded_shape))
    out = np.empty(n, dtype=np.float64)
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        out[s:e] = uniform_from_index(seed, np.arange(s, e, dtype=np.uint64))
    return out.reshape(tuple(int(x) for x in padded_shape))


def _classes(ndim: int, radius: int, star: bool):
    """Symmetry classes: sorted |offset| tuples, lexicographically ranked."""
    cls = sorted({tuple(sorted(t)) for t in itertools.product(range(radius + 1), repeat=ndim)})
    if star:
        cls = [c for c in cls if sum(1 for x in c if x) <= 1]
    return cls


def grid_torch(padded_shape, seed: int, device="cuda", chunk: int = 1 << 26):
    """The same SplitMix64 grid as `grid`, generated with torch int64 arithmetic on `device`
    (bit-identical: int64 multiply wraps like uint64; logical shifts are emulated with masks).
    For grids too large to build on the host."""
    import torch
    n = 1
    for d in padded_shape:
        n *= int(d)
    out = torch.empty(n, dtype=torch.float64, device=device)

    def u64(x):  # python int -> int64 with the same bits
        x &= (1 << 64) - 1
        return x - (1 << 64) if x >= 1 << 63 else x

    gamma, m1, m2 = u64(0x9E3779B97F4A7C15), u64(0xBF58476D1CE4E5B9), u64(0x94D049BB133111EB)

    def lsr(z, k):
        return (z >> k) & ((1 << (64 - k)) - 1)

    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        i = torch.arange(s, e, dtype=torch.int64, device=device)
        z = u64(seed) + (i + 1) * gamma
        z = (z ^ lsr(z, 30)) * m1
        z = (z ^ lsr(z, 27)) * m2
        z = z ^ lsr(z, 31)
        out[s:e] = 0.5 + lsr(z, 11).to(torch.float64) * (2.0 ** -53)
    return out.view(*[int(d) for d in padded_shape])


def rsym_weights(ndim: int, radius: int, seed: int, star: bool = False) -> np.ndarray:
    """Random radially symmetric weights: one U[0.1,1) value per class, sum 1."""
    cls = _classes(ndim, radius, star)
    draws = 0.1 + 0.9 * (splitmix64(seed + 7777, np.arange(len(cls), dtype=np.uint64)) >> np.uint64(11)).astype(
        np.float64) * (2.0 ** -53)
    val = {c: float(draws[i]) for i, c in enumerate(cls)}
    n = 2 * radius + 1
    W = np.zeros((n,) * ndim)
    for off in itertools.product(range(n), repeat=ndim):
        key = tuple(sorted(abs(o - radius) for o in off))
        if key in val:
            W[off] = val[key]
    return W / W.sum()


def star_weights(ndim: int, radius: int, seed: int) -> np.ndarray:
    return rsym_weights(ndim, radius, seed, star=True)


def asym_weights(ndim: int, radius: int, seed: int, signed: bool = False) -> np.ndarray:
    """General (non-symmetric) weights; convex unless ``signed`` (then ||W||_1 = 1.5)."""
    n = (2 * radius + 1) ** ndim
    u = uniform_from_index(seed + 4242, np.arange(n, dtype=np.uint64)) - 0.5  # [0,1)
    if signed:
        w = (2.0 * u - 1.0)
        w = 1.5 * w / np.abs(w).sum()
    else:
        w = 0.1 + u
        w = w / w.sum()
    return w.reshape((2 * radius + 1,) * ndim)


def dyadic_box_weights(ndim: int) -> np.ndarray:
    """[1,2,1]^{(x)d} / 4^d: exactly representable, sums to exactly 1 (pin P2)."""
    v = np.array([1.0, 2.0, 1.0]) / 4.0
    W = v
    for _ in range(ndim - 1):
        W = np.multiply.outer(W, v)
    return W


def preset(name: str) -> np.ndarray:
    """Named textbook weights (not from the paper, which prints none: P:390)."""
    if name == "heat2d":  # 5-point star, c = 0.5, arms 0.125
        W = np.zeros((3, 3)); W[1, 1] = 0.5; W[0, 1] = W[2, 1] = W[1, 0] = W[1, 2] = 0.125
        return W
    if name == "heat1d":  # 3-point, c = 0.5, arms 0.25
        return np.array([0.25, 0.5, 0.25])
    if name == "heat3d":  # 7-point star, c = 0.25, arms 0.125
        W = np.zeros((3, 3, 3)); W[1, 1, 1] = 0.25
        for a in range(3):
            for s in (0, 2):
                idx = [1, 1, 1]; idx[a] = s; W[tuple(idx)] = 0.125
        return W
    raise KeyError(name)


def integer_pyramid_weights():
    """Integer-exact mode (pin P9): W = sum_r s_r u_r u_r^T with integer palindromic u_r
    (u_r[0] = 1) nested as a pyramid plus an integer centre.  Returns (W, terms) where
    terms = [(s, u)] and the centre scalar is the last entry with u = [1]."""
    u1 = np.array([1, 2, 3, 4, 3, 2, 1], dtype=np.float64)
    u2 = np.array([1, 1, 2, 1, 1], dtype=np.float64)
    u3 = np.array([1, 2, 1], dtype=np.float64)
    W = np.zeros((7, 7))
    W += 1.0 * np.outer(u1, u1)
    W[1:6, 1:6] += 1.0 * np.outer(u2, u2)
    W[2:5, 2:5] += 2.0 * np.outer(u3, u3)
    W[3, 3] += 3.0
    return W


def integer_grid(padded_shape, seed: int) -> np.ndarray:
    """Integers in {0,1,2,3} from the same SplitMix64 stream (z >> 62)."""
    n = int(np.prod(padded_shape))
    z = splitmix64(seed, np.arange(n, dtype=np.uint64))
    return (z >> np.uint64(62)).astype(np.float64).reshape(tuple(padded_shape))


def constant_grid(padded_shape, value: float = 0.75) -> np.ndarray:
    return np.full(tuple(padded_shape), value, dtype=np.float64)


def sine_grid(interior_shape, modes) -> np.ndarray:
    """Zero-Dirichlet sine mode prod_i sin(pi p_i x_i/(N_i+1)) on a radius-1 padded grid
    (x_i = padded index, so the halo rows x_i = 0 and N_i+1 are exactly zero)."""
    axes = []
    for n, p in zip(interior_shape, modes):
        x = np.arange(n + 2, dtype=np.float64)
        s = np.sin(math.pi * p * x / (n + 1))
        s[0] = 0.0; s[-1] = 0.0
        axes.append(s)
    G = axes[0]
    for a in axes[1:]:
        G = np.multiply.outer(G, a)
    return G


def plane_wave_grid(padded_shape, theta) -> np.ndarray:
    """cos(theta . x) over the padded index x (halo included)."""
    idx = np.meshgrid(*[np.arange(n, dtype=np.float64) for n in padded_shape], indexing="ij")
    ph = sum(t * x for t, x in zip(theta, idx))
    return np.cos(ph)


# BASELINE.json configs (index = config id; seed = 20240101 + id).
CONFIGS = {
    "heat2d-256": dict(id=0, ndim=2, radius=1, shape=(256, 256), T=10, weights="heat2d"),
    "box2d9p-10240": dict(id=1, ndim=2, radius=1, shape=(10240, 10240), T=100, weights="rsym"),
    "box2d49p-10240": dict(id=2, ndim=2, radius=3, shape=(10240, 10240), T=100, weights="rsym"),
    "heat3d-512": dict(id=3, ndim=3, radius=1, shape=(512, 512, 512), T=100, weights="heat3d"),
    "box3d27p-512": dict(id=4, ndim=3, radius=1, shape=(512, 512, 512), T=100, weights="rsym"),
    "box2d49p-40960": dict(id=5, ndim=2, radius=3, shape=(40960, 40960), T=100, weights="rsym"),
    "box3d27p-1024": dict(id=6, ndim=3, radius=1, shape=(1024, 1024, 1024), T=100, weights="rsym"),
    # the remaining Table II kernels at BASELINE-like sizes
    "star2d13p-10240": dict(id=7, ndim=2, radius=3, shape=(10240, 10240), T=100, weights="star"),
    "heat1d-10240000": dict(id=8, ndim=1, radius=1, shape=(10240000,), T=100, weights="heat1d"),
    "1d5p-10240000": dict(id=9, ndim=1, radius=2, shape=(10240000,), T=100, weights="rsym"),
}


def config(name: str):
    """Returns (W, cfg) for a named config; W from its weight recipe and seed."""
    c = dict(CONFIGS[name])
    c["seed"] = 20240101 + c["id"]
    if c["weights"] == "rsym":
        W = rsym_weights(c["ndim"], c["radius"], c["seed"])
    elif c["weights"] == "star":
        W = star_weights(c["ndim"], c["radius"], c["seed"])
    else:
        W = preset(c["weights"])
    c["padded"] = tuple(n + 2 * c["radius"] for n in c["shape"])
    return W, c
