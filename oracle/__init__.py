"""TEST INFRASTRUCTURE ONLY — CPU oracle for the LoRAStencil hot path.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product package never imports it; the
two share no code (the seeded generators in ``synth/`` are the only common module).

Contents
* ``run``      — the direct Dirichlet-halo Jacobi stencil (eq. 2),
                 plain C loops in ``stencil_oracle.c`` (fp64, no FMA contraction, OpenMP).
* ``point``    — one output value at full size, by running ``run`` on the domain of
                 dependence of that point (a window of half-width T*h + h).  Same arithmetic
                 as ``run``; no new formula.
* ``pma``      — Pyramidal Matrix Adaptation step by step as PAPER.md §III-C (eq 15).
* ``rdg``      — the banded Toeplitz U, V of eq. 5-6 and the chain U X V of eq. 7.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "stencil_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C, OpenMP).  Returns the .so path."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.oracle_stencil_run.restype = ctypes.c_int
        _lib.oracle_stencil_run.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                                            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int]
        _lib.oracle_max_threads.restype = ctypes.c_int
    return _lib


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def run(W: np.ndarray, grid: np.ndarray, T: int, threads: int = 0) -> np.ndarray:
    """T Jacobi steps of the direct stencil on a padded grid; returns a new padded array.

    W has shape (2h+1,)*d, grid has shape (N_i + 2h) per axis (d = 1, 2 or 3)."""
    W = np.ascontiguousarray(W, dtype=np.float64)
    grid = np.ascontiguousarray(grid, dtype=np.float64)
    d = W.ndim
    h = (W.shape[0] - 1) // 2
    assert d in (1, 2, 3) and all(s == 2 * h + 1 for s in W.shape) and grid.ndim == d
    N = np.array([s - 2 * h for s in grid.shape], dtype=np.int64)
    out = np.empty_like(grid)
    rc = _load().oracle_stencil_run(W.ctypes.data, d, h, N.ctypes.data, grid.ctypes.data, out.ctypes.data,
                                    int(T), int(threads))
    if rc != 0:
        raise ValueError("oracle_stencil_run rejected its arguments")
    return out


def point(W: np.ndarray, grid: np.ndarray, T: int, idx, threads: int = 0) -> float:
    """Value at padded index ``idx`` after T steps, from the domain of dependence only.

    A window of half-width T*h + h around idx (clipped to the padded array) is stepped with
    ``run``: its outer ring of width h is held fixed; where that ring is not the true halo it
    is stale from step 2 on, and the staleness advances h cells per step, so it reaches
    (T-1)*h cells inward after T steps — never the centre.  Halo points return the input."""
    W = np.asarray(W, dtype=np.float64)
    h = (W.shape[0] - 1) // 2
    idx = tuple(int(i) for i in idx)
    if any(i < h or i >= s - h for i, s in zip(idx, grid.shape)) or T == 0:
        return float(grid[idx])
    R = T * h + h
    lo = [max(0, i - R) for i in idx]
    hi = [min(s, i + R + 1) for i, s in zip(idx, grid.shape)]
    win = np.ascontiguousarray(grid[tuple(slice(a, b) for a, b in zip(lo, hi))])
    res = run(W, win, T, threads)
    return float(res[tuple(i - a for i, a in zip(idx, lo))])


def pma(W: np.ndarray):
    """Pyramidal Matrix Adaptation, §III-C P:265-288 (Fig. 5, eq. 15), in its order.

    For the current (2k+1)x(2k+1) radially symmetric remainder R (initially W):
      u = R[:, 0] / R[0, 0]   ("the i-th row of C1 is w_{i,1}/w_{1,1} x w_{1,:}")
      v = R[0, :]
      C = u (x) v^T;  R <- (R - C)[1:-1, 1:-1]  (the border of R - C is zero)
    until R is 1x1, which is the scalar term C_{h+1} ("no additional MM").
    Returns a list of (u, v) with len(u) = 2h+3-2i for i = 1..h+1 (eq. 15).  Raises
    ZeroDivisionError when a pivot R[0,0] is zero (the paper assumes rank(W) = h+1, P:262;
    DESIGN.md reading Q6 covers what the product does then)."""
    R = np.array(W, dtype=np.float64)
    terms = []
    while R.shape[0] > 1:
        if R[0, 0] == 0.0:
            raise ZeroDivisionError("PMA pivot w_{1,1} is zero")
        u = R[:, 0] / R[0, 0]
        v = R[0, :].copy()
        terms.append((u, v))
        R = (R - np.outer(u, v))[1:-1, 1:-1]
    terms.append((np.array([1.0]), np.array([R[0, 0]])))
    return terms


def pma_reconstruct(terms, n: int) -> np.ndarray:
    """Sum of the pyramid of rank-1 matrices C_i embedded centred in an n x n matrix (eq. 15)."""
    W = np.zeros((n, n))
    for u, v in terms:
        m = len(u)
        o = (n - m) // 2
        W[o:o + m, o:o + m] += np.outer(u, v)
    return W


def rdg_band_U(u: np.ndarray, m: int) -> np.ndarray:
    """Eq. 5: U is m x (m+2h), u_{i,j} = u_{j-i+1} for i <= j <= i+2h (1-based)."""
    n = len(u)
    h = (n - 1) // 2
    U = np.zeros((m, m + 2 * h))
    for i in range(1, m + 1):
        for j in range(i, i + 2 * h + 1):
            U[i - 1, j - 1] = u[j - i]          # u_{j-i+1}, 1-based -> index j-i
    return U


def rdg_band_V(v: np.ndarray, m: int) -> np.ndarray:
    """Eq. 6: V is (m+2h) x m, v_{i,j} = v_{i-j+1} for j <= i <= j+2h (1-based)."""
    n = len(v)
    h = (n - 1) // 2
    V = np.zeros((m + 2 * h, m))
    for j in range(1, m + 1):
        for i in range(j, j + 2 * h + 1):
            V[i - 1, j - 1] = v[i - j]
    return V


def rdg_tile(u: np.ndarray, v: np.ndarray, X: np.ndarray) -> np.ndarray:
    """Eq. 7: <C, X>_FT = U X V for an (m+2h) x (m+2h) tile X -> m x m results."""
    m = X.shape[0] - (len(u) - 1)
    return rdg_band_U(u, m) @ X @ rdg_band_V(v, m)
