"""Closed-form pins through the CUDA path (-m gpu), at the sizes SURVEY.md §8(c) names.

These compare the GPU result with the MATHEMATICS, not with the oracle: P3 (zero-Dirichlet sine
eigenmode), P4 (plane wave inside the domain of dependence), P6 (rank-1 W: one term, two 1D
passes), P8 (linearity).  The same pins hold the oracle in tests/test_oracle_pins.py."""
import itertools
import math

import numpy as np
import pytest

import synth
from tests._gpu_helpers import rel_err, run_gpu

pytestmark = pytest.mark.gpu


def _lambda_sine(W, shape, p):
    lam = 0.0
    for a in itertools.product(range(3), repeat=len(shape)):
        lam += W[a] * np.prod([math.cos(math.pi * pi * (ai - 1) / (n + 1)) for pi, ai, n in zip(p, a, shape)])
    return lam


@pytest.mark.parametrize("engine", ["auto", "tc", "rdg_cuda", "direct"])
@pytest.mark.parametrize("name", ["heat2d", "box2d9p", "heat3d", "box3d27p"])
def test_P3_sine_eigenmode_gpu_T100(name, engine):
    """P3: radius-1 reflection-symmetric W, zero halo, A0 = prod sin(pi p x/(N+1))
    => A_T = lambda^T A0, at 1024^2 / 128^3 and T = 100 (every engine; auto fuses)."""
    if name == "heat2d":
        W = synth.preset("heat2d"); shape, p = (1024, 1024), (1, 2)
    elif name == "box2d9p":
        W = synth.rsym_weights(2, 1, 9); shape, p = (1024, 1000), (2, 1)
    elif name == "heat3d":
        W = synth.preset("heat3d"); shape, p = (128, 128, 128), (1, 1, 2)
    else:
        W = synth.rsym_weights(3, 1, 9); shape, p = (128, 120, 128), (1, 2, 1)
    A0 = synth.sine_grid(shape, p)
    T = 100
    lam = _lambda_sine(W, shape, p)
    out, _ = run_gpu(W, A0, T, engine=engine)
    assert rel_err(out, lam ** T * A0) <= 1e-13


@pytest.mark.parametrize("engine", ["auto", "tc", "rdg_cuda"])
@pytest.mark.parametrize("kind", ["rsym", "asym"])
def test_P4_plane_wave_box2d49p_gpu(kind, engine):
    """P4: A0 = cos(theta.x) => A_T(x) = Re(lambda^T e^{i theta.x}) at distance >= T h from the
    halo; Box-2D49P (h = 3) at 1024^2, T = 100 (both weight kinds are convex, so |lambda| <= 1)."""
    h = 3
    T = 100
    W = synth.rsym_weights(2, h, 21) if kind == "rsym" else synth.asym_weights(2, h, 22)
    theta = (0.011, -0.007)
    shape = (1024, 1024)
    g = synth.plane_wave_grid(tuple(n + 2 * h for n in shape), theta)
    lam = sum(W[a0, a1] * np.exp(1j * (theta[0] * (a0 - h) + theta[1] * (a1 - h)))
              for a0 in range(2 * h + 1) for a1 in range(2 * h + 1))
    out, _ = run_gpu(W, g, T, engine=engine)
    X0, X1 = np.meshgrid(np.arange(g.shape[0]), np.arange(g.shape[1]), indexing="ij")
    exact = np.real(lam ** T * np.exp(1j * (theta[0] * X0 + theta[1] * X1)))
    lo = h + T * h
    sl = (slice(lo, g.shape[0] - lo), slice(lo, g.shape[1] - lo))
    assert rel_err(out[sl], exact[sl]) <= 1e-13


@pytest.mark.parametrize("engine", ["auto", "tc", "rdg_cuda"])
def test_P4_plane_wave_box3d27p_gpu(engine):
    h, T = 1, 40
    W = synth.rsym_weights(3, h, 23)
    theta = (0.05, 0.03, -0.02)
    shape = (128, 128, 128)
    g = synth.plane_wave_grid(tuple(n + 2 * h for n in shape), theta)
    lam = 0.0
    for a in itertools.product(range(3), repeat=3):
        lam += W[a] * np.exp(1j * sum(t * (ai - h) for t, ai in zip(theta, a)))
    out, _ = run_gpu(W, g, T, engine=engine)
    X = np.meshgrid(*[np.arange(n) for n in g.shape], indexing="ij")
    exact = np.real(lam ** T * np.exp(1j * sum(t * x for t, x in zip(theta, X))))
    lo = h + T * h
    sl = tuple(slice(lo, n - lo) for n in g.shape)
    assert rel_err(out[sl], exact[sl]) <= 1e-13


@pytest.mark.parametrize("engine", ["auto", "tc", "rdg_cuda", "direct"])
@pytest.mark.parametrize("d", [2, 3])
def test_P8_linearity_gpu(engine, d):
    """P8: run(alpha A + beta B) = alpha run(A) + beta run(B) (signed weights, T = 4)."""
    h = 2 if d == 2 else 1
    W = synth.asym_weights(d, h, 9, signed=True)
    shape = (70, 131) if d == 2 else (9, 17, 33)
    pad = tuple(n + 2 * h for n in shape)
    a, b = synth.grid(pad, 1), synth.grid(pad, 2)
    lhs, _ = run_gpu(W, 0.3 * a - 1.7 * b, 4, engine=engine)
    ra, _ = run_gpu(W, a, 4, engine=engine)
    rb, _ = run_gpu(W, b, 4, engine=engine)
    assert rel_err(lhs, 0.3 * ra - 1.7 * rb) <= 1e-13


@pytest.mark.parametrize("engine", ["auto", "tc", "rdg_cuda"])
@pytest.mark.parametrize("h", [1, 2, 3, 4])
def test_P6_rank1_is_two_1d_passes(engine, h):
    """P6 ("LoRAStencil-Best"): W = u v^T plans ONE term and equals a vertical 1D pass
    followed by a horizontal one (computed here with numpy slicing, T = 3)."""
    rng = np.random.default_rng(100 + h)
    u = rng.uniform(0.1, 1.0, 2 * h + 1); u /= u.sum()
    v = rng.uniform(0.1, 1.0, 2 * h + 1); v /= v.sum()
    W = np.multiply.outer(u, v)
    shape = (67, 129)
    g = synth.grid(tuple(n + 2 * h for n in shape), 7 + h)
    T = 3
    out, info = run_gpu(W, g, T, engine=engine)
    assert info["n_terms"] == 1
    A = g.copy()
    for _ in range(T):
        tmp = np.zeros((shape[0], shape[1] + 2 * h))
        for i in range(2 * h + 1):             # vertical pass over every padded column
            tmp += u[i] * A[i:i + shape[0], :]
        B = A.copy()
        B[h:-h, h:-h] = 0.0
        for j in range(2 * h + 1):             # horizontal pass
            B[h:-h, h:-h] += v[j] * tmp[:, j:j + shape[1]]
        A = B
    assert rel_err(out, A) <= 1e-13
