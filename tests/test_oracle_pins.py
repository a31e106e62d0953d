"""Pins for the CPU oracle (oracle/) against what the paper and mathematics fix — never
against the CUDA path.  Each test names the fact it checks (SURVEY §8(c) pins P1-P9)."""
import itertools
import math

import numpy as np
import pytest

import oracle
import synth


def rel(a, b):
    return float(np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300))


# ---------------------------------------------------------------- P1 brute force (tiny grids)
def _slicing_stencil(W, g, T):
    """Independent formulation: out = sum over offsets of W[a] * shifted view (numpy slicing)."""
    h = (W.shape[0] - 1) // 2
    d = W.ndim
    A = g.copy()
    inner = tuple(slice(h, s - h) for s in g.shape)
    for _ in range(T):
        acc = np.zeros_like(A[inner])
        for a in itertools.product(range(2 * h + 1), repeat=d):
            sl = tuple(slice(ai, ai + s - 2 * h) for ai, s in zip(a, g.shape))
            acc += W[a] * A[sl]
        B = A.copy()
        B[inner] = acc
        A = B
    return A


@pytest.mark.parametrize("d,h,shape", [(2, 1, (7, 13)), (2, 3, (9, 11)), (2, 4, (5, 12)), (3, 1, (5, 6, 7)),
                                        (3, 2, (6, 5, 7))])
@pytest.mark.parametrize("kind", ["rsym", "asym"])
def test_P1_matches_slicing_formulation(d, h, shape, kind):
    W = synth.rsym_weights(d, h, 11) if kind == "rsym" else synth.asym_weights(d, h, 12)
    g = synth.grid(tuple(n + 2 * h for n in shape), 20240101)
    assert rel(oracle.run(W, g, 3), _slicing_stencil(W, g, 3)) <= 1e-14


def test_P1_single_point_grid():
    W = synth.rsym_weights(2, 2, 3)
    g = synth.grid((5, 5), 1)
    out = oracle.run(W, g, 1)
    assert out[2, 2] == pytest.approx(float(np.sum(W * g)), rel=1e-15)
    mask = np.ones_like(g, dtype=bool); mask[2, 2] = False
    assert np.array_equal(out[mask], g[mask])


# ---------------------------------------------------------------- P2 constant invariance
@pytest.mark.parametrize("d", [2, 3])
def test_P2_constant_field_bitwise_with_dyadic_weights(d):
    W = synth.dyadic_box_weights(d)
    assert W.sum() == 1.0
    g = synth.constant_grid((12,) * d, 0.75)
    assert np.array_equal(oracle.run(W, g, 10), g)


@pytest.mark.parametrize("d,h", [(2, 3), (3, 1), (2, 1)])
def test_P2_constant_field_rsym(d, h):
    W = synth.rsym_weights(d, h, 5)
    g = synth.constant_grid((10 + 2 * h,) * d, 1.25)
    assert rel(oracle.run(W, g, 20), g) <= 1e-14


# ---------------------------------------------------------------- P3 sine eigenmodes
@pytest.mark.parametrize("name", ["heat2d", "box2d9p", "heat3d", "box3d27p"])
def test_P3_zero_dirichlet_sine_eigenmode(name):
    """Radius-1 reflection-symmetric W with zero halo: A0 = prod sin(pi p_i x_i/(N_i+1)) is an
    eigenvector of one step with lambda = sum_a w_a prod_i cos(pi p_i (a_i - 1)/(N_i+1))."""
    if name == "heat2d":
        W = synth.preset("heat2d"); shape, p = (24, 31), (2, 3)
    elif name == "box2d9p":
        W = synth.rsym_weights(2, 1, 9); shape, p = (24, 31), (3, 1)
    elif name == "heat3d":
        W = synth.preset("heat3d"); shape, p = (12, 9, 14), (1, 2, 3)
    else:
        W = synth.rsym_weights(3, 1, 9); shape, p = (12, 9, 14), (2, 1, 1)
    A0 = synth.sine_grid(shape, p)
    lam = 0.0
    for a in itertools.product(range(3), repeat=len(shape)):
        lam += W[a] * np.prod([math.cos(math.pi * pi * (ai - 1) / (n + 1)) for pi, ai, n in zip(p, a, shape)])
    T = 10
    assert rel(oracle.run(W, A0, T), lam ** T * A0) <= 1e-14


# ---------------------------------------------------------------- P4 plane wave
@pytest.mark.parametrize("kind,T", [("rsym", 12), ("asym", 6)])
def test_P4_plane_wave_in_domain_of_dependence(kind, T):
    """A0 = cos(theta.x) => A_T(x) = Re(lambda^T e^{i theta.x}), lambda = sum_a w_a e^{i theta.(a-h)},
    exact at points at distance >= T*h from the halo (any W, any h)."""
    h = 3
    W = synth.rsym_weights(2, h, 21) if kind == "rsym" else synth.asym_weights(2, h, 22)
    theta = (0.11, -0.07)
    shape = (2 * T * h + 20, 2 * T * h + 17)
    g = synth.plane_wave_grid(tuple(n + 2 * h for n in shape), theta)
    lam = sum(W[a0, a1] * np.exp(1j * (theta[0] * (a0 - h) + theta[1] * (a1 - h)))
              for a0 in range(2 * h + 1) for a1 in range(2 * h + 1))
    out = oracle.run(W, g, T)
    X0, X1 = np.meshgrid(np.arange(g.shape[0]), np.arange(g.shape[1]), indexing="ij")
    exact = np.real(lam ** T * np.exp(1j * (theta[0] * X0 + theta[1] * X1)))
    lo = h + T * h
    sl = (slice(lo, g.shape[0] - lo), slice(lo, g.shape[1] - lo))
    assert rel(out[sl], exact[sl]) <= 1e-13


# ---------------------------------------------------------------- P7 identity / shift
@pytest.mark.parametrize("d", [2, 3])
def test_P7_identity_is_bitwise_copy(d):
    h = 2
    W = np.zeros((2 * h + 1,) * d); W[(h,) * d] = 1.0
    g = synth.grid((9,) * d, 3)
    assert np.array_equal(oracle.run(W, g, 7), g)


def test_P7_shift_with_halo_inflow():
    """W = delta at offset s: A_t[x] = A_{t-1}[x+s]; tracing back, A_T[x] = in[x + k s] for the
    first k <= T that lands in the halo, else in[x + T s].  Exact (bitwise)."""
    h = 2
    s = (1, -2)
    W = np.zeros((5, 5)); W[h + s[0], h + s[1]] = 1.0
    g = synth.grid((11, 14), 8)
    T = 4
    out = oracle.run(W, g, T)
    P0, P1 = g.shape
    exp = g.copy()
    for x0 in range(h, P0 - h):
        for x1 in range(h, P1 - h):
            y0, y1 = x0, x1
            for _ in range(T):
                y0 += s[0]; y1 += s[1]
                if not (h <= y0 < P0 - h and h <= y1 < P1 - h):
                    break
            exp[x0, x1] = g[y0, y1]
    assert np.array_equal(out, exp)


# ---------------------------------------------------------------- P9 integer-exact
@pytest.mark.parametrize("d", [2, 3])
def test_P9_integer_exact_matches_exact_integer_arithmetic(d):
    if d == 2:
        W = synth.integer_pyramid_weights()
        shape = (23, 19)
    else:
        W = np.array([[[1, 2, 1], [2, 4, 2], [1, 2, 1]], [[2, 4, 2], [4, 9, 4], [2, 4, 2]],
                      [[1, 2, 1], [2, 4, 2], [1, 2, 1]]], dtype=np.float64)
        shape = (9, 8, 7)
    h = (W.shape[0] - 1) // 2
    norm1 = np.abs(W).sum()
    T = int((53 - math.log2(3)) // math.log2(norm1))
    assert T >= 3
    g = synth.integer_grid(tuple(n + 2 * h for n in shape), 77)
    Wi = W.astype(np.int64)
    A = g.astype(np.int64)
    inner = tuple(slice(h, s - h) for s in g.shape)
    for _ in range(T):
        acc = np.zeros_like(A[inner])
        for a in itertools.product(range(2 * h + 1), repeat=d):
            sl = tuple(slice(ai, ai + s - 2 * h) for ai, s in zip(a, g.shape))
            acc += Wi[a] * A[sl]
        B = A.copy(); B[inner] = acc; A = B
    assert np.abs(A).max() < 2 ** 53
    assert np.array_equal(oracle.run(W, g, T), A.astype(np.float64))


# ---------------------------------------------------------------- structural properties
def test_thread_count_invariance_bitwise():
    W = synth.rsym_weights(2, 3, 2)
    g = synth.grid((70, 53), 4)
    assert np.array_equal(oracle.run(W, g, 5, threads=1), oracle.run(W, g, 5, threads=8))


def test_T0_is_copy_and_halo_never_written():
    W = synth.rsym_weights(3, 1, 2)
    g = synth.grid((8, 9, 10), 5)
    assert np.array_equal(oracle.run(W, g, 0), g)
    out = oracle.run(W, g, 3)
    inner = np.zeros_like(g, dtype=bool); inner[1:-1, 1:-1, 1:-1] = True
    assert np.array_equal(out[~inner], g[~inner])


def test_linearity():
    W = synth.asym_weights(2, 2, 9, signed=True)
    a = synth.grid((20, 21), 1); b = synth.grid((20, 21), 2)
    lhs = oracle.run(W, 0.3 * a - 1.7 * b, 4)
    rhs = 0.3 * oracle.run(W, a, 4) - 1.7 * oracle.run(W, b, 4)
    assert rel(lhs, rhs) <= 1e-13


@pytest.mark.parametrize("d,h,shape,T", [(2, 3, (60, 47), 5), (3, 1, (13, 17, 11), 4)])
def test_point_window_equals_full_run(d, h, shape, T):
    W = synth.rsym_weights(d, h, 31)
    g = synth.grid(tuple(n + 2 * h for n in shape), 6)
    full = oracle.run(W, g, T)
    rng = np.random.default_rng(0)
    pts = [tuple(h for _ in shape), tuple(s + h - 1 for s in shape)]
    pts += [tuple(int(rng.integers(0, s + 2 * h)) for s in shape) for _ in range(6)]
    for p in pts:
        assert oracle.point(W, g, T, p) == full[p]


# ---------------------------------------------------------------- PMA (paper §III-C, eq. 15)
@pytest.mark.parametrize("h", [1, 2, 3, 4])
def test_pma_pyramid_sizes_reconstruction_and_rank(h):
    W = synth.rsym_weights(2, h, 100 + h)
    terms = oracle.pma(W)
    assert [len(u) for u, _ in terms] == [2 * h + 3 - 2 * i for i in range(1, h + 2)]   # eq. 15
    assert np.abs(oracle.pma_reconstruct(terms, 2 * h + 1) - W).max() <= 1e-15 * np.abs(W).max()
    assert np.linalg.matrix_rank(W) <= h + 1
    # C1 shares W's first/last row and the first/last element of the middle rows
    u, v = terms[0]
    C1 = np.outer(u, v)
    R = W - C1
    assert np.abs(R[0, :]).max() <= 1e-17 and np.abs(R[-1, :]).max() <= 1e-17
    assert np.abs(R[:, 0]).max() <= 1e-17 and np.abs(R[:, -1]).max() <= 1e-17
    for u, v in terms:                                                                    # P:271 symmetry
        assert np.allclose(u, u[::-1], rtol=0, atol=1e-15) and np.allclose(v, v[::-1], rtol=0, atol=1e-17)


def test_pma_integer_pyramid_is_exact():
    W = synth.integer_pyramid_weights()
    terms = oracle.pma(W)
    assert np.array_equal(terms[0][0], [1, 2, 3, 4, 3, 2, 1]) and np.array_equal(terms[0][1], [1, 2, 3, 4, 3, 2, 1])
    assert np.array_equal(terms[1][0], [1, 1, 2, 1, 1]) and np.array_equal(terms[1][1], [1, 1, 2, 1, 1])
    assert np.array_equal(terms[2][0], [1, 2, 1]) and np.array_equal(terms[2][1], [2, 4, 2])
    assert terms[3][1][0] == 3.0
    assert np.array_equal(oracle.pma_reconstruct(terms, 7), W)


def test_pma_zero_pivot_raises_for_star():
    with pytest.raises(ZeroDivisionError):
        oracle.pma(synth.preset("heat2d"))


# ---------------------------------------------------------------- RDG (eq. 5-9)
@pytest.mark.parametrize("h,m", [(1, 8), (3, 8), (4, 16)])
def test_rdg_chain_equals_direct_correlation(h, m):
    """Eq. 7: for C = u v^T, U X V equals the one-step stencil on the (m+2h)^2 tile."""
    rng = np.random.default_rng(h)
    u = rng.uniform(0.1, 1, 2 * h + 1); v = rng.uniform(0.1, 1, 2 * h + 1)
    X = synth.grid((m + 2 * h, m + 2 * h), 3)
    got = oracle.rdg_tile(u, v, X)
    ref = oracle.run(np.outer(u, v), X, 1)[h:-h, h:-h]
    assert rel(got, ref) <= 1e-14


def test_rdg_band_shapes_eq5_eq6():
    u = np.array([1.0, 2.0, 3.0])
    U = oracle.rdg_band_U(u, 4)
    assert U.shape == (4, 6) and np.array_equal(U[0, :3], u) and np.array_equal(U[3, 3:], u) and U[0, 3] == 0
    V = oracle.rdg_band_V(u, 4)
    assert V.shape == (6, 4) and np.array_equal(V[:3, 0], u) and np.array_equal(V[3:, 3], u)


def test_rdg_pma_sum_equals_direct_eq9():
    h = 3
    W = synth.rsym_weights(2, h, 44)
    X = synth.grid((8 + 2 * h, 8 + 2 * h), 9)
    acc = np.zeros((8, 8))
    for u, v in oracle.pma(W):
        k = (len(u) - 1) // 2
        o = h - k
        Xs = X[o:X.shape[0] - o, o:X.shape[1] - o]
        acc += oracle.rdg_tile(u, v, Xs)
    ref = oracle.run(W, X, 1)[h:-h, h:-h]
    assert rel(acc, ref) <= 1e-14


# ---------------------------------------------------------------- 1D (Table II Heat-1D / 1D5P)
def test_1d_sine_eigenmode():
    """Radius-1 or -2 symmetric 1D stencil with zero halo: A0 = sin(pi p x/(N+1)) (x = padded
    index, radius-1 halo) is an eigenvector with lambda = sum_a w_a cos(pi p (a-1)/(N+1))."""
    W = np.array([0.25, 0.5, 0.25]); N, p = 37, 3
    A0 = np.sin(math.pi * p * np.arange(N + 2) / (N + 1)); A0[0] = A0[-1] = 0.0
    lam = sum(W[a] * math.cos(math.pi * p * (a - 1) / (N + 1)) for a in range(3))
    assert rel(oracle.run(W, A0, 20), lam ** 20 * A0) <= 1e-14


def test_1d_plane_wave_and_bruteforce():
    W = np.array([0.1, 0.2, 0.4, 0.2, 0.1])   # 1D5P-like
    h, T, N = 2, 7, 80
    theta = 0.13
    g = np.cos(theta * np.arange(N + 2 * h))
    lam = sum(W[a] * np.exp(1j * theta * (a - h)) for a in range(5))
    out = oracle.run(W, g, T)
    x = np.arange(N + 2 * h)
    sl = slice(h + T * h, N + h - T * h)
    assert rel(out[sl], np.real(lam ** T * np.exp(1j * theta * x))[sl]) <= 1e-13
    g2 = synth.grid((N + 2 * h,), 5)
    assert rel(oracle.run(W, g2, 3), _slicing_stencil(W, g2, 3)) <= 1e-14


def test_1d_integer_exact():
    W = np.array([1.0, 2.0, 1.0])
    g = synth.integer_grid((50,), 3)
    A = g.astype(np.int64)
    for _ in range(20):
        B = A.copy(); B[1:-1] = A[:-2] + 2 * A[1:-1] + A[2:]; A = B
    assert np.array_equal(oracle.run(W, g, 20), A.astype(np.float64))
