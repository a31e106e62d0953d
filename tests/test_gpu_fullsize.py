"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (-m gpu):
the CUDA path runs the whole config (full grid, full T); the oracle computes sampled outputs one
by one on their domain of dependence (oracle.point).  Bar: the north star's 1e-10 relative."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

CONFIGS = ["heat2d-256", "box2d9p-10240", "box2d49p-10240", "heat3d-512", "box3d27p-512"]


def _sample_points(padded, h, n_random=5, seed=0):
    rng = np.random.default_rng(seed)
    P = padded
    pts = [tuple(h for _ in P), tuple(s - h - 1 for s in P), tuple(s // 2 for s in P),
           tuple(h if i == 0 else s - h - 1 for i, s in enumerate(P)), tuple(h + 1 for _ in P)]
    pts += [tuple(int(rng.integers(h, s - h)) for s in P) for _ in range(n_random)]
    return pts


@pytest.mark.parametrize("engine", ["auto", "tc"])
@pytest.mark.parametrize("name", CONFIGS)
def test_fullsize_sampled_parity(name, engine):
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W, c = synth.config(name)
    g = synth.grid(c["padded"], c["seed"])
    st = L.Stencil(W, c["shape"], engine=engine)
    x = torch.from_numpy(g).cuda()
    y = torch.empty_like(x)
    st.run(x, y, c["T"])
    torch.cuda.synchronize()
    h = c["radius"]
    pts = _sample_points(c["padded"], h, n_random=4 if c["ndim"] == 3 else 6)
    idx = tuple(torch.tensor([p[i] for p in pts]) for i in range(c["ndim"]))
    got = y[idx].cpu().numpy()
    scale = float(torch.max(torch.abs(y)).item())
    for p, gv in zip(pts, got):
        ref = oracle.point(W, g, c["T"], p)
        assert abs(gv - ref) / scale <= 1e-10, (name, p, gv, ref)
    # the halo is a bitwise copy of the input halo
    ys = y.cpu().numpy()
    sl = tuple(slice(h, -h) for _ in range(c["ndim"]))
    mask = np.ones(c["padded"], dtype=bool)
    mask[sl] = False
    assert np.array_equal(ys[mask], g[mask])
    st.close()


@pytest.mark.parametrize("name", ["box2d49p-10240", "box3d27p-512"])
def test_fullsize_constant_field_invariance(name):
    """Sum(W) = 1 => a constant field is a fixed point (north-star pin), at full size and T."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W, c = synth.config(name)
    st = L.Stencil(W, c["shape"])
    x = torch.full(c["padded"], 0.75, dtype=torch.float64, device="cuda")
    y = torch.empty_like(x)
    st.run(x, y, c["T"])
    torch.cuda.synchronize()
    assert float(torch.max(torch.abs(y - 0.75)).item()) <= 1e-13
    st.close()


@pytest.mark.parametrize("name,T", [("box2d49p-40960", 2), ("box3d27p-1024", 2)])
def test_multigpu_global_size_on_one_gpu(name, T):
    """The multi-GPU global shapes (40960^2: 13.4 GB per buffer; 1024^3) on one B200: sampled
    outputs vs the oracle on their domain of dependence (grid generated on the GPU, bit-identical
    to synth.grid; the oracle's windows are rebuilt on the host from the same index formula)."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W, c = synth.config(name)
    h = c["radius"]
    P = c["padded"]
    x = synth.grid_torch(P, c["seed"])
    y = torch.empty_like(x)
    st = L.Stencil(W, c["shape"])
    st.run(x, y, T)
    torch.cuda.synchronize()
    rng = np.random.default_rng(1)
    pts = [tuple(h for _ in P), tuple(s - h - 1 for s in P), tuple(s // 2 for s in P)]
    pts += [tuple(int(rng.integers(h, s - h)) for s in P) for _ in range(3)]
    scale = 1.5
    for p in pts:
        Rw = T * h + h
        lo = [max(0, i - Rw) for i in p]
        hi = [min(s, i + Rw + 1) for i, s in zip(p, P)]
        idx = np.stack(np.meshgrid(*[np.arange(a, b) for a, b in zip(lo, hi)], indexing="ij"), -1)
        lin = np.ravel_multi_index(tuple(np.moveaxis(idx, -1, 0)), P).astype(np.uint64)
        win = synth.uniform_from_index(c["seed"], lin)
        ref = oracle.run(W, win, T)[tuple(i - a for i, a in zip(p, lo))]
        got = float(y[p].item())
        assert abs(got - ref) / scale <= 1e-12, (name, p, got, ref)
    st.close()
    del x, y
    torch.cuda.empty_cache()
