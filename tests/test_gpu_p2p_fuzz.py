"""Seeded random sweep of the device-initiated halo exchange (lora_stencil_run_dist_p2p) on one
GPU (-m gpu): 2-4 slab ranks in one process on concurrent streams, random global shapes, uneven
splits (every slab >= the deep-halo depth), fusion depths with remainder launches, 2D and 3D, the
CUDA-core engine and the direct kernel.  The gathered slabs must equal the single-GPU run of the
global grid BITWISE (pin P10)."""
import numpy as np
import pytest

import synth
from tests.test_gpu_p2p import _global, _run_local, _weights

pytestmark = pytest.mark.gpu


def _case(i):
    rng = np.random.default_rng(4048 + i)
    d = 2 if rng.random() < 0.65 else 3
    h = int(rng.integers(1, 4)) if d == 2 else 1
    kind = str(rng.choice(["rsym", "star", "asym"] if d == 2 else ["rsym", "heat3d", "asym"]))
    engine = "direct" if rng.random() < 0.15 else "rdg_cuda"
    if engine == "direct" or kind == "asym":
        k = 1
    else:
        k = int(rng.integers(1, ({1: 4, 2: 3, 3: 2}[h] if d == 2 else 3) + 1))
    P = int(rng.integers(2, 5))
    H = k * h
    counts = [int(c) for c in rng.integers(H, H + 40, size=P)]
    tail = [int(x) for x in (rng.integers(h + 1, 90, size=1) if d == 2 else rng.integers(3, 20, size=2))]
    shape = (sum(counts),) + tuple(tail) if d == 2 else (sum(counts), tail[0], int(rng.integers(5, 70)))
    T = int(rng.integers(1, 8))
    return d, h, kind, engine, k, shape, counts, T


@pytest.mark.parametrize("i", range(120))
def test_random_p2p_case_bitwise(i):
    d, h, kind, engine, k, shape, counts, T = _case(i)
    W = synth.preset("heat3d") if kind == "heat3d" else _weights(kind, d, h, 60 + i)
    g = synth.grid(tuple(n + 2 * h for n in shape), 70 + i)
    ref = _global(W, g, T, engine, fuse_k=k)
    out = _run_local(W, g, h, shape, T, engine, counts, fuse_k=k)
    assert np.array_equal(out, ref), (i, d, h, kind, engine, k, shape, counts, T, float(np.nanmax(np.abs(out - ref))))
