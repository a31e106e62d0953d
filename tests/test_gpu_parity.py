"""CUDA path vs the CPU oracle, element by element on the same seeded inputs (-m gpu).

Tolerance: the north star's 1e-10 max relative error is the bar; these small cases use
1e-12 (the error budget in DESIGN.md gives ~1e-14 per step for convex weights)."""
import numpy as np
import pytest

import oracle
import synth
from tests._gpu_helpers import rel_err, run_gpu

pytestmark = pytest.mark.gpu

ENGINES_2D = ["direct", "tc", "rdg_cuda"]


def _weights(kind, d, h, seed):
    if kind == "rsym":
        return synth.rsym_weights(d, h, seed)
    if kind == "star":
        return synth.star_weights(d, h, seed)
    if kind == "asym":
        return synth.asym_weights(d, h, seed)
    if kind == "separable":
        v = synth.rsym_weights(1, h, seed) if False else np.linspace(1, 2, 2 * h + 1)
        v = v + v[::-1]
        W = np.multiply.outer(v, v)
        return W / W.sum()
    raise KeyError(kind)


@pytest.mark.parametrize("engine", ENGINES_2D)
@pytest.mark.parametrize("h", [1, 2, 3, 4])
@pytest.mark.parametrize("kind", ["rsym", "star", "asym", "separable"])
@pytest.mark.parametrize("shape", [(1, 1), (3, 5), (67, 129), (130, 70)])
def test_2d_parity_small(engine, h, kind, shape):
    W = _weights(kind, 2, h, 7 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 20240101 + h)
    for T in (1, 2, 3):
        out, info = run_gpu(W, g, T, engine=engine)
        ref = oracle.run(W, g, T)
        assert info["engine_name"] == engine
        assert rel_err(out, ref) <= 1e-12, (T, rel_err(out, ref))
        # halo: bitwise copy of the input halo
        mask = np.ones_like(g, dtype=bool)
        mask[h:-h, h:-h] = False
        assert np.array_equal(out[mask], g[mask])


@pytest.mark.parametrize("engine", ENGINES_2D + ["auto"])
def test_T0_is_bitwise_copy(engine):
    W = synth.rsym_weights(2, 3, 1)
    g = synth.grid((40, 37), 3)
    out, _ = run_gpu(W, g, 0, engine=engine)
    assert np.array_equal(out, g)


@pytest.mark.parametrize("engine", ENGINES_2D)
def test_integer_exact_bitwise(engine):
    """P9: integer pyramid weights (PMA recovers integer factors exactly), inputs in {0..3},
    every intermediate < 2^53 for T <= 6 => the GPU result equals the oracle bitwise."""
    W = synth.integer_pyramid_weights()
    g = synth.integer_grid((256 + 6, 256 + 6), 99)
    out, _ = run_gpu(W, g, 6, engine=engine)
    ref = oracle.run(W, g, 6)
    assert np.array_equal(out, ref)


@pytest.mark.parametrize("engine,fuse_k", [("rdg_cuda", 0), ("rdg_cuda", 1), ("direct", 0), ("tc", 0)])
def test_integer_exact_bitwise_3d(engine, fuse_k):
    """P9 in 3D (SURVEY §8(c) parity matrix: 64³): an integer 27-point box whose planes are rank-1 +
    centre (PMA recovers them with dyadic unit-centre factors), inputs in {0..3}, T one below the
    2^53 bound => every intermediate is exact and the GPU result equals the oracle bitwise, for the
    fused (default k = 2) and unfused CUDA-core kernels, the direct kernel and the tensor-core chain."""
    import math
    W = np.array([[[1, 2, 1], [2, 4, 2], [1, 2, 1]], [[2, 4, 2], [4, 9, 4], [2, 4, 2]],
                  [[1, 2, 1], [2, 4, 2], [1, 2, 1]]], dtype=np.float64)
    T = int((53 - math.log2(3)) // math.log2(np.abs(W).sum())) - 1
    g = synth.integer_grid((66, 66, 66), 98)
    out, _ = run_gpu(W, g, T, engine=engine, fuse_k=fuse_k)
    assert np.array_equal(out, oracle.run(W, g, T)), T


ENGINES_3D = ["direct", "rdg_cuda", "tc"]


@pytest.mark.parametrize("engine", ENGINES_3D)
@pytest.mark.parametrize("h", [1, 2])
@pytest.mark.parametrize("kind", ["rsym", "star", "asym", "heat3d"])
@pytest.mark.parametrize("shape", [(1, 1, 1), (3, 4, 5), (17, 9, 33), (70, 12, 40), (130, 6, 66)])
def test_3d_parity_small(engine, h, kind, shape):
    if kind == "heat3d":
        if h != 1:
            pytest.skip("preset is radius 1")
        W = synth.preset("heat3d")
    else:
        W = _weights(kind, 3, h, 3 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 5)
    if engine == "tc" and h != 1:
        pytest.skip("tensor-core 3D engine is radius 1 (register budget of the z-ring)")
    for T in (1, 2, 3):
        out, info = run_gpu(W, g, T, engine=engine)
        ref = oracle.run(W, g, T)
        assert info["engine_name"] == engine
        assert rel_err(out, ref) <= 1e-12, (T, rel_err(out, ref))


@pytest.mark.parametrize("engine", ENGINES_3D)
def test_3d_staging_paths_agree(engine, monkeypatch):
    W = synth.rsym_weights(3, 1, 8)
    g = synth.grid((34, 20, 66), 12)
    a, _ = run_gpu(W, g, 3, engine=engine)
    monkeypatch.setenv("LORA_NO_TMA", "1")
    b, _ = run_gpu(W, g, 3, engine=engine)
    assert np.array_equal(a, b)
    assert rel_err(a, oracle.run(W, g, 3)) <= 1e-12


@pytest.mark.parametrize("engine", ENGINES_2D)
def test_constant_field_invariance(engine):
    W = synth.rsym_weights(2, 3, 17)
    g = synth.constant_grid((200, 150), 0.75)
    out, _ = run_gpu(W, g, 20, engine=engine)
    assert rel_err(out, g) <= 1e-14


def test_errors_alias_and_args():
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W = synth.rsym_weights(2, 1, 1)
    st = L.Stencil(W, (10, 10))
    x = torch.zeros(12, 12, dtype=torch.float64, device="cuda")
    with pytest.raises(L.LoraError) as e:
        L.lora_stencil_run(st.plan, x.data_ptr(), x.data_ptr() + 8, 1, 0)
    assert e.value.code == L.LORA_ERR_ALIAS
    with pytest.raises(L.LoraError) as e:
        L.lora_stencil_run(st.plan, x.data_ptr(), 0, 1, 0)
    assert e.value.code == L.LORA_ERR_INVALID_ARG


@pytest.mark.parametrize("engine", ENGINES_2D)
@pytest.mark.parametrize("shape", [(64, 64), (200, 130), (129, 66)])
def test_2d_staging_paths_agree(engine, shape, monkeypatch):
    """TMA staging (even padded width) and the LDGSTS fallback (LORA_NO_TMA=1) give the same
    per-point arithmetic => bitwise equal results; both match the oracle."""
    h = 3
    W = synth.rsym_weights(2, h, 5)
    g = synth.grid(tuple(n + 2 * h for n in shape), 11)
    a, _ = run_gpu(W, g, 3, engine=engine)
    monkeypatch.setenv("LORA_NO_TMA", "1")
    b, _ = run_gpu(W, g, 3, engine=engine)
    assert np.array_equal(a, b)
    assert rel_err(a, oracle.run(W, g, 3)) <= 1e-12


FUSE_MAX = {1: 4, 2: 3, 3: 2, 4: 2}


@pytest.mark.parametrize("h", [1, 2, 3, 4])
@pytest.mark.parametrize("kind", ["rsym", "star"])
@pytest.mark.parametrize("shape", [(1, 1), (3, 5), (67, 129), (300, 200), (130, 70)])
def test_2d_temporal_fusion_exact(h, kind, shape):
    """Exact temporal blocking (Q5): k fused sub-steps with the halo re-imposed every
    sub-step equal k single steps BITWISE (same per-point arithmetic) and the oracle to 1e-12,
    for T = 1, k-1, k, k+1, 2k+1 (remainder launches) and ragged / tiny grids."""
    W = _weights(kind, 2, h, 40 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 77 + h)
    for k in range(2, FUSE_MAX[h] + 1):
        for T in sorted({1, k - 1, k, k + 1, 2 * k + 1}):
            a, info = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=k)
            assert info["fuse_k"] == k
            b, _ = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=1)
            assert np.array_equal(a, b), (k, T, float(np.max(np.abs(a - b))))
            assert rel_err(a, oracle.run(W, g, T)) <= 1e-12


@pytest.mark.parametrize("h", [3, 4])
@pytest.mark.parametrize("shape", [(3, 5), (67, 129), (300, 200)])
def test_rows_and_pma_forms(h, shape, monkeypatch):
    """The CUDA-core engine's two rank-1 splits of a doubly reflection-symmetric W (row pairs,
    Plan::rdg_rows, the default at radius >= 3; PMA with LORA_RDG_PMA=1) both match the oracle,
    unfused and fused, and the fused form equals the unfused one bitwise."""
    W = synth.rsym_weights(2, h, 60 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 91 + h)
    for pma in ("0", "1"):
        monkeypatch.setenv("LORA_RDG_PMA", pma)
        for T in (1, 2, 5):
            a, info = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=1)
            n = h + 1
            # row pairs with unit centre taps: h pair sums + h DFMA per row term + 2h DFMA + 1 DMUL
            want = (h + n * h + 2 * h + 1) if pma == "0" else (h + 1 + sum((h - k) + (2 * (h - k) + 1) for k in range(h)))
            assert info["fma_per_point_issued"] == want
            assert rel_err(a, oracle.run(W, g, T)) <= 1e-12
            b, _ = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=2)
            assert np.array_equal(a, b)


def test_fusion_staging_paths_agree(monkeypatch):
    W = synth.rsym_weights(2, 3, 5)
    g = synth.grid((206, 136), 11)
    a, _ = run_gpu(W, g, 5, engine="rdg_cuda", fuse_k=2)
    monkeypatch.setenv("LORA_NO_TMA", "1")
    b, _ = run_gpu(W, g, 5, engine="rdg_cuda", fuse_k=2)
    assert np.array_equal(a, b)


def test_graph_replay_matches_eager(monkeypatch):
    """Small grids replay the time loop as a CUDA graph from the second identical call on; the
    replays must equal the eager run bitwise, and a changed input must be honoured."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W = synth.preset("heat2d")
    g = synth.grid((258, 258), 9)
    st = L.Stencil(W, (256, 256))
    x = torch.from_numpy(g).cuda()
    side = torch.cuda.Stream()
    torch.cuda.set_stream(side)  # capture needs a non-default stream
    outs = []
    for _ in range(4):
        y = torch.zeros_like(x)
        st.run(x, y, 10)
        torch.cuda.synchronize()
        outs.append(y.cpu().numpy())
    # distinct y buffers => new key each time; reuse one buffer to exercise capture + replay
    y = torch.zeros_like(x)
    for _ in range(4):
        st.run(x, y, 10)
        torch.cuda.synchronize()
        outs.append(y.cpu().numpy())
    x.mul_(0.5)
    st.run(x, y, 10)
    torch.cuda.synchronize()
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])
    assert rel_err(outs[0], oracle.run(W, g, 10)) <= 1e-12
    assert rel_err(y.cpu().numpy(), oracle.run(W, 0.5 * g, 10)) <= 1e-12
    torch.cuda.set_stream(torch.cuda.default_stream())


@pytest.mark.parametrize("kind", ["rsym", "heat3d", "asym", "star"])
@pytest.mark.parametrize("shape", [(1, 1, 1), (3, 4, 5), (17, 9, 33), (40, 30, 130), (70, 15, 61)])
def test_3d_temporal_fusion_exact(kind, shape):
    """Two fused 3D steps (kernels_rdg3df.cu, halo re-imposed on the step-1 plane) equal two single
    steps bitwise and the oracle to 1e-12; odd T exercises the remainder launch."""
    W = synth.preset("heat3d") if kind == "heat3d" else _weights(kind, 3, 1, 21)
    g = synth.grid(tuple(n + 2 for n in shape), 31)
    for k in (2, 3):
        for T in (1, 2, 3, 5, 7):
            a, info = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=k)
            assert info["fuse_k"] == k
            b, _ = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=1)
            assert np.array_equal(a, b), (k, T, float(np.max(np.abs(a - b))))
            assert rel_err(a, oracle.run(W, g, T)) <= 1e-12


def test_3d_fusion_staging_paths_agree(monkeypatch):
    W = synth.rsym_weights(3, 1, 8)
    g = synth.grid((34, 20, 66), 12)
    for k in (2, 3):
        monkeypatch.delenv("LORA_NO_TMA", raising=False)
        a, _ = run_gpu(W, g, 4, engine="rdg_cuda", fuse_k=k)
        monkeypatch.setenv("LORA_NO_TMA", "1")
        b, _ = run_gpu(W, g, 4, engine="rdg_cuda", fuse_k=k)
        assert np.array_equal(a, b)


@pytest.mark.parametrize("h", [1, 2, 3, 4])
@pytest.mark.parametrize("n", [1, 7, 1000, 4097, 100001])
def test_1d_parity_and_fusion(h, n):
    """1D (Table II Heat-1D / 1D5P): one banded pass; k fused steps per launch (halo
    re-imposed) equal k single steps bitwise and the oracle to 1e-12."""
    W = synth.rsym_weights(1, h, 50 + h)
    g = synth.grid((n + 2 * h,), 60 + h)
    for T in (1, 3, 8, 11):
        a, info = run_gpu(W, g, T)               # planner default (fused)
        b, _ = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=1)
        c, _ = run_gpu(W, g, T, engine="direct")
        assert info["engine_name"] == "rdg_cuda" and info["fuse_k"] > 1
        assert np.array_equal(a, b) and np.array_equal(b, c), T
        assert rel_err(a, oracle.run(W, g, T)) <= 1e-12


def test_star2d13p_arms():
    W, c = synth.config("star2d13p-10240")
    g = synth.grid((300 + 6, 257 + 6), 1)
    for eng in ("auto", "tc", "direct"):
        out, info = run_gpu(W, g, 4, engine=eng)
        assert rel_err(out, oracle.run(W, g, 4)) <= 1e-12


@pytest.mark.parametrize("h", [1, 2, 3])
def test_tc_without_bvs_ablation_parity(h, monkeypatch):
    """The Fig. 9 ablation variant (stage-2 A fragments gathered with shuffles, no BVS) computes
    the same chains: matches the oracle and the BVS kernel to rounding."""
    W = synth.rsym_weights(2, h, 90 + h)
    g = synth.grid((130 + 2 * h, 70 + 2 * h), 91)
    a, _ = run_gpu(W, g, 3, engine="tc")
    monkeypatch.setenv("LORA_TC_NO_BVS", "1")
    b, _ = run_gpu(W, g, 3, engine="tc")
    ref = oracle.run(W, g, 3)
    assert rel_err(b, ref) <= 1e-12 and rel_err(a, b) <= 1e-13


@pytest.mark.parametrize("name", ["box2d49p", "box3d27p", "heat1d"])
def test_run_host_matches_device_run(name):
    """lora_stencil_run_host (host buffers, the e2e path) == lora_stencil_run on device buffers."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    if name == "box2d49p":
        W, shape = synth.rsym_weights(2, 3, 1), (300, 257)
    elif name == "box3d27p":
        W, shape = synth.rsym_weights(3, 1, 1), (40, 33, 66)
    else:
        W, shape = synth.preset("heat1d"), (100003,)
    h = (W.shape[0] - 1) // 2
    g = synth.grid(tuple(n + 2 * h for n in shape), 5)
    dev, _ = run_gpu(W, g, 9)
    st = L.Stencil(W, shape)
    hin = torch.from_numpy(g).pin_memory()
    hout = torch.empty_like(hin).pin_memory()
    st.run_host(hin, hout, 9)
    assert np.array_equal(hout.numpy(), dev)
    out2 = np.empty_like(g)            # pageable numpy buffers work too
    st.run_host(g, out2, 9)
    assert np.array_equal(out2, dev)
    # async form: two plans on two streams in flight at once (the bench e2e pipeline)
    st2 = L.Stencil(W, shape)
    g2 = synth.grid(g.shape, 6)
    dev2, _ = run_gpu(W, g2, 9)
    hin2 = torch.from_numpy(g2).pin_memory()
    outs = [torch.zeros_like(hin).pin_memory(), torch.zeros_like(hin).pin_memory()]
    ss = [torch.cuda.Stream(), torch.cuda.Stream()]
    for _ in range(2):
        L.lora_stencil_run_host_async(st.plan, hin, outs[0], 9, ss[0].cuda_stream)
        L.lora_stencil_run_host_async(st2.plan, hin2, outs[1], 9, ss[1].cuda_stream)
    for s in ss:
        s.synchronize()
    assert np.array_equal(outs[0].numpy(), dev) and np.array_equal(outs[1].numpy(), dev2)
    with pytest.raises(L.LoraError):
        L.lora_stencil_run_host_async(st.plan, hin, outs[0], 9, 0)   # the legacy stream is refused
    st.close()
    st2.close()


@pytest.mark.parametrize("h,k", [(1, 2), (1, 3), (1, 4), (2, 2)])
@pytest.mark.parametrize("kind", ["rsym", "star", "asym"])
@pytest.mark.parametrize("shape", [(1, 1), (3, 5), (7, 13), (67, 129), (130, 70)])
def test_tc_composed_fusion(h, k, kind, shape):
    """The paper's kernel fusion (§IV-A) on the tensor-core engine, made exact: the
    composed (2kh+1)^2 kernel on points farther than (k-1)h from the Dirichlet halo, the band next
    to it recomputed stepwise (Q5).  Matches the oracle for T = 1, k, k+1, 2k+1."""
    W = _weights(kind, 2, h, 70 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 71)
    for T in sorted({1, 2, k, k + 1, 2 * k - 1, 2 * k + 1}):
        out, info = run_gpu(W, g, T, engine="tc", fuse_k=k)
        assert info["fuse_k"] == k
        assert rel_err(out, oracle.run(W, g, T)) <= 1e-12, (T, rel_err(out, oracle.run(W, g, T)))


@pytest.mark.parametrize("engine", ["auto", "tc", "rdg_cuda", "direct"])
@pytest.mark.parametrize("d", [2, 3])
def test_identity_shift_zero_weights(engine, d):
    """P7 on the GPU: W = delta copies bitwise for any T; a single off-centre weight 1 shifts exactly
    (bitwise, halo inflow included); W = 0 gives a zero interior and the untouched halo."""
    if engine == "tc" and d == 3:
        pytest.skip("TC 3D needs a multi-point plane")
    h = 1
    shape = (20, 17) if d == 2 else (9, 8, 7)
    g = synth.grid(tuple(n + 2 * h for n in shape), 8)
    I = np.zeros((3,) * d); I[(1,) * d] = 1.0
    out, _ = run_gpu(I, g, 5, engine=engine)
    assert np.array_equal(out, g)
    S = np.zeros((3,) * d); S[(2,) + (0,) * (d - 1)] = 1.0      # in[x + (1, -1, ...)]
    out, _ = run_gpu(S, g, 3, engine=engine)
    assert np.array_equal(out, oracle.run(S, g, 3))
    Z = np.zeros((3,) * d)
    try:
        out, _ = run_gpu(Z, g, 2, engine=engine)
    except Exception as e:   # the tensor-core engine has no terms to run for W = 0
        assert engine == "tc", e
        return
    ref = g.copy()
    ref[tuple(slice(1, -1) for _ in range(d))] = 0.0
    assert np.array_equal(out, ref)


def _zero_centre_tap_2d(h):
    """Reflection-symmetric 2D W whose PMA chain factor v has a zero centre tap (the centre column
    of W vanishes outside the centre): the unit-centre rescaling of the CUDA-core engine cannot apply
    (kernels_rdg.cu signature() falls back to the general rank-1 form)."""
    n = 2 * h + 1
    W = np.zeros((n, n))
    for a in range(n):
        for b in range(n):
            if b != h and a != h:
                W[a, b] = 1.0 + 0.25 * (abs(a - h) + 2 * abs(b - h))
    W[h, h] = 2.0
    return W / W.sum()


@pytest.mark.parametrize("h", [1, 2])
def test_zero_centre_tap_fallback_2d(h):
    """PMA factors with v[R] == 0 (no unit-centre rescaling possible) still match the oracle, on
    every engine and at the planner's default fusion depth."""
    W = _zero_centre_tap_2d(h)
    g = synth.grid((67 + 2 * h, 129 + 2 * h), 5)
    ref = oracle.run(W, g, 4)
    for eng in ("auto", "rdg_cuda", "tc", "direct"):
        out, _ = run_gpu(W, g, 4, engine=eng)
        assert rel_err(out, ref) <= 1e-12, eng


def test_zero_centre_tap_fallback_3d():
    """Radius-1 3D W whose planes have zero edge taps (PMA v[1] == 0): pma1_unit_centre declines and
    both 3D CUDA-core kernels take the general chain mode; fused == unfused bitwise, both match the
    oracle."""
    W = np.zeros((3, 3, 3))
    for z in range(3):
        for y in range(3):
            for x in range(3):
                if (y == 1) == (x == 1):   # corners and centre of each plane
                    W[z, y, x] = 1.0 + 0.5 * abs(z - 1) + 0.25 * (y != 1)
    W /= W.sum()
    g = synth.grid((17 + 2, 9 + 2, 33 + 2), 8)
    ref = oracle.run(W, g, 3)
    a, _ = run_gpu(W, g, 3, engine="rdg_cuda", fuse_k=1)
    b, info = run_gpu(W, g, 3, engine="rdg_cuda", fuse_k=2)
    assert info["fuse_k"] == 2
    assert np.array_equal(a, b)
    assert rel_err(a, ref) <= 1e-12


@pytest.mark.parametrize("kind,h", [("heat2d", 1), ("star", 1), ("star", 2), ("star", 3), ("star", 4)])
@pytest.mark.parametrize("shape", [(256, 256), (64, 100), (48, 33), (32, 258)])
def test_small_cluster_path_bitwise(kind, h, shape, monkeypatch):
    """Small 2D star grids run all T steps in one launch (kernels_small.cu): the 2D-tile variant
    (default for T R <= 16), the cooperative-grid variant and the thread-block-cluster (DSMEM)
    variant are each bitwise equal to the streaming engine's per-step launches (LORA_NO_SMALL=1)
    and within 1e-12 of the oracle, for T on both sides of the fusion depth."""
    W = synth.preset("heat2d") if kind == "heat2d" else synth.star_weights(2, h, 11 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 20240101 + h)
    for T in (1, 2, 5, 10, 17):
        out, info = run_gpu(W, g, T)                      # default: tiles (T R <= 16), else the grid variant
        assert info["single_launch"] == 1, info
        monkeypatch.setenv("LORA_SMALL_MODE", "grid")     # the cooperative-grid variant
        out_gr, _ = run_gpu(W, g, T)
        monkeypatch.setenv("LORA_SMALL_MODE", "cluster")  # the thread-block-cluster (DSMEM) variant
        out_cl, _ = run_gpu(W, g, T)
        monkeypatch.delenv("LORA_SMALL_MODE")
        monkeypatch.setenv("LORA_NO_SMALL", "1")
        ref_stream, info2 = run_gpu(W, g, T)
        monkeypatch.delenv("LORA_NO_SMALL")
        assert info2["single_launch"] == 0
        assert np.array_equal(out, ref_stream), (T, float(np.max(np.abs(out - ref_stream))))
        assert np.array_equal(out_cl, ref_stream), (T, float(np.max(np.abs(out_cl - ref_stream))))
        assert np.array_equal(out_gr, ref_stream), (T, float(np.max(np.abs(out_gr - ref_stream))))
        assert rel_err(out, oracle.run(W, g, T)) <= 1e-12


@pytest.mark.parametrize("kind", ["rsym", "heat3d"])
@pytest.mark.parametrize("shape", [(40, 37, 70), (9, 130, 66)])
def test_3d_symmetric_plane_forms(kind, shape, monkeypatch):
    """3D CUDA-core engine, reading Q18: the joint evaluation of the symmetric planes
    (Box-3D27P, PM_SYM3) and the FMA-accumulated Heat-3D form agree with the oracle to 1e-12 and with
    the PMA / per-plane form (LORA_NO_SYM3=1) to rounding; fused (k = 2) and unfused runs of the
    same form are bitwise equal."""
    W = synth.rsym_weights(3, 1, 31) if kind == "rsym" else synth.preset("heat3d")
    g = synth.grid(tuple(n + 2 for n in shape), 20240131)
    T = 5
    ref = oracle.run(W, g, T)
    fused, info = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=2)
    unfused, _ = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=1)
    assert info["fuse_k"] == 2
    assert np.array_equal(fused, unfused)
    assert rel_err(fused, ref) <= 1e-12
    monkeypatch.setenv("LORA_NO_SYM3", "1")
    pma, info_p = run_gpu(W, g, T, engine="rdg_cuda", fuse_k=2)
    monkeypatch.delenv("LORA_NO_SYM3")
    assert rel_err(pma, ref) <= 1e-12
    if kind == "rsym":
        assert info["fma_per_point_issued"] == 12.5 and info_p["fma_per_point_issued"] == 15


def test_p2p_view_pointers():
    """lora_stencil_p2p_view: the caller-layout view of an exchange buffer (R-deep halos, same row pitch)
    starts hl - R rows into the buffer; out-of-range indices give NULL."""
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W = synth.rsym_weights(2, 3, 4)
    st = L.Stencil(W, (64, 100), engine="rdg_cuda", fuse_k=2)
    for nranks, rank in ((1, 0), (2, 0), (2, 1), (3, 1)):
        ep = L.lora_stencil_p2p_create(st.plan, nranks, rank)
        row = (100 + 6) * 8
        hl = 6 if rank > 0 else 3                      # H = k R = 6 deep towards a lower neighbour
        for i in (0, 1):
            assert L.lora_stencil_p2p_view(ep, i) - L.lora_stencil_p2p_buffer(ep, i) == (hl - 3) * row
        assert L.lora_stencil_p2p_view(ep, 2) == 0 and L.lora_stencil_p2p_view(ep, -1) == 0
        L.lora_stencil_p2p_destroy(ep)
    st.close()
