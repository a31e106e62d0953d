"""Host-side tests (no GPU): the C-ABI library loads and exports every symbol the header declares,
and the planner's factorisation satisfies what the paper fixes (eq. 8/9/15)
and DESIGN.md reading Q6 for the cases the paper leaves open."""
import json
import math
import os
import re

import numpy as np
import pytest

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_sc_zhanglyczcy24_b200 import _build
    _build.build()
    import paper_conf_sc_zhanglyczcy24_b200 as L
    return L


def test_library_exports_every_header_symbol(L):
    hdr = open(os.path.join(ROOT, "include", "lora_stencil.h")).read()
    declared = set(re.findall(r"\b(lora_stencil_\w+)\s*\(", hdr))
    assert len(declared) >= 14
    import ctypes
    lib = ctypes.CDLL(L.LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name
    assert set(L.EXPORTED) == declared
    assert "sm_100a" in L.lora_stencil_version()


def test_library_has_no_oracle_dependency():
    """The product library must not link or embed the oracle (task rule ③)."""
    import subprocess
    lib = os.path.join(ROOT, "paper_conf_sc_zhanglyczcy24_b200", "liblora_stencil.so")
    syms = subprocess.run(["nm", "-D", lib], capture_output=True, text=True).stdout
    assert "oracle" not in syms
    deps = subprocess.run(["ldd", lib], capture_output=True, text=True).stdout
    assert "oracle" not in deps


def _recon(terms, plane_shape_n, nplanes=1):
    n = plane_shape_n
    W = np.zeros((nplanes, n, n))
    for t in terms:
        W[t["plane"]] += np.outer(t["u"], t["v"])
    return W


@pytest.mark.parametrize("h", [1, 2, 3, 4])
def test_pma_rsym_plan_matches_paper_pyramid(L, h):
    """Radially symmetric W: h+1 terms, sizes 2h+3-2i (eq. 15), the last a scalar,
    reconstruction <= 1e-14, and the same factors as the oracle's step-by-step PMA."""
    W = synth.rsym_weights(2, h, 200 + h)
    st = L.Stencil(W, (100, 100), engine="rdg_cuda")
    terms = st.terms()
    assert [t["radius"] for t in terms] == list(range(h, 0, -1)) + [0]
    assert [t["kind"] for t in terms] == [0] * h + [2]
    R = _recon(terms, 2 * h + 1)[0]
    assert np.abs(R - W).max() <= 1e-14 * np.abs(W).max()
    ref = oracle.pma(W)
    for t, (u, v) in zip(terms, ref):
        m = len(u)
        o = h - (m - 1) // 2
        np.testing.assert_allclose(t["u"][o:o + m], u, rtol=0, atol=1e-15)
        np.testing.assert_allclose(t["v"][o:o + m], v, rtol=0, atol=1e-17)
    info = st.info()
    assert info["recon_err"] <= 1e-14 and info["n_tc_chain"] == h and info["n_cuda"] == 1


def test_star_gives_two_arms(L):
    for h in (1, 2, 3):
        W = synth.star_weights(2, h, 5)
        st = L.Stencil(W, (10, 10))
        terms = st.terms()
        assert [t["kind"] for t in terms] == [1, 1]
        assert np.abs(_recon(terms, 2 * h + 1)[0] - W).max() <= 1e-16


def test_separable_weights_give_one_term_no_nan(L):
    """A separable W (Box-2D9P composed, Gaussian) makes naive PMA divide 0/0 in ring 2;
    the rank-revealing stop must give a single term (Q6)."""
    v = np.array([1.0, 4.0, 6.0, 4.0, 1.0]); W = np.outer(v, v) / 256.0
    st = L.Stencil(W, (10, 10))
    terms = st.terms()
    assert len(terms) == 1 and all(np.isfinite(t["u"]).all() and np.isfinite(t["v"]).all() for t in terms)
    assert st.info()["recon_err"] <= 1e-15


def test_asymmetric_uses_elimination(L):
    for h in (1, 2, 3, 4):
        W = synth.asym_weights(2, h, 7)
        st = L.Stencil(W, (10, 10))
        terms = st.terms()
        assert len(terms) <= 2 * h + 1
        assert np.abs(_recon(terms, 2 * h + 1)[0] - W).max() <= 1e-14 * np.abs(W).max()


def test_zero_and_single_weight_planes(L):
    W = np.zeros((3, 3)); W[0, 2] = 0.5
    st = L.Stencil(W, (4, 4))
    t = st.terms()
    assert len(t) == 1 and t[0]["kind"] == 2
    W = np.zeros((3, 3, 3)); W[1] = synth.rsym_weights(2, 1, 3) * 0.5; W[0, 1, 1] = W[2, 1, 1] = 0.25
    st = L.Stencil(W, (4, 4, 4))
    info = st.info()
    assert info["n_planes_pointwise"] == 2 and info["z_symmetric"] == 1


def test_integer_pyramid_factors_are_exact(L):
    W = synth.integer_pyramid_weights()
    terms = L.Stencil(W, (8, 8)).terms()
    assert np.array_equal(terms[0]["u"], [1, 2, 3, 4, 3, 2, 1])
    assert np.array_equal(terms[1]["v"][1:6], [1, 1, 2, 1, 1])
    assert np.array_equal(terms[2]["v"][2:5], [2, 4, 2]) and terms[3]["v"][3] == 3.0
    assert np.array_equal(_recon(terms, 7)[0], W)


@pytest.mark.parametrize("name", ["heat3d", "box3d27p"])
def test_3d_plane_decomposition_alg2(L, name):
    """Alg. 2: every plane factored; sum over planes reconstructs W; Heat-3D has
    two single-weight planes (CUDA-core point-wise) and a star centre plane."""
    W = synth.preset("heat3d") if name == "heat3d" else synth.rsym_weights(3, 1, 9)
    st = L.Stencil(W, (8, 8, 8))
    R = _recon(st.terms(), 3, 3)
    assert np.abs(R - W).max() <= 1e-15
    info = st.info()
    assert info["z_symmetric"] == 1
    if name == "heat3d":
        assert info["n_planes_pointwise"] == 2 and info["n_tc_single"] == 2


def test_invalid_arguments(L):
    W = synth.rsym_weights(2, 1, 1)
    with pytest.raises(L.LoraError):
        L.lora_stencil_plan(W, 4, 1, [10, 10])
    with pytest.raises(L.LoraError):
        L.lora_stencil_plan(np.zeros((11, 11)), 2, 5, [10, 10])          # radius > 4
    with pytest.raises(L.LoraError):
        L.lora_stencil_plan(W, 2, 1, [0, 10])
    bad = W.copy(); bad[0, 0] = np.nan
    with pytest.raises(L.LoraError):
        L.lora_stencil_plan(bad, 2, 1, [10, 10])
    assert "finite" in L.lora_stencil_last_error()


def test_cost_model_reproduces_paper_counts(L):
    """Pin P11: the library's cost model (lora_stencil_plan_query, include/lora_stencil.h) reproduces
    the analytic counts the paper PRINTS (tests/golden/paper_counts.json): eq. 14 ConvStencil / RDG
    3.25x at h = 3 and 4.2x at h = 4 and the redundancy they eliminate (69.23 %,
    76.19 %); eq. 16 36 LoRAStencil MMAs vs ConvStencil's 26 for Box-2D49P; the fusion
    fragment waste 96/156.  The expected values are the paper's numbers, not re-derived here."""
    gold = json.load(open(os.path.join(ROOT, "tests", "golden", "paper_counts.json")))
    info = {h: L.Stencil(synth.rsym_weights(2, h, 3), (64, 64)).info() for h in (1, 2, 3, 4)}
    for h in (3, 4):
        assert info[h]["paper_convstencil_over_rdg"] == pytest.approx(gold["eq14_convstencil_over_rdg"][f"h{h}"], rel=1e-12)
        assert round(1 - 1 / info[h]["paper_convstencil_over_rdg"], 4) == gold["eq14_redundancy_eliminated"][f"h{h}"]
        assert info[h]["paper_convstencil_frag_per_point"] / info[h]["paper_rdg_frag_per_point"] == pytest.approx(
            info[h]["paper_convstencil_over_rdg"], rel=1e-12)    # eq. 13 / eq. 12 == eq. 14
    i3 = info[3]
    assert i3["paper_points_per_update"] == 64                  # 32 ceil(3/2) ceil(3/4): the 8x8 tile of P:207
    assert i3["paper_mma_per_point"] * 64 == pytest.approx(gold["eq16_mma_ratio_h3"]["lora"], abs=1e-9)
    assert i3["paper_convstencil_mma_per_point"] * 64 == pytest.approx(gold["eq16_mma_ratio_h3"]["convstencil"], abs=1e-9)
    w = gold["fusion_fragment_waste"]
    assert info[1]["paper_fragment_waste"] == w["total"]               # Box-2D9P: 156 of 256 elements wasted
    assert info[1]["paper_fragment_waste"] - info[3]["paper_fragment_waste"] == w["saved"]   # 3x fused: 96 saved
    assert (info[1]["paper_fragment_waste"] - info[3]["paper_fragment_waste"]) / info[1]["paper_fragment_waste"] == \
        pytest.approx(w["pct"], abs=1e-4)


def test_tc_engine_default_is_unfused(L):
    """engine='tc' without an explicit fuse_k runs the paper's chain unfused; the composed
    kernel is opt-in."""
    for name in ("box2d9p-10240", "heat2d-256", "box2d49p-10240"):
        W, c = synth.config(name)
        assert L.Stencil(W, c["shape"], engine="tc").info()["fuse_k"] == 1, name
    W, c = synth.config("box2d9p-10240")
    assert L.Stencil(W, c["shape"], engine="tc", fuse_k=2).info()["fuse_k"] == 2


def test_host_buffers_are_validated(L):
    """run_host(_async) refuses buffers the C side would over-read / over-write
    (checked before any CUDA call, so this runs without a GPU)."""
    W = synth.rsym_weights(2, 1, 3)
    st = L.Stencil(W, (10, 12))
    good = np.zeros((12, 14))
    for bad in (np.zeros((12, 14), np.float32), np.zeros((12, 13)), np.zeros((14, 12)).T):
        with pytest.raises(ValueError):
            L.lora_stencil_run_host(st.plan, bad, good, 1)
        with pytest.raises(ValueError):
            L.lora_stencil_run_host_async(st.plan, good, bad, 1, 1)
    with pytest.raises(ValueError):
        st.run_host(np.zeros(12 * 14), np.zeros(12 * 14), 1)
    with pytest.raises(ValueError):
        L.lora_stencil_plan_terms(st.plan, 2)      # radius must match the plan's
    assert len(L.lora_stencil_plan_terms(st.plan)) == len(st.terms())


def test_default_engine_and_fusion_choices(L):
    """The planner's defaults follow the measured B200 costs: CUDA-core RDG,
    fused only where the pass is HBM-bound."""
    expect = {"heat2d-256": 3, "box2d9p-10240": 3, "box2d49p-10240": 2, "star2d13p-10240": 2,
              "heat3d-512": 2, "box3d27p-512": 2, "heat1d-10240000": 8, "1d5p-10240000": 8}
    for name, k in expect.items():
        W, c = synth.config(name)
        info = L.Stencil(W, c["shape"]).info()
        assert info["engine_name"] == "rdg_cuda" and info["fuse_k"] == k, (name, info["fuse_k"])
        assert info["halo_depth"] == k * c["radius"]


def test_cuda_core_rank1_forms(L, monkeypatch):
    """CUDA-core engine: doubly reflection-symmetric W at radius >= 3 is evaluated as the row-pair
    split with unit centre taps (R + R(R+1) + 2R + 1 FP64 ops per point: 22 for Box-2D49P, against
    the PMA pyramid's R + 1 + sum_H (H + 2H + 1) = 25), PMA with LORA_RDG_PMA=1 or when a centre-
    column weight is zero; an asymmetric W or radius <= 2 keeps the planner's factors."""
    W = synth.rsym_weights(2, 3, 4)
    assert L.Stencil(W, (64, 64), engine="rdg_cuda").info()["fma_per_point_issued"] == 22
    assert L.Stencil(synth.rsym_weights(2, 4, 4), (64, 64), engine="rdg_cuda").info()["fma_per_point_issued"] == 33
    Wz = W.copy(); Wz[0, 3] = Wz[6, 3] = 0.0   # a zero centre-column weight: no unit centre tap for row pair 3
    assert L.Stencil(Wz, (64, 64), engine="rdg_cuda").info()["fma_per_point_issued"] != 22
    assert L.Stencil(synth.rsym_weights(2, 1, 4), (64, 64), engine="rdg_cuda").info()["fma_per_point_issued"] == 6
    monkeypatch.setenv("LORA_RDG_PMA", "1")
    assert L.Stencil(W, (64, 64), engine="rdg_cuda").info()["fma_per_point_issued"] == 25


def test_3d_joint_symmetric_planes(L, monkeypatch):
    """3D CUDA-core engine (reading Q18): a radius-1 W whose planes 0 and 1 are
    [a b a; b c b; a b a] with plane 2 = plane 0 (Box-3D27P) is evaluated on the shared class sums
    (12.5 FP64 ops per point in the planner's count, against 15 for the two PMA planes); a plane
    without the transposition symmetry, or LORA_NO_SYM3=1, keeps the PMA planes."""
    W = synth.rsym_weights(3, 1, 7)
    assert L.Stencil(W, (16, 16, 16), engine="rdg_cuda").info()["fma_per_point_issued"] == 12.5
    Wa = W.copy()
    Wa[1, 0, 1] = Wa[1, 2, 1] = W[1, 0, 1] * 1.5   # plane 1: b_vertical != b_horizontal (still PMA)
    assert L.Stencil(Wa, (16, 16, 16), engine="rdg_cuda").info()["fma_per_point_issued"] == 15
    monkeypatch.setenv("LORA_NO_SYM3", "1")
    assert L.Stencil(W, (16, 16, 16), engine="rdg_cuda").info()["fma_per_point_issued"] == 15


def test_plan_query_fields(L):
    W = synth.rsym_weights(2, 3, 4)
    info = L.Stencil(W, (100, 200), engine="tc").info()
    assert info["ndim"] == 2 and info["radius"] == 3 and info["grid"][:2] == [100, 200]
    assert info["n_terms"] == 4 and info["n_tc_chain"] == 3 and info["n_cuda"] == 1
    assert info["fma_per_point_direct"] == 49 and info["fma_per_point_separable"] == 31
    assert 80 <= info["fma_per_point_issued"] <= 100 and info["tile_m"] == 64
    with pytest.raises(L.LoraError):
        L.Stencil(W, (100, 200), engine="rdg_cuda", fuse_k=3)   # exceeds the radius-3 maximum
    with pytest.raises(L.LoraError):
        L.Stencil(synth.preset("heat1d"), (100,), engine="tc")   # no tensor-core 1D engine


def test_single_launch_path_selection(L, monkeypatch):
    """Small 2D star grids (Heat-2D 256^2, BASELINE configs[0]) take the single-launch cluster path;
    large or non-star plans and LORA_NO_SMALL=1 do not (host-only planning, no GPU needed)."""
    W, c = synth.config("heat2d-256")
    assert L.Stencil(W, c["shape"]).info()["single_launch"] == 1
    assert L.Stencil(W, c["shape"], engine="tc").info()["single_launch"] == 0
    assert L.Stencil(W, (257, 256)).info()["single_launch"] == 0          # 257 rows: no cluster divides it
    assert L.Stencil(W, (4096, 4096)).info()["single_launch"] == 0        # does not fit shared memory
    W2, c2 = synth.config("box2d49p-10240")
    assert L.Stencil(W2, (256, 256)).info()["single_launch"] == 0         # not a star
    monkeypatch.setenv("LORA_NO_SMALL", "1")
    assert L.Stencil(W, c["shape"]).info()["single_launch"] == 0


def test_plan_failure_status_codes(L):
    """lora_stencil_last_status reports why a plan call returned NULL (the binding raises it)."""
    W = synth.rsym_weights(2, 1, 1)
    with pytest.raises(L.LoraError) as e:
        L.lora_stencil_plan(W, 2, 1, [0, 10])
    assert e.value.code == L.LORA_ERR_INVALID_ARG
    with pytest.raises(L.LoraError) as e:
        L.lora_stencil_plan(np.zeros((11, 11)), 2, 5, [10, 10])
    assert e.value.code == L.LORA_ERR_UNSUPPORTED
    with pytest.raises(L.LoraError) as e:
        L.Stencil(synth.preset("heat1d"), (100,), engine="tc")
    assert e.value.code == L.LORA_ERR_UNSUPPORTED
    L.lora_stencil_plan(W, 2, 1, [10, 10])
    assert L._lib.lora_stencil_last_status() == L.LORA_OK
