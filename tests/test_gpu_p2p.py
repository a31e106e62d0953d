"""Device-initiated halo exchange (lora_stencil_run_dist_p2p) on one GPU (-m gpu).

Several slab ranks share the B200: in one process they are wired with p2p_connect_local and run on
their own streams concurrently (the boundary tiles of one rank spin on the step counters the
neighbour's kernel publishes, exactly as across NVLink); across two processes they are wired with
CUDA IPC handles.  The gathered slabs must equal a single-GPU run of the global grid BITWISE (the
same kernels compute every point from the same neighbourhood; pin P10) and the oracle to 1e-12."""
import os

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
import synth
from tests._gpu_helpers import rel_err

pytestmark = pytest.mark.gpu


def _weights(kind, d, h, seed):
    if kind == "rsym":
        return synth.rsym_weights(d, h, seed)
    if kind == "star":
        return synth.star_weights(d, h, seed)
    if kind == "asym":
        return synth.asym_weights(d, h, seed)
    if kind == "heat3d":
        return synth.preset("heat3d")
    raise KeyError(kind)


def _split(n0, counts):
    starts = np.concatenate([[0], np.cumsum(counts)[:-1]]).astype(int)
    assert sum(counts) == n0
    return list(zip(starts.tolist(), counts))


def _run_local(W, g, h, shape, T, engine, counts, zero_copy=False, repeat=1, fuse_k=1):
    """P slab ranks in this process; returns the gathered global padded result (halo = input)."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    from paper_conf_sc_zhanglyczcy24_b200 import dist as D
    slabs = _split(shape[0], counts)
    P = len(slabs)
    sts, eps, xs, ys, streams = [], [], [], [], []
    for r, (s0, c) in enumerate(slabs):
        st = L.Stencil(W, (c,) + tuple(shape[1:]), engine=engine, fuse_k=fuse_k)
        sts.append(st)
        eps.append(L.lora_stencil_p2p_create(st.plan, P, r))
        xs.append(torch.from_numpy(np.ascontiguousarray(D.local_slice(g, s0, c, h))).cuda())
        ys.append(torch.full_like(xs[-1], float("nan")))
        streams.append(torch.cuda.Stream())
    for r in range(P):
        L.lora_stencil_p2p_connect_local(eps[r], eps[r - 1] if r > 0 else None, eps[r + 1] if r < P - 1 else None)
    torch.cuda.synchronize()
    nl = -(-T // max(1, sts[0].info()["fuse_k"])) if engine == "rdg_cuda" else T   # launches per run
    for _ in range(repeat):
        if zero_copy:
            # fill every rank's view 0 (the caller layout inside exchange buffer 0; with deep halos it
            # starts H - h rows in) BEFORE any run is enqueued: a device-wide synchronize between the
            # ranks' enqueues would wait on a kernel that spins for a neighbour whose run is not enqueued yet
            for r in range(P):
                torch.as_tensor(_DevBuf(L.lora_stencil_p2p_view(eps[r], 0), xs[r].shape), device="cuda").copy_(xs[r])
            torch.cuda.synchronize()
        for r in range(P):
            inp, outp = xs[r].data_ptr(), ys[r].data_ptr()
            if zero_copy:
                inp = L.lora_stencil_p2p_view(eps[r], 0)
                outp = L.lora_stencil_p2p_view(eps[r], nl % 2)
            L.lora_stencil_run_dist_p2p(sts[r].plan, eps[r], inp, outp, T, streams[r].cuda_stream)
        torch.cuda.synchronize()
    for r in range(P):
        L.lora_stencil_p2p_status(eps[r])
    out = g.copy()
    for r, (s0, c) in enumerate(slabs):
        if zero_copy:
            res = torch.as_tensor(_DevBuf(L.lora_stencil_p2p_view(eps[r], nl % 2), xs[r].shape), device="cuda")
            res = res.cpu().numpy()
        else:
            res = ys[r].cpu().numpy()
        out[h + s0:h + s0 + c] = res[h:h + c]
    for r in range(P):
        L.lora_stencil_p2p_destroy(eps[r])
        sts[r].close()
    return out


class _DevBuf:
    """__cuda_array_interface__ view of a library-owned device buffer (float64, C order)."""

    def __init__(self, ptr, shape):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": "<f8", "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def _global(W, g, T, engine, fuse_k=1):
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    h = (W.shape[0] - 1) // 2
    shape = tuple(s - 2 * h for s in g.shape)
    st = L.Stencil(W, shape, engine=engine, fuse_k=fuse_k)
    x = torch.from_numpy(g).cuda()
    y = torch.empty_like(x)
    st.run(x, y, T)
    torch.cuda.synchronize()
    st.close()
    return y.cpu().numpy()


CASES = [
    # d, h, kind, engine, global interior shape, slab row counts
    (2, 3, "rsym", "rdg_cuda", (300, 200), [150, 150]),
    (2, 3, "rsym", "rdg_cuda", (301, 130), [100, 3, 198]),        # a slab of exactly R rows
    (2, 1, "rsym", "rdg_cuda", (517, 300), [129, 130, 128, 130]),
    (2, 2, "star", "rdg_cuda", (260, 190), [130, 130]),
    (2, 2, "asym", "rdg_cuda", (200, 77), [67, 133]),
    (2, 3, "rsym", "direct", (257, 99), [128, 129]),
    (3, 1, "rsym", "rdg_cuda", (96, 20, 66), [48, 48]),
    (3, 1, "heat3d", "rdg_cuda", (130, 12, 40), [65, 1, 64]),
    (3, 2, "rsym", "rdg_cuda", (70, 9, 33), [35, 35]),
    (3, 1, "asym", "direct", (64, 10, 70), [30, 34]),
]


@pytest.mark.parametrize("case", CASES)
def test_p2p_local_ranks_bitwise(case):
    d, h, kind, engine, shape, counts = case
    W = _weights(kind, d, h, 21 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 31)
    for T in (1, 2, 5):
        ref = _global(W, g, T, engine)
        out = _run_local(W, g, h, shape, T, engine, counts)
        assert np.array_equal(out, ref), (T, float(np.nanmax(np.abs(out - ref))))
    if shape[0] * int(np.prod(shape[1:])) <= 40000:
        assert rel_err(out, oracle.run(W, g, 5)) <= 1e-12


FUSED = [
    # d, h, kind, global interior shape, slab row counts, fusion depth k (deep halos H = k h)
    (3, "rsym", (300, 200), [150, 150], 2),            # Box-2D49P row-pair form, the bench default
    (3, "rsym", (301, 130), [100, 6, 195], 2),          # a slab of exactly H rows
    (1, "rsym", (517, 300), [129, 130, 128, 130], 3),   # Box-2D9P default depth
    (1, "rsym", (260, 70), [70, 60, 130], 4),
    (2, "star", (260, 190), [130, 130], 3),
    (2, "rsym", (200, 77), [67, 133], 2),
    (3, "star", (256, 300), [128, 128], 2),
]


@pytest.mark.parametrize("case", FUSED)
def test_p2p_fused_deep_halo_bitwise(case):
    """k fused steps per launch across slab ranks: internal edges carry H = k h deep halos (the kernel
    recomputes the rows between h and H redundantly and stores only its own rows); T covers remainder
    launches (T mod k != 0) whose band geometry differs from the full launches."""
    h, kind, shape, counts, k = case
    W = _weights(kind, 2, h, 41 + h)
    g = synth.grid(tuple(n + 2 * h for n in shape), 43)
    for T in sorted({1, k, k + 1, 2 * k + 1, 7}):
        ref = _global(W, g, T, "rdg_cuda")
        out = _run_local(W, g, h, shape, T, "rdg_cuda", counts, fuse_k=k)
        assert np.array_equal(out, ref), (T, float(np.nanmax(np.abs(out - ref))))
    out = _run_local(W, g, h, shape, 5, "rdg_cuda", counts, fuse_k=k, repeat=2)
    assert np.array_equal(out, _global(W, g, 5, "rdg_cuda"))
    # zero-copy through the caller-layout views of the deep-halo buffers (lora_stencil_p2p_view)
    for T in (2 * k, 2 * k + 1):
        out = _run_local(W, g, h, shape, T, "rdg_cuda", counts, fuse_k=k, zero_copy=True, repeat=2)
        assert np.array_equal(out, _global(W, g, T, "rdg_cuda")), T


FUSED3D = [
    # kind, global interior shape (z, y, x), slab plane counts, fusion depth k (deep halos H = k)
    ("rsym", (96, 20, 66), [48, 48], 2),                 # Box-3D27P signature, the planner default k = 2
    ("heat3d", (130, 12, 40), [64, 2, 64], 2),           # Heat-3D signature; a slab of exactly H planes
    ("rsym", (64, 33, 130), [16, 16, 16, 16], 2),        # 4 ranks, several x bands / y blocks per slab
    ("asym", (60, 17, 70), [20, 21, 19], 3),             # general plane signature, k = 3
    ("rsym", (400, 30, 62), [200, 200], 2),              # several z chunks per column (interior chunks)
]


@pytest.mark.parametrize("case", FUSED3D)
def test_p2p_fused3d_deep_halo_bitwise(case):
    """3D: the fused radius-1 kernel (rdg3df, k steps per launch) with the in-kernel exchange: internal
    slab edges carry H = k deep halo planes, the boundary z-chunks wait on / publish the per-column
    step counters; T covers remainder launches (the unfused kernel, another column geometry).  Bitwise
    against the single-GPU run of the global grid at the same fusion depth and unfused."""
    kind, shape, counts, k = case
    W = _weights(kind, 3, 1, 47)
    g = synth.grid(tuple(n + 2 for n in shape), 53)
    for T in sorted({1, k, k + 1, 2 * k + 1, 6}):
        ref = _global(W, g, T, "rdg_cuda", fuse_k=k)
        out = _run_local(W, g, 1, shape, T, "rdg_cuda", counts, fuse_k=k)
        assert np.array_equal(out, ref), (T, float(np.nanmax(np.abs(out - ref))))
        assert np.array_equal(ref, _global(W, g, T, "rdg_cuda", fuse_k=1)), T
    out = _run_local(W, g, 1, shape, 5, "rdg_cuda", counts, fuse_k=k, repeat=2)
    assert np.array_equal(out, _global(W, g, 5, "rdg_cuda", fuse_k=k))
    if int(np.prod(shape)) <= 200000:
        assert rel_err(out, oracle.run(W, g, 5)) <= 1e-12


def test_p2p_repeated_runs_and_zero_copy():
    """Epochs: the same endpoints run three times (monotonic step counters, no reset); zero-copy
    mode reads buffer 0 and leaves the result in buffer T % 2."""
    W = synth.rsym_weights(2, 3, 8)
    shape, h = (256, 150), 3
    g = synth.grid(tuple(n + 2 * h for n in shape), 9)
    for T in (3, 4):
        ref = _global(W, g, T, "rdg_cuda")
        assert np.array_equal(_run_local(W, g, h, shape, T, "rdg_cuda", [128, 128], repeat=3), ref)
        assert np.array_equal(_run_local(W, g, h, shape, T, "rdg_cuda", [100, 156], zero_copy=True, repeat=2), ref)


def test_p2p_large_slabs_many_items():
    """Box-2D49P slabs large enough for a full persistent grid (many boundary items per step)."""
    W, c = synth.config("box2d49p-10240")
    shape, h = (2048, 4096), 3
    g = synth.grid(tuple(n + 2 * h for n in shape), 20240103)
    T = 3
    ref = _global(W, g, T, "rdg_cuda")
    out = _run_local(W, g, h, shape, T, "rdg_cuda", [512, 512, 512, 512])
    assert np.array_equal(out, ref)
    out = _run_local(W, g, h, shape, 5, "rdg_cuda", [512, 512, 512, 512], fuse_k=2)   # the bench default
    assert np.array_equal(out, _global(W, g, 5, "rdg_cuda"))


def test_p2p_unsupported_and_errors():
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W = synth.rsym_weights(2, 1, 2)
    st = L.Stencil(W, (64, 64), engine="tc")
    with pytest.raises(L.LoraError) as e:
        L.lora_stencil_p2p_create(st.plan, 2, 0)
    assert e.value.code == L.LORA_ERR_UNSUPPORTED
    st.close()
    st = L.Stencil(W, (64, 64), engine="rdg_cuda")
    ep = L.lora_stencil_p2p_create(st.plan, 2, 0)
    with pytest.raises(L.LoraError):   # not connected to its upper neighbour
        L.lora_stencil_run_dist_p2p(st.plan, ep, L.lora_stencil_p2p_buffer(ep, 0), L.lora_stencil_p2p_buffer(ep, 1), 1)
    with pytest.raises(L.LoraError):   # rank 0 has no lower neighbour: a handle there is an error
        L.lora_stencil_p2p_connect(ep, b"\0" * 128, b"\0" * 128)
    other = L.Stencil(W, (64, 66), engine="rdg_cuda")
    ep2 = L.lora_stencil_p2p_create(other.plan, 2, 1)
    with pytest.raises(L.LoraError):   # trailing extents differ
        L.lora_stencil_p2p_connect_local(ep, None, ep2)
    L.lora_stencil_p2p_destroy(ep)
    L.lora_stencil_p2p_destroy(ep2)
    st.close()
    other.close()


def _ipc_rank(rank, world, q_out, q_h, q_go):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import paper_conf_sc_zhanglyczcy24_b200 as L
        from paper_conf_sc_zhanglyczcy24_b200 import dist as D
        torch.cuda.set_device(0)
        W = synth.rsym_weights(2, 3, 5)
        shape, h, T = (200, 130), 3, 3
        g = synth.grid(tuple(n + 2 * h for n in shape), 6)
        start, cnt = D.slab_bounds(shape[0], world, rank)
        st = L.Stencil(W, (cnt, shape[1]), engine="rdg_cuda", fuse_k=1)
        ep = L.lora_stencil_p2p_create(st.plan, world, rank)
        q_h.put((rank, L.lora_stencil_p2p_get_handle(ep)))
        hs = dict(q_go[rank].get(timeout=120))
        L.lora_stencil_p2p_connect(ep, hs.get(rank - 1), hs.get(rank + 1))
        x = torch.from_numpy(np.ascontiguousarray(D.local_slice(g, start, cnt, h))).cuda()
        y = torch.empty_like(x)
        L.lora_stencil_run_dist_p2p(st.plan, ep, x.data_ptr(), y.data_ptr(), T, torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        L.lora_stencil_p2p_status(ep)
        q_out.put((rank, start, y[h:h + cnt].cpu().numpy()))
        q_go[rank].get(timeout=120)      # keep the mapping alive until every rank is done
        L.lora_stencil_p2p_destroy(ep)
    except Exception:
        import traceback
        q_out.put((rank, -1, traceback.format_exc()))


def test_p2p_two_processes_cuda_ipc():
    """Two processes on the one GPU, wired by CUDA IPC handles (the multi-GPU wiring path)."""
    import torch
    world = 2
    ctx = mp.get_context("spawn")
    q_out, q_h = ctx.Queue(), ctx.Queue()
    q_go = [ctx.Queue() for _ in range(world)]
    procs = [ctx.Process(target=_ipc_rank, args=(r, world, q_out, q_h, q_go)) for r in range(world)]
    for p in procs:
        p.start()
    hs = dict(q_h.get(timeout=180) for _ in range(world))
    for r in range(world):
        q_go[r].put(list(hs.items()))
    res = [q_out.get(timeout=300) for _ in range(world)]
    for r in range(world):
        q_go[r].put(None)
    for p in procs:
        p.join(timeout=60)
    for r, s, a in res:
        assert s >= 0, a
    W = synth.rsym_weights(2, 3, 5)
    g = synth.grid((206, 136), 6)
    ref = _global(W, g, 3, "rdg_cuda")
    for r, s, a in res:
        assert np.array_equal(a, ref[3 + s:3 + s + a.shape[0]])
