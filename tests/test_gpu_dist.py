"""lora_stencil_run_dist on GPUs (-m gpu).  One rank: must equal lora_stencil_run bitwise.
Two ranks over NCCL (needs >= 2 GPUs; skipped on the 1-GPU box): the gathered slabs must equal
the single-GPU run of the global grid bitwise (pin P10) and the oracle within 1e-12."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("d,h,shape,engine", [(2, 3, (200, 130), "rdg_cuda"), (2, 3, (130, 64), "tc"),
                                              (3, 1, (40, 20, 66), "rdg_cuda")])
def test_run_dist_one_rank_equals_run(d, h, shape, engine):
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W = synth.rsym_weights(d, h, 3)
    g = synth.grid(tuple(n + 2 * h for n in shape), 4)
    st = L.Stencil(W, shape, engine=engine)
    x = torch.from_numpy(g).cuda()
    a = torch.empty_like(x); b = torch.empty_like(x)
    st.run(x, a, 5)
    comm = L.lora_stencil_comm_init(1, 0, b"\0" * L.lora_stencil_comm_id_size())
    L.lora_stencil_run_dist(st.plan, comm, x.data_ptr(), b.data_ptr(), 5, torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert torch.equal(a, b)
    L.lora_stencil_comm_destroy(comm)


@pytest.mark.parametrize("d,h,shape,engine", [(2, 3, (300, 130), "rdg_cuda"), (2, 3, (300, 64), "tc"),
                                              (2, 2, (257, 99), "direct"), (3, 1, (200, 20, 66), "rdg_cuda"),
                                              (3, 1, (150, 24, 40), "tc"), (2, 1, (301, 67), "rdg_cuda")])
def test_run_dist_split_strips_bitwise(d, h, shape, engine, monkeypatch):
    """The overlapped schedule computes each step as two edge strips + the interior on row-range
    views of the arrays; it must equal the one-launch step bitwise (every point is computed by the
    same kernel code with the same neighbourhood)."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    monkeypatch.setenv("LORA_DIST_SPLIT", "1")
    W = synth.rsym_weights(d, h, 13)
    g = synth.grid(tuple(n + 2 * h for n in shape), 14)
    st = L.Stencil(W, shape, engine=engine, fuse_k=1)
    x = torch.from_numpy(g).cuda()
    a = torch.empty_like(x); b = torch.empty_like(x)
    st.run(x, a, 4)
    comm = L.lora_stencil_comm_init(1, 0, b"\0" * L.lora_stencil_comm_id_size())
    L.lora_stencil_run_dist(st.plan, comm, x.data_ptr(), b.data_ptr(), 4, torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert torch.equal(a, b)
    L.lora_stencil_comm_destroy(comm)


@pytest.mark.parametrize("d,h,shape", [(2, 3, (200, 130)), (2, 1, (150, 97)), (3, 1, (40, 20, 66))])
def test_run_dist_fused_path_one_rank(d, h, shape, monkeypatch):
    """The fused NCCL path (comm-owned deep-halo buffers, one exchange per fused launch; csrc/dist.cpp
    run_fused) on one rank (LORA_DIST_FUSED=1): equal to lora_stencil_run bitwise for T covering
    remainder launches, and repeated runs reuse the buffers."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    monkeypatch.setenv("LORA_DIST_FUSED", "1")
    W = synth.rsym_weights(d, h, 23)
    g = synth.grid(tuple(n + 2 * h for n in shape), 24)
    st = L.Stencil(W, shape)
    k = st.info()["fuse_k"]
    assert k > 1
    x = torch.from_numpy(g).cuda()
    comm = L.lora_stencil_comm_init(1, 0, b"\0" * L.lora_stencil_comm_id_size())
    for T in sorted({1, k, k + 1, 2 * k + 1}):
        a = torch.empty_like(x); b = torch.full_like(x, float("nan"))
        st.run(x, a, T)
        L.lora_stencil_run_dist(st.plan, comm, x.data_ptr(), b.data_ptr(), T, torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        assert torch.equal(a, b), T
    L.lora_stencil_comm_destroy(comm)


def _rank(rank, world, case, q, idq):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import paper_conf_sc_zhanglyczcy24_b200 as L
        from paper_conf_sc_zhanglyczcy24_b200 import dist as D
        torch.cuda.set_device(rank)
        d, h, shape, T, engine = case
        W = synth.rsym_weights(d, h, 5)
        g = synth.grid(tuple(n + 2 * h for n in shape), 6)
        start, cnt = D.slab_bounds(shape[0], world, rank, 64)
        local = np.ascontiguousarray(D.local_slice(g, start, cnt, h))
        st = L.Stencil(W, (cnt,) + tuple(shape[1:]), engine=engine)
        if rank == 0:
            uid = L.lora_stencil_comm_get_id()
            for _ in range(world - 1):
                idq.put(uid)
        else:
            uid = idq.get(timeout=60)
        comm = L.lora_stencil_comm_init(world, rank, uid)
        x = torch.from_numpy(local).cuda()
        y = torch.empty_like(x)
        L.lora_stencil_run_dist(st.plan, comm, x.data_ptr(), y.data_ptr(), T, torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        q.put((rank, start, y[h:h + cnt].cpu().numpy()))
        L.lora_stencil_comm_destroy(comm)
    except Exception:
        import traceback
        q.put((rank, -1, traceback.format_exc()))


@pytest.mark.parametrize("case", [(2, 3, (1000, 300), 7, "rdg_cuda"), (2, 3, (512, 200), 4, "tc"),
                                  (3, 1, (128, 40, 66), 5, "rdg_cuda")])
def test_run_dist_two_ranks_nccl_bitwise(case):
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs >= 2 GPUs")
    import paper_conf_sc_zhanglyczcy24_b200 as L
    world = 2
    ctx = mp.get_context("spawn")
    q, idq = ctx.Queue(), ctx.Queue()
    procs = [ctx.Process(target=_rank, args=(r, world, case, q, idq)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r, s, a in res:
        assert s >= 0, a
    d, h, shape, T, engine = case
    W = synth.rsym_weights(d, h, 5)
    g = synth.grid(tuple(n + 2 * h for n in shape), 6)
    st = L.Stencil(W, shape, engine=engine)
    x = torch.from_numpy(g).cuda(); y = torch.empty_like(x)
    st.run(x, y, T)
    ref = y.cpu().numpy()
    for r, s, a in res:
        assert np.array_equal(a, ref[h + s:h + s + a.shape[0]])


def test_nccl_binding_one_rank_communicator(monkeypatch):
    """Exercises the run-time NCCL binding on one GPU: dlopen of libnccl.so.2, ncclGetUniqueId,
    ncclCommInitRank with the 128-byte id passed by value, and ncclCommDestroy (LORA_FORCE_NCCL=1
    builds a real 1-rank communicator); a dist run on it equals the plain run."""
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    monkeypatch.setenv("LORA_FORCE_NCCL", "1")
    uid = L.lora_stencil_comm_get_id()
    assert len(uid) == 128 and any(uid)
    comm = L.lora_stencil_comm_init(1, 0, uid)
    W = synth.rsym_weights(2, 1, 2)
    g = synth.grid((130, 66), 3)
    st = L.Stencil(W, (128, 64))
    x = torch.from_numpy(g).cuda()
    a = torch.empty_like(x); b = torch.empty_like(x)
    st.run(x, a, 3)
    L.lora_stencil_run_dist(st.plan, comm, x.data_ptr(), b.data_ptr(), 3, torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert torch.equal(a, b)
    L.lora_stencil_comm_destroy(comm)
