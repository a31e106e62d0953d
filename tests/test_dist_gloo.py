"""Multi-process (world_size 2 and 3, gloo, CPU) tests of the slab-decomposition host logic:
the slab split (dist.slab_bounds), the local padded slices, and the native halo-exchange plan
(lora_stencil_dist_exchange_plan, the same plan csrc/dist.cpp issues through NCCL) executed with
torch.distributed send/recv.  Each rank steps its slab with the oracle (test infrastructure);
the gathered result must equal the single-domain oracle bitwise (pin P10's host half)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, case, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import torch.distributed as dist

        import oracle
        import paper_conf_sc_zhanglyczcy24_b200 as L
        import synth
        from paper_conf_sc_zhanglyczcy24_b200 import dist as D

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        d, h, shape, T, align = case
        W = synth.rsym_weights(d, h, 77) if d == 2 else synth.rsym_weights(d, h, 78)
        g = synth.grid(tuple(n + 2 * h for n in shape), 123)
        start, cnt = D.slab_bounds(shape[0], world, rank, align)
        local = np.ascontiguousarray(D.local_slice(g, start, cnt, h)).copy()
        lshape = (cnt,) + tuple(shape[1:])
        plan = L.lora_stencil_plan(W, d, h, lshape)
        xplan = L.lora_stencil_dist_exchange_plan(plan, rank, world)
        flat = torch.from_numpy(local).view(-1)
        for _ in range(T):
            local = oracle.run(W, local, 1)          # one step of this slab (halo rows held fixed)
            flat = torch.from_numpy(local).view(-1)
            reqs = []
            for kind, peer, off, n in xplan:
                buf = flat[off:off + n]
                reqs.append(dist.isend(buf.clone(), peer) if kind == "send" else (dist.irecv(buf_r := torch.empty(n, dtype=torch.float64), peer), buf, buf_r))
            for r in reqs:
                if isinstance(r, tuple):
                    r[0].wait()
                    r[1].copy_(r[2])
                else:
                    r.wait()
            local = flat.view(local.shape).numpy()
        inner = torch.from_numpy(np.ascontiguousarray(local[h:h + cnt]))
        parts = [None] * world
        dist.all_gather_object(parts, (start, inner.numpy()))
        if rank == 0:
            full = oracle.run(W, g, T)
            out = g.copy()
            for s, a in parts:
                out[h + s:h + s + a.shape[0]] = a
            # interior rows must match bitwise; columns' halo is carried along in each slab
            q.put(("ok", bool(np.array_equal(out, full)), float(np.max(np.abs(out - full)))))
            # exchanged halos of each slab equal the neighbours' rows of the global result
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - surfaced by the parent
        import traceback
        q.put(("err", traceback.format_exc(), 0.0))


@pytest.mark.parametrize("world,case", [
    (2, (2, 3, (37, 29), 4, 1)),
    (2, (2, 1, (64, 40), 5, 8)),
    (3, (2, 2, (23, 17), 3, 1)),     # uneven split
    (2, (3, 1, (13, 9, 11), 3, 1)),
    (3, (3, 2, (14, 7, 9), 2, 1)),
])
def test_slab_exchange_gloo_equals_single_domain(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=120)
    assert res[0] == "ok", res[1]
    assert res[1], f"max diff {res[2]}"


def test_slab_bounds_cover_and_align():
    from paper_conf_sc_zhanglyczcy24_b200 import dist as D
    for N0, P, a in [(10240, 8, 64), (100, 3, 1), (37, 2, 4), (5, 5, 1)]:
        spans = [D.slab_bounds(N0, P, r, a) for r in range(P)]
        assert spans[0][0] == 0 and sum(c for _, c in spans) == N0
        for (s0, c0), (s1, _) in zip(spans, spans[1:]):
            assert s0 + c0 == s1
        for s, _ in spans:
            assert s % a == 0


def test_exchange_plan_offsets():
    import synth
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W = synth.rsym_weights(2, 3, 1)
    plan = L.lora_stencil_plan(W, 2, 3, (50, 20))
    row = 26
    assert L.lora_stencil_dist_exchange_plan(plan, 0, 1) == []
    assert L.lora_stencil_dist_exchange_plan(plan, 0, 2) == [("send", 1, 50 * row, 3 * row), ("recv", 1, 53 * row, 3 * row)]
    assert L.lora_stencil_dist_exchange_plan(plan, 1, 2) == [("send", 0, 3 * row, 3 * row), ("recv", 0, 0, 3 * row)]
    assert len(L.lora_stencil_dist_exchange_plan(plan, 1, 3)) == 4


def _worker_fused(rank, world, port, case, q):
    """Deep-halo variant (the fused NCCL path of csrc/dist.cpp run_fused): each rank holds its slab
    with H = k R deep halos at internal edges (hl + n0 + hh rows), steps the WHOLE buffer k steps at a
    time as one padded array (the oracle stands in for the fused kernel: its deep-halo rows are
    recomputed and go stale), then exchanges H rows per side with the native deep-halo plan
    (lora_stencil_dist_exchange_plan_ex).  Own rows must equal the single-domain oracle bitwise."""
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import torch.distributed as dist

        import oracle
        import paper_conf_sc_zhanglyczcy24_b200 as L
        import synth
        from paper_conf_sc_zhanglyczcy24_b200 import dist as D

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        d, h, shape, T, k = case
        W = synth.rsym_weights(d, h, 79)
        g = synth.grid(tuple(n + 2 * h for n in shape), 125)
        start, cnt = D.slab_bounds(shape[0], world, rank, 1)
        H = k * h
        hl = H if rank > 0 else h
        hh = H if rank < world - 1 else h
        lo = start + h - hl                         # global padded row of buffer row 0
        buf = np.ascontiguousarray(g[lo:lo + hl + cnt + hh]).copy()
        plan = L.lora_stencil_plan(W, d, h, (cnt,) + tuple(shape[1:]))
        xplan = L.lora_stencil_dist_exchange_plan(plan, rank, world, halo_depth=H)

        def exchange(b):
            flat = torch.from_numpy(b).view(-1)
            reqs = []
            for kind, peer, off, n in xplan:
                if kind == "send":
                    reqs.append(dist.isend(flat[off:off + n].clone(), peer))
                else:
                    tmp = torch.empty(n, dtype=torch.float64)
                    reqs.append((dist.irecv(tmp, peer), off, n, tmp))
            for r in reqs:
                if isinstance(r, tuple):
                    r[0].wait()
                    flat[r[1]:r[1] + r[2]].copy_(r[3])
                else:
                    r.wait()
            return flat.view(b.shape).numpy()

        done = 0
        while done < T:
            kk = min(k, T - done)
            buf = exchange(oracle.run(W, buf, kk))
            done += kk
        own = buf[hl:hl + cnt]
        parts = [None] * world
        dist.all_gather_object(parts, (start, own))
        if rank == 0:
            full = oracle.run(W, g, T)
            ok = all(np.array_equal(a, full[h + s:h + s + a.shape[0]]) for s, a in parts)
            q.put(("ok", ok, 0.0))
        dist.destroy_process_group()
    except Exception:  # pragma: no cover - surfaced by the parent
        import traceback
        q.put(("err", traceback.format_exc(), 0.0))


@pytest.mark.parametrize("world,case", [
    (2, (2, 3, (40, 23), 5, 2)),       # Box-2D49P radius, k = 2 (the fused NCCL depth), remainder step
    (3, (2, 1, (30, 17), 7, 3)),       # radius 1, k = 3, uneven split
    (3, (3, 1, (12, 7, 9), 5, 2)),     # 3D, slabs of exactly H = 2 planes in the middle
])
def test_deep_halo_exchange_gloo_equals_single_domain(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_fused, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=120)
    assert res[0] == "ok", res[1]
    assert res[1]


def test_deep_halo_exchange_plan_offsets():
    import synth
    import paper_conf_sc_zhanglyczcy24_b200 as L
    W = synth.rsym_weights(2, 3, 1)
    plan = L.lora_stencil_plan(W, 2, 3, (50, 20))
    row, H = 26, 6
    # halo_depth = R reproduces the caller-layout plan
    assert L.lora_stencil_dist_exchange_plan(plan, 1, 3, halo_depth=3) == L.lora_stencil_dist_exchange_plan(plan, 1, 3)
    assert L.lora_stencil_dist_exchange_plan(plan, 0, 2, halo_depth=H) == [("send", 1, (3 + 50 - H) * row, H * row),
                                                                            ("recv", 1, (3 + 50) * row, H * row)]
    assert L.lora_stencil_dist_exchange_plan(plan, 1, 2, halo_depth=H) == [("send", 0, H * row, H * row), ("recv", 0, 0, H * row)]
    with pytest.raises(L.LoraError):
        L.lora_stencil_dist_exchange_plan(plan, 0, 2, halo_depth=2)   # shallower than the radius
