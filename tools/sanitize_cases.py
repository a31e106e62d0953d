"""Small runs of every engine / staging path / fusion depth, for compute-sanitizer (tests/test_gpu_sanitizer.py)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sc_zhanglyczcy24_b200 as L
import synth

cases = [
    (2, 3, (67, 129), "rdg_cuda", 1), (2, 3, (67, 130), "rdg_cuda", 2), (2, 1, (70, 131), "rdg_cuda", 3),
    (2, 3, (67, 129), "tc", 1), (2, 1, (40, 66), "direct", 1),
    (3, 1, (17, 9, 33), "rdg_cuda", 1), (3, 1, (17, 20, 66), "rdg_cuda", 2), (3, 1, (17, 9, 34), "tc", 1),
    (3, 1, (9, 9, 33), "direct", 1),
]
for d, h, shape, eng, k in cases:
    W = synth.rsym_weights(d, h, 3)
    g = synth.grid(tuple(n + 2 * h for n in shape), 4)
    st = L.Stencil(W, shape, engine=eng, fuse_k=k)
    x = torch.from_numpy(g).cuda()
    y = torch.empty_like(x)
    st.run(x, y, 3)
    torch.cuda.synchronize()
    assert np.isfinite(y.cpu().numpy()).all()
    st.close()
# the device-initiated exchange path on one rank (no neighbours: the active-argument code paths, the
# view and the store window; kernels are serialised under the sanitizer, so two spinning ranks cannot run)
for d, h, shape, k in [(2, 3, (67, 129), 2), (2, 1, (70, 131), 1), (3, 1, (17, 9, 33), 1)]:
    W = synth.rsym_weights(d, h, 5)
    g = synth.grid(tuple(n + 2 * h for n in shape), 6)
    st = L.Stencil(W, shape, engine="rdg_cuda", fuse_k=k)
    ep = L.lora_stencil_p2p_create(st.plan, 1, 0)
    x = torch.from_numpy(g).cuda()
    y = torch.empty_like(x)
    L.lora_stencil_run_dist_p2p(st.plan, ep, x.data_ptr(), y.data_ptr(), 3, 0)
    torch.cuda.synchronize()
    L.lora_stencil_p2p_status(ep)
    assert np.isfinite(y.cpu().numpy()).all()
    L.lora_stencil_p2p_destroy(ep)
    st.close()
# 3D fused launches through the device-initiated exchange path (one rank: deep-halo view, store window)
for shape in [(17, 20, 66), (9, 9, 33)]:
    W = synth.rsym_weights(3, 1, 7)
    g = synth.grid(tuple(n + 2 for n in shape), 8)
    st = L.Stencil(W, shape, engine="rdg_cuda", fuse_k=2)
    ep = L.lora_stencil_p2p_create(st.plan, 1, 0)
    x = torch.from_numpy(g).cuda()
    y = torch.empty_like(x)
    L.lora_stencil_run_dist_p2p(st.plan, ep, x.data_ptr(), y.data_ptr(), 3, 0)
    torch.cuda.synchronize()
    L.lora_stencil_p2p_status(ep)
    assert np.isfinite(y.cpu().numpy()).all()
    L.lora_stencil_p2p_destroy(ep)
    st.close()
# the fused NCCL-path schedule on one rank (comm-owned deep-halo buffers)
os.environ["LORA_DIST_FUSED"] = "1"
W = synth.rsym_weights(2, 3, 9)
g = synth.grid((67 + 6, 130 + 6), 10)
st = L.Stencil(W, (67, 130), engine="rdg_cuda", fuse_k=2)
comm = L.lora_stencil_comm_init(1, 0, b"\0" * L.lora_stencil_comm_id_size())
x = torch.from_numpy(g).cuda()
y = torch.empty_like(x)
L.lora_stencil_run_dist(st.plan, comm, x.data_ptr(), y.data_ptr(), 5, 0)
torch.cuda.synchronize()
assert np.isfinite(y.cpu().numpy()).all()
L.lora_stencil_comm_destroy(comm)
st.close()
del os.environ["LORA_DIST_FUSED"]
# small 2D star grids: the single-launch kernels (cooperative grid, then the cluster variant)
for mode in ("grid", "cluster"):
    os.environ["LORA_SMALL_MODE"] = mode
    for h, shape in [(1, (64, 100)), (2, (48, 33))]:
        W = synth.star_weights(2, h, 11)
        g = synth.grid(tuple(n + 2 * h for n in shape), 12)
        st = L.Stencil(W, shape)
        assert st.info()["single_launch"] == 1
        x = torch.from_numpy(g).cuda()
        y = torch.empty_like(x)
        st.run(x, y, 6)
        torch.cuda.synchronize()
        assert np.isfinite(y.cpu().numpy()).all()
        st.close()
del os.environ["LORA_SMALL_MODE"]
print("sanitize cases ok")
