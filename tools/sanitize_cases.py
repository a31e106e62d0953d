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
print("sanitize cases ok")
