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
print("sanitize cases ok")
