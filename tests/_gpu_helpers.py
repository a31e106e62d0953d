"""Helpers for the -m gpu parity tests: run the CUDA path through the C-ABI on torch tensors."""
import numpy as np


def run_gpu(W, grid, T, engine="auto", fuse_k=0, stream=None):
    import torch
    import paper_conf_sc_zhanglyczcy24_b200 as L
    h = (W.shape[0] - 1) // 2
    shape = tuple(s - 2 * h for s in grid.shape)
    st = L.Stencil(W, shape, engine=engine, fuse_k=fuse_k)
    x = torch.from_numpy(np.ascontiguousarray(grid)).cuda()
    y = torch.full_like(x, float("nan"))
    st.run(x, y, T, stream)
    torch.cuda.synchronize()
    out = y.cpu().numpy()
    info = st.info()
    st.close()
    return out, info


def rel_err(a, b):
    return float(np.max(np.abs(a - b)) / max(float(np.max(np.abs(b))), 1e-300))
