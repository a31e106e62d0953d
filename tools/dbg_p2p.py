"""Debug: run the fused P2P case per T and dump the flag words after a timeout."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_zhanglyczcy24_b200 as L
from paper_conf_sc_zhanglyczcy24_b200 import dist as D
import synth

h, shape, counts, k = 3, (300, 200), [150, 150], 2
W = synth.rsym_weights(2, h, 44)
g = synth.grid(tuple(n + 2 * h for n in shape), 43)
class DB:
    def __init__(self, ptr, n, t="<u8"):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": t, "data": (int(ptr), False), "version": 3, "strides": None}
for T in [int(a) for a in sys.argv[1:]] or [1, 2, 3]:
    P = len(counts); starts = [0, 150]
    sts, eps, xs, ys, ss = [], [], [], [], []
    for r in range(P):
        c = counts[r]
        st = L.Stencil(W, (c, shape[1]), engine="rdg_cuda", fuse_k=k); sts.append(st)
        eps.append(L.lora_stencil_p2p_create(st.plan, P, r))
        xs.append(torch.from_numpy(np.ascontiguousarray(D.local_slice(g, starts[r], c, h))).cuda())
        ys.append(torch.empty_like(xs[-1])); ss.append(torch.cuda.Stream())
    for r in range(P):
        L.lora_stencil_p2p_connect_local(eps[r], eps[r-1] if r > 0 else None, eps[r+1] if r < P-1 else None)
    torch.cuda.synchronize()
    for r in range(P):
        L.lora_stencil_run_dist_p2p(sts[r].plan, eps[r], xs[r].data_ptr(), ys[r].data_ptr(), T, ss[r].cuda_stream)
    torch.cuda.synchronize()
    for r in range(P):
        hl = h if r == 0 else k * h; hh = h if r == P - 1 else k * h
        elems = (hl + counts[r] + hh) * (shape[1] + 2 * h)
        bb = (elems * 8 + 255) // 256 * 256
        fl = torch.as_tensor(DB(L.lora_stencil_p2p_buffer(eps[r], 0) + 2 * bb, 8), device="cuda").cpu().numpy()
        try:
            L.lora_stencil_p2p_status(eps[r]); ok = "ok"
        except L.LoraError as e:
            ok = "TIMEOUT"
        print("T", T, "rank", r, ok, "flags lo-side", fl[:4].tolist(), "hi-side", fl[4:8].tolist(), flush=True)
