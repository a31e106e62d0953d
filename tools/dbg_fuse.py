import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_zhanglyczcy24_b200 as L, synth, oracle
h = int(sys.argv[1]); k = int(sys.argv[2]); shape = (int(sys.argv[3]), int(sys.argv[4])); T = int(sys.argv[5])
W = synth.rsym_weights(2, h, 3)
g = synth.grid(tuple(n + 2*h for n in shape), 1)
st = L.Stencil(W, shape, engine="rdg_cuda", fuse_k=k)
x = torch.from_numpy(g).cuda(); y = torch.empty_like(x)
st.run(x, y, T); torch.cuda.synchronize()
ref = oracle.run(W, g, T)
print("h", h, "k", k, shape, "T", T, "err", float(np.max(np.abs(y.cpu().numpy() - ref))))
