"""Plain single-GPU timing of a workload's weights on an arbitrary interior shape (developer tool)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import json
import numpy as np
import torch
import paper_conf_sc_zhanglyczcy24_b200 as L
import synth

name = sys.argv[1]
shape = tuple(int(v) for v in sys.argv[2].split("x"))
T = int(sys.argv[3]) if len(sys.argv) > 3 else 100
W, c = synth.config(name)
R = (W.shape[0] - 1) // 2
x = torch.rand(tuple(n + 2 * R for n in shape), dtype=torch.float64, device="cuda") + 0.5
y = torch.empty_like(x)
st = L.Stencil(W, shape, engine="rdg_cuda")
st.run(x, y, 4)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
best = 1e9
for _ in range(3):
    e0.record(); st.run(x, y, T); e1.record(); torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1) / 1e3)
print(json.dumps({"workload": name, "shape": shape, "T": T, "GStencil_s": round(float(np.prod(shape)) * T / best / 1e9, 1)}))
