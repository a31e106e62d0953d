"""Tiny driver for ncu: plan one workload/engine and run a few steps (torch.rand input)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import argparse
import torch
import paper_conf_sc_zhanglyczcy24_b200 as L
import synth

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="box2d49p-10240")
ap.add_argument("--engine", default="auto")
ap.add_argument("--fuse", type=int, default=0)
ap.add_argument("--T", type=int, default=4)
a = ap.parse_args()
W, c = synth.config(a.workload)
st = L.Stencil(W, c["shape"], engine=a.engine, fuse_k=a.fuse)
x = torch.rand(c["padded"], dtype=torch.float64, device="cuda") + 0.5
y = torch.empty_like(x)
st.run(x, y, a.T)
torch.cuda.synchronize()
print(st.info())
