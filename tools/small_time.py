"""Developer timing of the small-grid single-launch variants (Heat-2D 256^2 x 10 by default): CUDA-event
time per run over back-to-back runs (launch gaps amortised) and with an L2 flush before each run.
usage: python tools/small_time.py [--T 10] [--modes tile,grid,cluster]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import argparse
import json

import torch

import paper_conf_sc_zhanglyczcy24_b200 as L
import synth

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="heat2d-256")
ap.add_argument("--T", type=int, default=10)
ap.add_argument("--modes", default="tile,grid,cluster")
args = ap.parse_args()
W, c = synth.config(args.config)
x = torch.rand(c["padded"], dtype=torch.float64, device="cuda") + 0.5
y = torch.empty_like(x)
flush = torch.empty(64 << 20, dtype=torch.float64, device="cuda")
pts = float(c["shape"][0] * c["shape"][1]) * args.T
for mode in args.modes.split(","):
    os.environ["LORA_SMALL_MODE"] = "" if mode == "tile" else mode
    st = L.Stencil(W, c["shape"], engine="rdg_cuda")
    for _ in range(3):
        st.run(x, y, args.T)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 200
    e0.record()
    for _ in range(n):
        st.run(x, y, args.T)
    e1.record()
    torch.cuda.synchronize()
    b2b = e0.elapsed_time(e1) * 1e3 / n
    fl = []
    for _ in range(20):
        flush.zero_()
        e0.record(); st.run(x, y, args.T); e1.record()
        torch.cuda.synchronize()
        fl.append(e0.elapsed_time(e1) * 1e3)
    fl.sort()
    print(json.dumps({"mode": mode, "T": args.T, "us_back_to_back": round(b2b, 2), "us_flushed_median": round(fl[len(fl) // 2], 2),
                      "GS_s_flushed": round(pts / (fl[len(fl) // 2] * 1e-6) / 1e9, 1), "lib": os.environ.get("LORA_LIB", "in-tree")}), flush=True)
    st.close()
