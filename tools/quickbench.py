"""Developer timing loop: GS/s per config x engine (CUDA events), not the bench contract."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import argparse
import json
import time

import numpy as np
import torch

import paper_conf_sc_zhanglyczcy24_b200 as L
import synth

ap = argparse.ArgumentParser()
ap.add_argument("--configs", default="box2d9p-10240,box2d49p-10240,heat3d-512,box3d27p-512")
ap.add_argument("--engines", default="direct,tc")
ap.add_argument("--T", type=int, default=20)
ap.add_argument("--fuse", default="1")
args = ap.parse_args()
torch.cuda.set_stream(torch.cuda.Stream())  # a capturable stream (CUDA graphs for small grids)
for name in args.configs.split(","):
    W, c = synth.config(name)
    x = torch.rand(c["padded"], dtype=torch.float64, device="cuda") + 0.5
    y = torch.empty_like(x)
    for eng in args.engines.split(","):
        for fk in [int(f) for f in args.fuse.split(",")]:
            try:
                st = L.Stencil(W, c["shape"], engine=eng, fuse_k=fk)
            except Exception as e:
                print(json.dumps({"config": name, "engine": eng, "error": str(e)}))
                continue
            st.run(x, y, 2)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            best = 1e9
            for _ in range(3):
                e0.record(); st.run(x, y, args.T); e1.record(); torch.cuda.synchronize()
                best = min(best, e0.elapsed_time(e1) / 1e3)
            pts = float(np.prod(c["shape"])) * args.T
            print(json.dumps({"config": name, "engine": eng, "fuse_k": fk, "T": args.T, "s": round(best, 5),
                              "GStencil_s": round(pts / best / 1e9, 2), "info": {k: st.info()[k] for k in ("engine_name", "fma_per_point_issued", "n_terms")}}), flush=True)
            st.close()
