"""B200 analogue of PAPER.md Fig. 9 (performance breakdown on Box-2D9P), over growing
grid sizes: RDG on CUDA cores -> tensor cores without BVS -> + BVS -> staging by LDGSTS vs TMA,
plus this build's defaults (CUDA-core RDG with exact temporal fusion) and the direct kernel.
Prints one JSON line per (size, variant)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_sc_zhanglyczcy24_b200 as L
import synth

VARIANTS = [
    ("rdg_cuda_core", dict(engine="rdg_cuda", fuse_k=1), {}),
    ("tc_no_bvs_ldgsts", dict(engine="tc"), {"LORA_TC_NO_BVS": "1", "LORA_NO_TMA": "1"}),
    ("tc_bvs_ldgsts", dict(engine="tc"), {"LORA_NO_TMA": "1"}),
    ("tc_bvs_tma", dict(engine="tc"), {}),
    ("tc_no_bvs_tma", dict(engine="tc"), {"LORA_TC_NO_BVS": "1"}),
    ("direct_cuda_core", dict(engine="direct"), {}),
    ("rdg_cuda_fused_k3", dict(engine="rdg_cuda", fuse_k=3), {}),
]
T = int(os.environ.get("ABL_T", "20"))
torch.cuda.set_stream(torch.cuda.Stream())
W = synth.rsym_weights(2, 1, 20240102)
for n in (1024, 2048, 4096, 8192, 10240):
    x = torch.rand((n + 2, n + 2), dtype=torch.float64, device="cuda") + 0.5
    y = torch.empty_like(x)
    for name, kw, env in VARIANTS:
        for k in ("LORA_TC_NO_BVS", "LORA_NO_TMA"):
            os.environ.pop(k, None)
        os.environ.update(env)
        st = L.Stencil(W, (n, n), **kw)
        st.run(x, y, T)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        best = 1e9
        for _ in range(3):
            e0.record(); st.run(x, y, T); e1.record(); torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1) / 1e3)
        print(json.dumps({"size": n, "variant": name, "T": T, "GStencil_s": round(n * n * T / best / 1e9, 2),
                          "fma_per_point_issued": st.info()["fma_per_point_issued"]}), flush=True)
        st.close()
    for k in ("LORA_TC_NO_BVS", "LORA_NO_TMA"):
        os.environ.pop(k, None)
