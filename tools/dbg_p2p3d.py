"""Debug: one 3D fused p2p case per T in a subprocess with a timeout; prints pass/fail per T."""
import os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CODE = r'''
import sys; sys.path.insert(0, %r)
import numpy as np
from tests.test_gpu_p2p import _weights, _run_local, _global
import synth
kind, shape, counts, k, T = %r
W = _weights(kind, 3, 1, 47)
g = synth.grid(tuple(n + 2 for n in shape), 53)
ref = _global(W, g, T, "rdg_cuda", fuse_k=k)
try:
    out = _run_local(W, g, 1, shape, T, "rdg_cuda", counts, fuse_k=k)
    d = np.abs(out - ref); bad = np.argwhere(d > 0)
    print("T", T, "maxdiff", float(d.max()), "bad planes", sorted(set(bad[:, 0].tolist()))[:20])
except Exception as e:
    print("T", T, "ERROR", e)
'''
cases = [("heat3d", (130, 12, 40), [64, 2, 64], 2), ("rsym", (96, 20, 66), [48, 48], 2), ("rsym", (96, 20, 66), [48, 2, 46], 2),
         ("heat3d", (130, 12, 40), [64, 66], 2)]
for c in cases:
    for T in (1, 2, 3, 5):
        try:
            r = subprocess.run([sys.executable, "-c", CODE % (ROOT, c + (T,))], capture_output=True, text=True, timeout=120)
            print(c, (r.stdout.strip().splitlines() or [""])[-1], r.stderr.strip().splitlines()[-1:] if r.returncode else "")
        except subprocess.TimeoutExpired:
            print(c, "T", T, "TIMEOUT")
        sys.stdout.flush()
