"""CPU check of the single-launch cluster schedule of kernels_small.cu (host logic, -m "not gpu").

The kernel keeps each CTA's slab (rp own rows + an HK = k R deep halo on each side) in shared
memory, runs k steps per block on a shrinking row range, hands its first / last HK own rows to the
neighbours' double-buffered mailboxes and unpacks its own mailbox (interior columns only) after one
cluster barrier per block.  This numpy emulation runs exactly that schedule — buffer-row mapping,
per-step row ranges, mailbox rows and parities, unpack, write-back — with the star arms' update,
and must equal the oracle (eq. 2) for T spanning several blocks.  The GPU test
tests/test_gpu_parity.py::test_small_cluster_path_bitwise checks the kernel itself."""
import numpy as np
import pytest

import oracle
import synth


def _emulate(W, g, T, R, cs, kb):
    P0, P1 = g.shape
    N0, N1 = P0 - 2 * R, P1 - 2 * R
    rp, HK = N0 // cs, kb * R
    SR = rp + 2 * HK
    h = W[R, :].copy()
    v = W[:, R].copy()
    v[R] = 0.0
    mbox = [np.zeros((4, HK, P1)) for _ in range(cs)]
    bufs, cur = [], [0] * cs
    for c in range(cs):
        pr0 = c * rp + R - HK
        b = np.zeros((SR, P1))
        for j in range(SR):
            if 0 <= pr0 + j < P0:
                b[j] = g[pr0 + j]
        bufs.append([b.copy(), b.copy()])
    xs = np.arange(R, R + N1)
    t0 = blk = 0
    while t0 < T:
        ks, par = min(kb, T - t0), blk & 1
        for c in range(cs):
            pr0 = c * rp + R - HK
            jlo, jhi = max(R, R - pr0), min(SR - R, P0 - R - pr0)
            for st in range(1, ks + 1):
                src, dst = bufs[c][cur[c]], bufs[c][cur[c] ^ 1]
                for j in range(max(jlo, R * st + HK - R * ks), min(jhi, SR - R * st - (HK - R * ks))):
                    th = np.zeros(N1)
                    for b in range(-R, R + 1):
                        th = h[R + b] * src[j, xs + b] + th
                    acc = np.zeros(N1)
                    for a in range(-R, R + 1):
                        if a == 0:
                            acc = acc + th
                        acc = v[R + a] * src[j + a, xs] + acc
                    dst[j, xs] = acc
                    if st == ks and c > 0 and HK <= j < 2 * HK:
                        mbox[c - 1][2 * par + 1][j - HK, xs] = acc
                    if st == ks and c < cs - 1 and rp <= j < rp + HK:
                        mbox[c + 1][2 * par + 0][j - rp, xs] = acc
                cur[c] ^= 1
        if t0 + ks < T:
            for c in range(cs):
                d = bufs[c][cur[c]]
                if c > 0:
                    d[0:HK, xs] = mbox[c][2 * par + 0][:, xs]
                if c < cs - 1:
                    d[HK + rp:SR, xs] = mbox[c][2 * par + 1][:, xs]
        t0 += ks
        blk += 1
    out = np.zeros_like(g)
    for c in range(cs):
        pr0 = c * rp + R - HK
        w0 = HK - R if c == 0 else HK
        w1 = HK + rp + R if c == cs - 1 else HK + rp
        for j in range(w0, w1):
            out[pr0 + j] = bufs[c][cur[c]][j]
    return out


@pytest.mark.parametrize("R,cs,kb,shape", [(1, 16, 8, (256, 40)), (3, 16, 2, (256, 50)), (2, 8, 3, (48, 33)),
                                           (4, 4, 2, (32, 20))])
def test_cluster_schedule_matches_oracle(R, cs, kb, shape):
    W = synth.preset("heat2d") if R == 1 else synth.star_weights(2, R, 41 + R)
    g = synth.grid(tuple(n + 2 * R for n in shape), 43)
    for T in (1, kb, kb + 1, 2 * kb + 1, 3 * kb):
        out = _emulate(W, g, T, R, cs, kb)
        assert np.max(np.abs(out - oracle.run(W, g, T))) <= 1e-14, T
