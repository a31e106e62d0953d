// K6 — Residual Dimension Gathering on the FP64 CUDA-core pipe (Fig. 9 "RDG on CUDA
// cores"; §III-B/§III-C applied term by term, eq. 9).
//
// Each rank-1 term u_k v_k^T is applied as the same two gathers as the tensor-core chain
// U_k X V_k (eq. 7), but on the DFMA pipe and without band padding:
//   horizontal gather  T_k[r][x] = sum_b v_k[b] X[r][x+b]          (one input row r)
//   vertical gather    P[y][x]  += sum_a u_k[a] T_k[y+a][x]         (register ring over rows)
// On B200 DMMA.8x8x4 and DFMA share one FP64 budget (tools/ubench, DESIGN.md §Step 0), so the
// band zeros the tensor-core chain multiplies (K = 16 for a 7-tap band) are pure loss; this form
// issues the separable minimum sum_k (len u_k + len v_k) FMAs per point (+ halo rows per chunk).
//
// Mapping: one WARP streams a 64-column band of a chunk of RC output rows.  Lane p owns the
// output columns 2p, 2p+1.  Input rows arrive through a per-warp ring of NS shared-memory stages
// (TMA box SROWS x (64+2R), zero fill outside the array; LDGSTS fallback).  For every input row
// the lane reads its 2R+2 neighbours with R+1 LDS.128, forms T_k for every term (X is read once
// for all terms, the PMA reuse of P:290) and scatters u_k[a] T_k into the accumulator ring of the
// 2R+1 output rows in flight.  Output row y is complete after input row y + 2R and is stored.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "kernels.hpp"
#include "pipe.cuh"

namespace lora {
namespace {

constexpr int RDG_RC = 128;     // output rows per work item (chunk)
constexpr int RDG_WARPS = 4;    // warps per CTA (independent streams)
constexpr int RDG_NS = 4;       // ring stages per warp

enum { SIG_PMA = 0, SIG_STAR = 1, SIG_FULL = 2 };

struct RdgParams {
  int K;                     // number of (u, v) chain terms used by the signature
  double u[kMaxN][kMaxN];    // centred, length 2R+1
  double v[kMaxN][kMaxN];
  double c;                  // PMA scalar C_{h+1}
};

template <int R>
struct Geom {
  static constexpr int n = 2 * R + 1;
  static constexpr int m = n >= 6 ? 1 : 2;
  static constexpr int SROWS = n * m;                                  // rows per stage (multiple of n)
  static constexpr int BW = 64 + 2 * R;                                // staged columns
  static constexpr int STAGE = ((SROWS * BW * 8 + 127) / 128) * 128;   // bytes per stage
  static constexpr int SI = (RDG_RC + 2 * R + SROWS - 1) / SROWS;      // stages per work item
  static constexpr int WARP_BYTES = RDG_NS * STAGE;
  static constexpr int SMEM = 128 + RDG_WARPS * WARP_BYTES;
};

__host__ __device__ constexpr int pmod(int a, int n) { return ((a % n) + n) % n; }

// One input row r (r mod n == I mod n) of the stream: T for every term, scattered into the ring.
template <int R, int SIG, int I>
__device__ __forceinline__ void row_body(const double* __restrict__ xs, int p, double (&acc)[2 * R + 1][2],
                                         const RdgParams& P) {
  constexpr int n = 2 * R + 1;
  double x[2 * R + 2];
#pragma unroll
  for (int q = 0; q <= R; ++q) {
    const double2 t = *reinterpret_cast<const double2*>(xs + 2 * p + 2 * q);
    x[2 * q] = t.x;
    x[2 * q + 1] = t.y;
  }
  if constexpr (SIG == SIG_PMA) {
    // PMA pyramid (eq. 15): term k has radius R-k; the last one is the scalar C_{h+1}.
#pragma unroll
    for (int k = 0; k < R; ++k) {
      const int H = R - k;
      double t0 = 0.0, t1 = 0.0;
#pragma unroll
      for (int b = -H; b <= H; ++b) {
        t0 = fma(P.v[k][R + b], x[R + b], t0);
        t1 = fma(P.v[k][R + b], x[R + b + 1], t1);
      }
#pragma unroll
      for (int a = -H; a <= H; ++a) {
        const int s = pmod(I - R - a, n);
        acc[s][0] = fma(P.u[k][R + a], t0, acc[s][0]);
        acc[s][1] = fma(P.u[k][R + a], t1, acc[s][1]);
      }
    }
    constexpr int s0 = pmod(I - R, n);
    acc[s0][0] = fma(P.c, x[R], acc[s0][0]);
    acc[s0][1] = fma(P.c, x[R + 1], acc[s0][1]);
  } else if constexpr (SIG == SIG_STAR) {
    // star arms: horizontal arm (u = e_R) lands on the centre row; vertical arm (v = e_R) is X itself.
    double t0 = 0.0, t1 = 0.0;
#pragma unroll
    for (int b = -R; b <= R; ++b) {
      t0 = fma(P.v[0][R + b], x[R + b], t0);
      t1 = fma(P.v[0][R + b], x[R + b + 1], t1);
    }
    constexpr int s0 = pmod(I - R, n);
    acc[s0][0] += t0;
    acc[s0][1] += t1;
#pragma unroll
    for (int a = -R; a <= R; ++a) {
      const int s = pmod(I - R - a, n);
      acc[s][0] = fma(P.u[1][R + a], x[R], acc[s][0]);
      acc[s][1] = fma(P.u[1][R + a], x[R + 1], acc[s][1]);
    }
  } else {
    // general: K <= 2R+1 full-radius rank-1 terms (complete-pivot elimination, Q6)
#pragma unroll
    for (int k = 0; k < n; ++k) {
      if (k < P.K) {
        double t0 = 0.0, t1 = 0.0;
#pragma unroll
        for (int b = -R; b <= R; ++b) {
          t0 = fma(P.v[k][R + b], x[R + b], t0);
          t1 = fma(P.v[k][R + b], x[R + b + 1], t1);
        }
#pragma unroll
        for (int a = -R; a <= R; ++a) {
          const int s = pmod(I - R - a, n);
          acc[s][0] = fma(P.u[k][R + a], t0, acc[s][0]);
          acc[s][1] = fma(P.u[k][R + a], t1, acc[s][1]);
        }
      }
    }
  }
}

template <int R, int SIG, int I>
__device__ __forceinline__ void stage_rows(const double* __restrict__ st, int p, double (&acc)[2 * R + 1][2],
                                           const RdgParams& P, int rbase, double* __restrict__ orow0, int64_t P1,
                                           int rows_valid, bool c0ok, bool c1ok, bool vec) {
  constexpr int n = 2 * R + 1;
  if constexpr (I < Geom<R>::SROWS) {
    row_body<R, SIG, I % n>(st + I * Geom<R>::BW, p, acc, P);
    // output row y = r - 2R is complete; its ring slot is (I + 1) mod n
    constexpr int s = (I + 1) % n;
    const int y = rbase + I - 2 * R;
    if (y >= 0 && y < rows_valid) {
      double* o = orow0 + int64_t(y) * P1;
      if (vec) {
        *reinterpret_cast<double2*>(o) = make_double2(acc[s][0], acc[s][1]);
      } else {
        if (c0ok) o[0] = acc[s][0];
        if (c1ok) o[1] = acc[s][1];
      }
    }
    acc[s][0] = 0.0;
    acc[s][1] = 0.0;
    stage_rows<R, SIG, I + 1>(st, p, acc, P, rbase, orow0, P1, rows_valid, c0ok, c1ok, vec);
  }
}

template <int R, int SIG, bool TMA>
__global__ void __launch_bounds__(RDG_WARPS * 32, 4) rdg2d_kernel(const double* __restrict__ in, double* __restrict__ out,
                                                              int64_t N0, int64_t N1, int nbands, int nitems,
                                                              const __grid_constant__ CUtensorMap tmap,
                                                              const __grid_constant__ RdgParams prm) {
  using G = Geom<R>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw) + wl * RDG_NS;
  unsigned char* ring = smem_raw + 128 + wl * G::WARP_BYTES;
  const int64_t P1 = N1 + 2 * R, P0 = N0 + 2 * R;
  const int gw = blockIdx.x * RDG_WARPS + wl, TW = gridDim.x * RDG_WARPS;
  const int my_items = gw < nitems ? (nitems - 1 - gw) / TW + 1 : 0;
  const int nstages = my_items * G::SI;
  if (TMA && lane == 0) {
    for (int s = 0; s < RDG_NS; ++s) mbar_init(&bars[s], 1);
    fence_barrier_init();
  }
  __syncwarp();
  auto issue = [&](int q) {  // stage q of this warp's sequence into slot q % NS
    const int item = gw + (q / G::SI) * TW, j = q % G::SI;
    const int band = item % nbands, chunk = item / nbands;
    const int64_t y = int64_t(chunk) * RDG_RC + int64_t(j) * G::SROWS, x = int64_t(band) * 64;
    double* dst = reinterpret_cast<double*>(ring + (q % RDG_NS) * G::STAGE);
    if constexpr (TMA) {
      if (lane == 0) {
        mbar_arrive_expect_tx(&bars[q % RDG_NS], G::SROWS * G::BW * 8);
        tma_load_2d(dst, &tmap, (int)x, (int)y, &bars[q % RDG_NS]);
      }
    } else {
      for (int i = lane; i < G::SROWS * G::BW; i += 32) {
        const int r = i / G::BW, c = i - r * G::BW;
        const int64_t gy = y + r, gx = x + c;
        if (gy < P0 && gx < P1) cp_async8(dst + i, in + gy * P1 + gx);
        else dst[i] = 0.0;
      }
      cp_async_commit();
    }
  };
  for (int q = 0; q < RDG_NS - 1; ++q) {
    if (q < nstages) issue(q);
    else if constexpr (!TMA) cp_async_commit();  // empty group: keeps wait_group<NS-1> exact
  }
  double acc[2 * R + 1][2];
  for (int q = 0; q < nstages; ++q) {
    if (q + RDG_NS - 1 < nstages) issue(q + RDG_NS - 1);
    else if constexpr (!TMA) cp_async_commit();  // keep the group count uniform
    if constexpr (TMA) {
      mbar_wait(&bars[q % RDG_NS], (q / RDG_NS) & 1);
    } else {
      cp_async_wait<RDG_NS - 1>();
      __syncwarp();
    }
    const int item = gw + (q / G::SI) * TW, j = q % G::SI;
    const int band = item % nbands, chunk = item / nbands;
    if (j == 0) {
#pragma unroll
      for (int s = 0; s < 2 * R + 1; ++s) { acc[s][0] = 0.0; acc[s][1] = 0.0; }
    }
    const int64_t row0 = int64_t(chunk) * RDG_RC;             // first output row (interior) of the chunk
    const int64_t col = int64_t(band) * 64 + 2 * lane;        // first output column (interior) of the lane
    const int rows_valid = (int)std::min<int64_t>(RDG_RC, N0 - row0);
    double* orow0 = out + (row0 + R) * P1 + R + col;
    const bool c0ok = col < N1, c1ok = col + 1 < N1;
    const bool vec = c1ok && ((reinterpret_cast<uintptr_t>(orow0) & 15) == 0) && ((P1 & 1) == 0);
    const double* st = reinterpret_cast<const double*>(ring + (q % RDG_NS) * G::STAGE);
    stage_rows<R, SIG, 0>(st, lane, acc, prm, j * G::SROWS, orow0, P1, rows_valid, c0ok, c1ok, vec);
    __syncwarp();  // every lane is done with slot q % NS before it is refilled
  }
}

int signature(const Plan& p, RdgParams& prm) {
  std::memset(&prm, 0, sizeof(prm));
  const int R = p.R, n = 2 * R + 1;
  // PMA pyramid: chains of radius R, R-1, ..., 1 (in that order) + centre scalar
  bool pma = (int)p.terms.size() == R + 1;
  for (int k = 0; pma && k < R; ++k) pma = p.terms[k].kind == kChain && p.terms[k].r == R - k;
  if (pma) pma = p.terms[R].kind == kPoint && p.terms[R].u[R] == 1.0 && p.terms[R].r == 0;
  if (pma) {
    prm.K = R;
    for (int k = 0; k < R; ++k)
      for (int i = 0; i < n; ++i) { prm.u[k][i] = p.terms[k].u[i]; prm.v[k][i] = p.terms[k].v[i]; }
    prm.c = p.terms[R].v[R];
    return SIG_PMA;
  }
  // star: horizontal arm (u = e_R) then vertical arm (v = e_R)
  if (p.terms.size() == 2 && p.terms[0].kind == kArm && p.terms[1].kind == kArm && p.terms[0].u[R] == 1.0 &&
      p.terms[1].v[R] == 1.0) {
    bool ok = true;
    for (int i = 0; i < n; ++i) {
      if (i != R && (p.terms[0].u[i] != 0.0 || p.terms[1].v[i] != 0.0)) ok = false;
    }
    if (ok) {
      prm.K = 2;
      for (int i = 0; i < n; ++i) { prm.v[0][i] = p.terms[0].v[i]; prm.u[1][i] = p.terms[1].u[i]; }
      return SIG_STAR;
    }
  }
  if ((int)p.terms.size() > n) return -1;
  prm.K = (int)p.terms.size();
  for (int k = 0; k < prm.K; ++k)
    for (int i = 0; i < n; ++i) { prm.u[k][i] = p.terms[k].u[i]; prm.v[k][i] = p.terms[k].v[i]; }
  return SIG_FULL;
}

template <int R, int SIG, bool TMA>
cudaError_t rdg_launch(const Plan& p, const double* src, double* dst, cudaStream_t s, const CUtensorMap& map,
                       const RdgParams& prm) {
  using G = Geom<R>;
  static int max_grid = 0;
  if (max_grid == 0) {
    cudaError_t e = cudaFuncSetAttribute(rdg2d_kernel<R, SIG, TMA>, cudaFuncAttributeMaxDynamicSharedMemorySize, G::SMEM);
    if (e != cudaSuccess) return e;
    max_grid = persistent_grid((const void*)rdg2d_kernel<R, SIG, TMA>, RDG_WARPS * 32, G::SMEM, int64_t(1) << 40);
  }
  const int nbands = (int)((p.N[1] + 63) / 64), nchunks = (int)((p.N[0] + RDG_RC - 1) / RDG_RC);
  const int nitems = nbands * nchunks;
  const int grid = (int)std::min<int64_t>(max_grid, (nitems + RDG_WARPS - 1) / RDG_WARPS);
  rdg2d_kernel<R, SIG, TMA><<<grid, RDG_WARPS * 32, G::SMEM, s>>>(src, dst, p.N[0], p.N[1], nbands, nitems, map, prm);
  return cudaGetLastError();
}

template <int R, int SIG>
cudaError_t rdg_sig(const Plan& p, const double* src, double* dst, cudaStream_t s, const RdgParams& prm) {
  using G = Geom<R>;
  CUtensorMap map;
  const int64_t padded[2] = {p.P[0], p.P[1]};
  const int box[2] = {G::SROWS, G::BW};
  if (!p.force_no_tma && encode_tmap(&map, src, 2, padded, box)) return rdg_launch<R, SIG, true>(p, src, dst, s, map, prm);
  std::memset(&map, 0, sizeof(map));
  return rdg_launch<R, SIG, false>(p, src, dst, s, map, prm);
}

template <int R>
cudaError_t rdg_r(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  RdgParams prm;
  const int sig = signature(p, prm);
  if (sig == SIG_PMA) return rdg_sig<R, SIG_PMA>(p, src, dst, s, prm);
  if (sig == SIG_STAR) return rdg_sig<R, SIG_STAR>(p, src, dst, s, prm);
  if (sig == SIG_FULL) return rdg_sig<R, SIG_FULL>(p, src, dst, s, prm);
  return cudaErrorNotSupported;
}

}  // namespace

bool rdg2d_supported(const Plan& p) {
  if (p.ndim == 3) return rdg3d_supported(p);
  if (p.ndim != 2) return false;
  RdgParams prm;
  return signature(p, prm) >= 0;
}

cudaError_t launch_rdg2d(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  if (p.ndim == 3) return launch_rdg3d(p, src, dst, s);
  switch (p.R) {
    case 1: return rdg_r<1>(p, src, dst, s);
    case 2: return rdg_r<2>(p, src, dst, s);
    case 3: return rdg_r<3>(p, src, dst, s);
    case 4: return rdg_r<4>(p, src, dst, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace lora
