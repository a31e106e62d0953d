// K1 — LoRAStencil 2D on FP64 tensor cores (§III-B RDG, §III-C PMA, §III-D BVS).
//
// Per warp: an 8-row x 64-column output tile P (eight 8x8 accumulator fragments).  For every
// rank-1 term u_k v_k^T of the plan (eq. 9: P = sum_k U_k X V_k):
//   Stage 1 (vertical gather, eq. 10):  T = U_k X.  U_k is the 8 x K1 banded Toeplitz matrix
//     U[g][k] = u[k - g] (K1 = ceil4(8 + 2h_k)), held as K1/4 A-fragment registers per lane;
//     X is read from shared memory as B fragments (lane (g,t) reads X[4kk+t][8nb+g]).  T is
//     8 x 72 (nine 8x8 C fragments) and stays in registers.
//   Stage 2 (horizontal gather, eq. 11) with Butterfly Vector Swapping (eq. 17): the C
//     fragment of T block nb is reused AS an A fragment without any shuffle — register R0
//     holds the even columns 2t, R1 the odd columns 2t+1 — and the rows of V are permuted
//     the same way: B'[t][n] = V[8j + 2t + i][n] = v[8j + 2t + i - n]  (i = 0 for R0, 1 for R1).
//     Output block ob needs T blocks ob and ob+1: 4 DMMAs (P:219 counts 4 for the 7x7 case).
//   Star arms (u or v a unit vector) are a single banded stage; the scalar C_{h+1}
//   and any single-weight term are a DFMA on the staged tile.
// On sm_100a every mma.sync.m8n8k4.f64 is one DMMA.8x8x4 (SASS); there is no tcgen05 f64 kind.
//
// Tile staging: the (64+2R+4) x 72 input tile (padded coordinates, zero fill outside the
// array so that 0 * pad never makes NaN) goes to shared memory with a row pitch of 76 doubles
// (== 12 mod 16), which makes both the B-fragment (4 rows x 8 cols) and the A-fragment
// (8 rows x 4 cols) LDS.64 patterns bank-conflict free.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "kernels.hpp"
#include "pipe.cuh"
#include "tc_terms.cuh"

namespace lora {
namespace {

using namespace tc;

// Persistent CTAs walk the 64x64 output tiles; tile i+1 is staged (TMA + mbarrier, or LDGSTS when
// TMA's 16-byte pitch rule fails) while tile i is computed.
template <int R, bool TMA, bool NOBVS>
__global__ void __launch_bounds__(256, 2) tc2d_kernel(const double* __restrict__ in, double* __restrict__ out,
                                                      int64_t N0, int64_t N1, int ntx, int ntiles,
                                                      const __grid_constant__ CUtensorMap tmap,
                                                      const __grid_constant__ TcParams prm) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  constexpr int SH = tc_rows<R>();
  constexpr int BUF = ((SH * TC_PITCH * 8 + 127) / 128) * 128 / 8;  // doubles per buffer
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem_raw);
  double* buf0 = reinterpret_cast<double*>(smem_raw + 128);
  const int64_t P1 = N1 + 2 * R, P0 = N0 + 2 * R;
  const int tid = threadIdx.x;
  if (TMA && tid == 0) {
    prefetch_tmap(&tmap);
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_barrier_init();
  }
  __syncthreads();
  auto issue = [&](int tile, int b) {
    const int64_t y0 = int64_t(tile / ntx) * TC_BM, x0 = int64_t(tile % ntx) * TC_BN;
    double* dst = buf0 + b * BUF;
    if constexpr (TMA) {
      if (tid == 0) {
        mbar_arrive_expect_tx(&bar[b], SH * TC_PITCH * 8);
        tma_load_2d(dst, &tmap, (int)x0, (int)y0, &bar[b]);
      }
    } else {
      box_fill_cpasync(dst, in, P0, P1, y0, x0, SH, TC_PITCH);
      cp_async_commit();
    }
  };
  const int lane = tid & 31, w = tid >> 5;
  const int g = lane >> 2, t = lane & 3;
  int it = 0;
  int tile = blockIdx.x;
  if (tile < ntiles) issue(tile, 0);
  for (; tile < ntiles; tile += gridDim.x, ++it) {
    const int b = it & 1;
    const int next = tile + gridDim.x;
    if (next < ntiles) issue(next, b ^ 1);
    if constexpr (TMA) {
      mbar_wait(&bar[b], (it >> 1) & 1);
    } else {
      if (next < ntiles) cp_async_wait<1>(); else cp_async_wait<0>();
      __syncthreads();
    }
    const double* X = buf0 + b * BUF;
    double P[8][2];
    tc_tile<R, NOBVS>(X, w, g, t, prm, P);
    const int64_t y0 = int64_t(tile / ntx) * TC_BM, x0 = int64_t(tile % ntx) * TC_BN;
    const int64_t gy = y0 + 8 * w + g;
    if (gy < N0) {
      double* orow = out + (gy + R) * P1 + R;
#pragma unroll
      for (int ob = 0; ob < 8; ++ob) {
        const int64_t gx = x0 + 8 * ob + 2 * t;
        if (gx < N1) orow[gx] = P[ob][0];
        if (gx + 1 < N1) orow[gx + 1] = P[ob][1];
      }
    }
    __syncthreads();  // buffer b is free for the issue of iteration it+1
  }
}

TcParams make_params(const Plan& p) {
  TcParams prm{};
  const int R = p.R, n = 2 * R + 1;
  prm.nterms = 0;
  for (const Term& t : p.terms) {
    TcTerm& d = prm.t[prm.nterms++];
    d.r = t.r < 1 ? 1 : t.r;
    for (int i = 0; i < n; ++i) { d.u[i] = t.u[i]; d.v[i] = t.v[i]; }
    d.ic = R; d.jc = R;
    if (t.kind == kChain) d.kind = 0;
    else if (t.kind == kArm) {
      bool u_unit = true;  // u == e_R  -> horizontal arm
      for (int i = 0; i < n; ++i) if (t.u[i] != (i == R ? 1.0 : 0.0)) u_unit = false;
      d.kind = u_unit ? 1 : 2;
    } else {
      d.kind = 3;
      for (int i = 0; i < n; ++i) if (t.u[i] != 0.0) d.ic = i;
      for (int j = 0; j < n; ++j) if (t.v[j] != 0.0) d.jc = j;
    }
  }
  return prm;
}

template <int R, bool TMA, bool NOBVS>
cudaError_t tc_launch(const Plan& p, const double* src, double* dst, cudaStream_t s, const CUtensorMap& map) {
  constexpr int SH = tc_rows<R>();
  constexpr size_t BUF = ((SH * TC_PITCH * 8 + 127) / 128) * 128;
  const size_t smem = 128 + 2 * BUF;
  const int ntx = (int)((p.N[1] + TC_BN - 1) / TC_BN), nty = (int)((p.N[0] + TC_BM - 1) / TC_BM);
  const int64_t ntiles = int64_t(ntx) * nty;
  int max_grid = 0;
  {
    cudaError_t e = kernel_setup((const void*)tc2d_kernel<R, TMA, NOBVS>, 256, smem, &max_grid);
    if (e != cudaSuccess) return e;
  }
  const int grid = (int)std::min<int64_t>(max_grid, ntiles);
  const TcParams prm = make_params(p);
  tc2d_kernel<R, TMA, NOBVS><<<grid, 256, smem, s>>>(src, dst, p.N[0], p.N[1], ntx, (int)ntiles, map, prm);
  return cudaGetLastError();
}

template <int R>
cudaError_t tc_r(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  CUtensorMap map;
  const int64_t padded[2] = {p.P[0], p.P[1]};
  const int box[2] = {tc_rows<R>(), TC_PITCH};
  const bool tma = !p.force_no_tma && encode_tmap(&map, src, 2, padded, box);
  if (!tma) std::memset(&map, 0, sizeof(map));
  if (p.tc_no_bvs)  // Fig. 9 ablation only (LORA_TC_NO_BVS=1): separate instantiation, shuffles in stage 2
    return tma ? tc_launch<R, true, true>(p, src, dst, s, map) : tc_launch<R, false, true>(p, src, dst, s, map);
  return tma ? tc_launch<R, true, false>(p, src, dst, s, map) : tc_launch<R, false, false>(p, src, dst, s, map);
}

}  // namespace

bool tc2d_supported(const Plan& p) {
  if (p.ndim == 3) return tc3d_supported(p);
  return p.ndim == 2 && (int)p.terms.size() <= TC_MAXT;
}

namespace {
// Exact k-step values on the band of interior points within (k-1)R of the Dirichlet halo, where the
// composed kernel is not equal to k steps (the intermediate steps would read updated halo cells):
// one thread per band point re-runs the k Jacobi steps on its (2kR+1)^2 window with the halo fixed.
struct WB { double w[kMaxN * kMaxN]; };

template <int R, int K>
__global__ void band_kernel(const double* __restrict__ in, double* __restrict__ out, int64_t N0, int64_t N1,
                            int64_t nband, const __grid_constant__ WB W) {
  constexpr int n = 2 * R + 1, H = K * R, M = 2 * H + 1, B = (K - 1) * R;
  const int64_t id = blockIdx.x * int64_t(blockDim.x) + threadIdx.x;
  if (id >= nband) return;
  const int64_t P0 = N0 + 2 * R, P1 = N1 + 2 * R;
  const int64_t bt = std::min<int64_t>(B, N0), mid = std::max<int64_t>(0, N0 - 2 * B);
  const int64_t bw = std::min<int64_t>(B, N1);
  int64_t y, x;  // interior coordinates of this band point
  const int64_t top = bt * N1;
  if (id < top) { y = id / N1; x = id % N1; }
  else if (id < top + mid * (N1 > 2 * B ? 2 * bw : N1)) {
    const int64_t j = id - top, per = N1 > 2 * B ? 2 * bw : N1;
    y = B + j / per;
    const int64_t c = j % per;
    x = N1 > 2 * B ? (c < bw ? c : N1 - 2 * bw + c) : c;
  } else {
    const int64_t j = id - top - mid * (N1 > 2 * B ? 2 * bw : N1);
    y = std::max<int64_t>(B, N0 - B) + j / N1;
    x = j % N1;
  }
  const int64_t cy = y + R, cx = x + R;  // padded
  double a[M][M], b[M][M];
#pragma unroll
  for (int i = 0; i < M; ++i)
#pragma unroll
    for (int j = 0; j < M; ++j) {
      const int64_t gy = cy - H + i, gx = cx - H + j;
      a[i][j] = (gy >= 0 && gy < P0 && gx >= 0 && gx < P1) ? in[gy * P1 + gx] : 0.0;
    }
#pragma unroll
  for (int s = 1; s <= K; ++s) {
    const int r = (K - s) * R;  // cells within r of the centre are needed after step s
#pragma unroll
    for (int i = H - r; i <= H + r; ++i)
#pragma unroll
      for (int j = H - r; j <= H + r; ++j) {
        const int64_t gy = cy - H + i, gx = cx - H + j;
        const bool halo = gy < R || gy >= P0 - R || gx < R || gx >= P1 - R;
        double v = a[i][j];
        if (!halo) {
          v = 0.0;
#pragma unroll
          for (int p = 0; p < n; ++p)
#pragma unroll
            for (int q = 0; q < n; ++q) v = fma(W.w[p * n + q], a[i + p - R][j + q - R], v);
        }
        b[i][j] = v;
      }
#pragma unroll
    for (int i = H - r; i <= H + r; ++i)
#pragma unroll
      for (int j = H - r; j <= H + r; ++j) a[i][j] = b[i][j];
  }
  out[cy * P1 + cx] = a[H][H];
}

template <int R, int K>
cudaError_t band_launch(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  constexpr int B = (K - 1) * R;
  const int64_t N0 = p.N[0], N1 = p.N[1];
  const int64_t inner = std::max<int64_t>(0, N0 - 2 * B) * std::max<int64_t>(0, N1 - 2 * B);
  const int64_t nband = N0 * N1 - inner;
  if (nband == 0) return cudaSuccess;
  WB w{};
  for (int i = 0; i < (2 * R + 1) * (2 * R + 1); ++i) w.w[i] = p.W[i];
  band_kernel<R, K><<<(unsigned)((nband + 127) / 128), 128, 0, s>>>(src, dst, N0, N1, nband, w);
  return cudaGetLastError();
}

cudaError_t band_dispatch(const Plan& p, const double* src, double* dst, cudaStream_t s, int k) {
  if (p.R == 1 && k == 2) return band_launch<1, 2>(p, src, dst, s);
  if (p.R == 1 && k == 3) return band_launch<1, 3>(p, src, dst, s);
  if (p.R == 1 && k == 4) return band_launch<1, 4>(p, src, dst, s);
  if (p.R == 2 && k == 2) return band_launch<2, 2>(p, src, dst, s);
  return cudaErrorNotSupported;
}
}  // namespace

cudaError_t launch_tc2d(const Plan& p, const double* src, double* dst, cudaStream_t s, int k) {
  if (p.ndim == 3) return k == 1 ? launch_tc3d(p, src, dst, s) : cudaErrorNotSupported;
  if (!tc2d_supported(p)) return cudaErrorInvalidValue;
  if (k > 1) {
    // composed kernel on the view whose halo is kR wide (same memory: N' + 2kR = N + 2R) ...
    if (k != p.fuse_k || p.cR != k * p.R) return cudaErrorInvalidValue;
    const int64_t B = int64_t(k - 1) * p.R;
    if (p.N[0] > 2 * B && p.N[1] > 2 * B) {
      Plan v = p;
      v.R = p.cR; v.W = p.cW; v.terms = p.cterms;
      v.N[0] = p.N[0] - 2 * B; v.N[1] = p.N[1] - 2 * B;
      v.graph_exec = nullptr;
      cudaError_t e = launch_tc2d(v, src, dst, s, 1);
      if (e != cudaSuccess) return e;
    }
    // ... and the exact band next to the Dirichlet halo
    return band_dispatch(p, src, dst, s, k);
  }
  switch (p.R) {
    case 1: return tc_r<1>(p, src, dst, s);
    case 2: return tc_r<2>(p, src, dst, s);
    case 3: return tc_r<3>(p, src, dst, s);
    case 4: return tc_r<4>(p, src, dst, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace lora
