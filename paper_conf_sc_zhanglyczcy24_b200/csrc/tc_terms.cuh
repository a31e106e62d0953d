// Tensor-core RDG building blocks shared by the 2D (kernels_tc.cu) and 3D (kernels_tc3d.cu) kernels:
// the banded U/V fragments of eq. 5-6/10-11 built per lane, the two-stage DMMA chain with Butterfly
// Vector Swapping (eq. 17), single-stage star arms and point-wise DFMA terms.  X is a staged tile
// with row pitch TC_PITCH; a warp owns output rows 8w..8w+7 and 64 columns (8 C fragments P[ob]).
#pragma once
#include <cuda_runtime.h>

#include "plan.hpp"

namespace lora {
namespace tc {

constexpr int TC_MAXT = 16;
struct TcTerm {
  int kind, r, ic, jc;     // kind: 0 chain, 1 horizontal arm, 2 vertical arm, 3 point
  double u[kMaxN], v[kMaxN];
};
struct TcParams {
  int nterms;
  TcTerm t[TC_MAXT];
};

constexpr int TC_BM = 64, TC_BN = 64, TC_PITCH = 76;

// Not `volatile`: the compiler may interleave independent DMMAs (a volatile asm pins program order,
// which turned the per-block stage-2 accumulation into a dependent chain).
__device__ __forceinline__ void dmma(double (&c)[2], double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(c[0]), "+d"(c[1])
               : "d"(a), "d"(b));
}

template <int R>
__host__ __device__ constexpr int tc_rows() { return TC_BM + 2 * R + 4; }

// u/v are centred length 2R+1; a term of radius HR lives in [R-HR, R+HR].
template <int R, int HR, bool NOBVS = false>
__device__ __forceinline__ void chain_term(const double* __restrict__ X, int w, int g, int t, const TcTerm& tm,
                                           double (&P)[8][2]) {
  constexpr int K1 = ((8 + 2 * HR + 3) / 4) * 4, KS = K1 / 4;
  constexpr int o = R - HR;
  double a[KS];
#pragma unroll
  for (int kk = 0; kk < KS; ++kk) {
    const int j = 4 * kk + t - g;
    a[kk] = (j >= 0 && j <= 2 * HR) ? tm.u[o + j] : 0.0;
  }
  double T[9][2];
#pragma unroll
  for (int nb = 0; nb < 9; ++nb) { T[nb][0] = 0.0; T[nb][1] = 0.0; }
  if constexpr (NOBVS) {
    // Ablation "TC RDG without BVS" (Fig. 9): T keeps its natural column order and
    // the stage-2 A fragment A[g][t] = T[g][4h + t] is gathered from the C layout of lane
    // (g, 2h + t/2), register t % 2, with warp shuffles (4 SHFL.32 per fragment).
    const double* xr = X + (8 * w + o + t) * TC_PITCH + g;
#pragma unroll
    for (int kk = 0; kk < KS; ++kk) {
#pragma unroll
      for (int nb = 0; nb < 9; ++nb) dmma(T[nb], a[kk], xr[4 * kk * TC_PITCH + 8 * nb]);
    }
    double af[9][2];
#pragma unroll
    for (int nb = 0; nb < 9; ++nb)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int src = 4 * g + 2 * h + (t >> 1);
        const double v0 = __shfl_sync(0xffffffffu, T[nb][0], src);
        const double v1 = __shfl_sync(0xffffffffu, T[nb][1], src);
        af[nb][h] = (t & 1) ? v1 : v0;
      }
    double vn[2][2];
#pragma unroll
    for (int j = 0; j < 2; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int c = 8 * j + 4 * h + t - g;
        vn[j][h] = (c >= 0 && c <= 2 * R) ? tm.v[c] : 0.0;
      }
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], af[ob][0], vn[0][0]);
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], af[ob][1], vn[0][1]);
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], af[ob + 1][0], vn[1][0]);
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], af[ob + 1][1], vn[1][1]);
    return;
  }
  if constexpr (8 + 2 * HR <= 12) {
    // Column-grouped BVS (HR <= 2): an 8-column output block needs 8 + 2HR <= 12 consecutive T
    // columns, i.e. three groups of 4.  Stage 1 is free to choose which 8 tile columns form a T
    // block (they are just the B-fragment addresses), so T block nb holds group 2nb (tile columns
    // o + 8nb .. +3) in its even accumulator columns (R0) and group 2nb+1 (o + 8nb + 4 .. +7) in
    // its odd ones (R1).  Output block ob then reads groups 2ob, 2ob+1, 2ob+2 = R0, R1 of block ob
    // and R0 of block ob+1: 3 DMMAs instead of 4, still with no shuffle.
    // The odd group's slots are additionally rotated, slot t <-> group column (t + 2) mod 4 (another
    // eq. 17 permutation, undone in V'), so that each half-warp's 16 B-fragment addresses stay distinct
    // mod 16 doubles with the 76-double pitch: bank-conflict free, like the ungrouped layout.
    const int gc = (g & 1) ? 4 + (((g >> 1) + 2) & 3) : (g >> 1);   // tile column of T column n = g
    const double* xr = X + (8 * w + o + t) * TC_PITCH + o + gc;
#pragma unroll
    for (int kk = 0; kk < KS; ++kk) {
#pragma unroll
      for (int nb = 0; nb < 9; ++nb) dmma(T[nb], a[kk], xr[4 * kk * TC_PITCH + 8 * nb]);
    }
    double vg[3];
#pragma unroll
    for (int j = 0; j < 3; ++j) {
      const int slot = (j == 1) ? ((t + 2) & 3) : t;   // group column held in A slot t
      const int c = 4 * j + o + slot - g;              // its tap for output column g
      vg[j] = (c >= 0 && c <= 2 * R) ? tm.v[c] : 0.0;
    }
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], T[ob][0], vg[0]);     // pass-major: consecutive DMMAs
#pragma unroll                                                       // hit different accumulators
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], T[ob][1], vg[1]);
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], T[ob + 1][0], vg[2]);
    return;
  }
  const double* xr = X + (8 * w + o + t) * TC_PITCH + g;
#pragma unroll
  for (int kk = 0; kk < KS; ++kk) {
#pragma unroll
    for (int nb = 0; nb < 9; ++nb) dmma(T[nb], a[kk], xr[4 * kk * TC_PITCH + 8 * nb]);
  }
  double vb[2][2];
#pragma unroll
  for (int j = 0; j < 2; ++j)
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      const int c = 8 * j + 2 * t + i - g;
      vb[j][i] = (c >= 0 && c <= 2 * R) ? tm.v[c] : 0.0;
    }
#pragma unroll
  for (int ob = 0; ob < 8; ++ob) dmma(P[ob], T[ob][0], vb[0][0]);
#pragma unroll
  for (int ob = 0; ob < 8; ++ob) dmma(P[ob], T[ob][1], vb[0][1]);
#pragma unroll
  for (int ob = 0; ob < 8; ++ob) dmma(P[ob], T[ob + 1][0], vb[1][0]);
#pragma unroll
  for (int ob = 0; ob < 8; ++ob) dmma(P[ob], T[ob + 1][1], vb[1][1]);
}

// Horizontal arm (u = e_R): P[g][n] += sum_c X[8w+g+R][8ob+c] v[c-n]; A from smem, B = band of v.
template <int R, int HR>
__device__ __forceinline__ void harm_term(const double* __restrict__ X, int w, int g, int t, const TcTerm& tm,
                                          double (&P)[8][2]) {
  constexpr int K = ((8 + 2 * HR + 3) / 4) * 4, KS = K / 4;
  constexpr int o = R - HR;
  double b[KS];
#pragma unroll
  for (int kk = 0; kk < KS; ++kk) {
    const int j = 4 * kk + t - g;
    b[kk] = (j >= 0 && j <= 2 * HR) ? tm.v[o + j] : 0.0;
  }
  const double* xr = X + (8 * w + g + R) * TC_PITCH + o + t;
#pragma unroll
  for (int kk = 0; kk < KS; ++kk)
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], xr[8 * ob + 4 * kk], b[kk]);
}

// Vertical arm (v = e_R): P[g][n] += sum_k U[g][k] X[8w+o+k][8ob+n+R].
template <int R, int HR>
__device__ __forceinline__ void varm_term(const double* __restrict__ X, int w, int g, int t, const TcTerm& tm,
                                          double (&P)[8][2]) {
  constexpr int K1 = ((8 + 2 * HR + 3) / 4) * 4, KS = K1 / 4;
  constexpr int o = R - HR;
  double a[KS];
#pragma unroll
  for (int kk = 0; kk < KS; ++kk) {
    const int j = 4 * kk + t - g;
    a[kk] = (j >= 0 && j <= 2 * HR) ? tm.u[o + j] : 0.0;
  }
  const double* xr = X + (8 * w + o + t) * TC_PITCH + g + R;
#pragma unroll
  for (int kk = 0; kk < KS; ++kk)
#pragma unroll
    for (int ob = 0; ob < 8; ++ob) dmma(P[ob], a[kk], xr[4 * kk * TC_PITCH + 8 * ob]);
}

template <int R>
__device__ __forceinline__ void point_term(const double* __restrict__ X, int w, int g, int t, const TcTerm& tm,
                                           double (&P)[8][2]) {
  const double wgt = tm.v[tm.jc];
  const double* xr = X + (8 * w + g + tm.ic) * TC_PITCH + 2 * t + tm.jc;
#pragma unroll
  for (int ob = 0; ob < 8; ++ob) {
    P[ob][0] = fma(wgt, xr[8 * ob], P[ob][0]);
    P[ob][1] = fma(wgt, xr[8 * ob + 1], P[ob][1]);
  }
}


// Accumulates terms k0 .. k1-1 of prm into P (eq. 9: the sum of the rank-1 chains).
template <int R, bool NOBVS = false>
__device__ __forceinline__ void apply_terms(const double* __restrict__ X, int w, int g, int t, const TcParams& prm,
                                            int k0, int k1, double (&P)[8][2]) {
  for (int k = k0; k < k1; ++k) {
    const TcTerm& tm = prm.t[k];
    switch (tm.kind) {
      case 0:
        if (tm.r == 1) chain_term<R, 1, NOBVS>(X, w, g, t, tm, P);
        else if constexpr (R >= 2) {
          if (tm.r == 2) chain_term<R, (R >= 2 ? 2 : 1), NOBVS>(X, w, g, t, tm, P);
          else if constexpr (R >= 3) {
            if (tm.r == 3) chain_term<R, (R >= 3 ? 3 : 1), NOBVS>(X, w, g, t, tm, P);
            else if constexpr (R >= 4) chain_term<R, 4, NOBVS>(X, w, g, t, tm, P);
          }
        }
        break;
      case 1:
        if (tm.r <= 1) harm_term<R, 1>(X, w, g, t, tm, P);
        else if constexpr (R >= 2) {
          if (tm.r == 2) harm_term<R, (R >= 2 ? 2 : 1)>(X, w, g, t, tm, P);
          else if constexpr (R >= 3) {
            if (tm.r == 3) harm_term<R, (R >= 3 ? 3 : 1)>(X, w, g, t, tm, P);
            else if constexpr (R >= 4) harm_term<R, 4>(X, w, g, t, tm, P);
          }
        }
        break;
      case 2:
        if (tm.r <= 1) varm_term<R, 1>(X, w, g, t, tm, P);
        else if constexpr (R >= 2) {
          if (tm.r == 2) varm_term<R, (R >= 2 ? 2 : 1)>(X, w, g, t, tm, P);
          else if constexpr (R >= 3) {
            if (tm.r == 3) varm_term<R, (R >= 3 ? 3 : 1)>(X, w, g, t, tm, P);
            else if constexpr (R >= 4) varm_term<R, 4>(X, w, g, t, tm, P);
          }
        }
        break;
      default:
        point_term<R>(X, w, g, t, tm, P);
    }
  }
}


template <int R, bool NOBVS = false>
__device__ __forceinline__ void tc_tile(const double* __restrict__ X, int w, int g, int t, const TcParams& prm,
                                        double (&P)[8][2]) {
#pragma unroll
  for (int ob = 0; ob < 8; ++ob) { P[ob][0] = 0.0; P[ob][1] = 0.0; }
  apply_terms<R, NOBVS>(X, w, g, t, prm, 0, prm.nterms, P);
}

}  // namespace tc
}  // namespace lora
