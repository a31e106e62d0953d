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
#include "p2p.cuh"
#include "pipe.cuh"

namespace lora {
namespace {

#ifndef RDG_RC_ROWS
#define RDG_RC_ROWS 128   // experiments: chunk length
#endif
constexpr int RDG_RC = RDG_RC_ROWS;
#ifndef RDG_UNIFORM_WL
#define RDG_UNIFORM_WL 1
#endif
#ifndef RDG_LOOP_UNROLL
#define RDG_LOOP_UNROLL 2   // unroll factor of the fused row loop (Box-2D49P k=2: 1: 337, 2: 347, 3: 251, 4: 283, 7: 326 GS/s)
#endif
constexpr int kRowUnroll = RDG_LOOP_UNROLL;   // (#pragma arguments are not macro-expanded)   // output rows per work item (chunk)
#ifndef RDG_WARPS_PER_CTA
#define RDG_WARPS_PER_CTA 4   // (Box-2D49P k=2: 2 warps 351, 4 warps 350, 8 warps 270 GS/s; Box-2D9P k=3: 654 / 692)
#endif
constexpr int RDG_WARPS = RDG_WARPS_PER_CTA;   // warps per CTA (independent streams)
#ifndef RDG_S1LOAD
#define RDG_S1LOAD 0   // 1: load stage 1's row before stages K .. 2 run (r02zzb: Box-2D49P 450 -> 447)
#endif
#ifndef RDG_S1FIRST
#define RDG_S1FIRST 0   // 1: stage 1 before stages K .. 2 in each row iteration (r02zr: Box-2D49P 448 -> 426)
#endif
#ifndef RDG_PF_HALVES
#define RDG_PF_HALVES 2   // 64-column halves of the next row prefetched (RDG_PF, loop form)
#endif
#ifndef RDG_NS_STAGES
#define RDG_NS_STAGES 2   // r02zzg/h: Box-2D49P 449 -> 454, Box-2D9P 716 -> 748, Star-2D13P 476 -> 499 GS/s vs 3 stages
#endif
constexpr int RDG_NS = RDG_NS_STAGES;   // TMA ring stages per warp

enum { SIG_PMA = 0, SIG_STAR = 1, SIG_FULL = 2, SIG_DIRECT = 3, SIG_ROWS = 4 };   // DIRECT: W itself in u[][] (K11)

struct RdgParams {
  int K;                     // number of (u, v) chain terms used by the signature
  double u[kMaxN][kMaxN];    // centred, length 2R+1
  double v[kMaxN][kMaxN];
  double c;                  // PMA scalar C_{h+1}
};

// NH = 64-column halves per warp: lane p owns columns 64h + 2p, 64h + 2p + 1 (h < NH), so each
// staged row is read with the conflict-free 16-byte lane pattern of one half at a time; NH = 2
// halves the band-edge recomputation of the fused kernels and gives every warp two independent
// row pipelines (ILP for the 8-cycle DFMA latency).
template <int R, int NH = 1>
struct Geom {
  static constexpr int n = 2 * R + 1;
  static constexpr int m = n >= 6 ? 1 : 2;
  static constexpr int SROWS = n * m;                                  // rows per stage (multiple of n)
  static constexpr int BW = 64 * NH + 2 * R;                           // staged columns
  static constexpr int BUFD = ((BW + 15) / 16) * 16;                   // doubles per intermediate row buffer
  static constexpr int STAGE = ((SROWS * BW * 8 + 127) / 128) * 128;   // bytes per stage
  static constexpr int SI = (RDG_RC + 2 * R + SROWS - 1) / SROWS;      // stages per work item
  static constexpr int WARP_BYTES = RDG_NS * STAGE;
  static constexpr int SMEM = 128 + RDG_WARPS * WARP_BYTES;
};

__host__ __device__ constexpr int pmod(int a, int n) { return ((a % n) + n) % n; }

// One input row r (r mod n == I mod n) of the stream: T for every term, scattered into the ring.
// The lane's 2R + 2 inputs of one row (columns 2p - R .. 2p + R + 1 of the band): R + 1 LDS.128.
template <int R>
__device__ __forceinline__ void load_x(const double* __restrict__ xs, int p, double (&x)[2 * R + 2]) {
#pragma unroll
  for (int q = 0; q <= R; ++q) {
    const double2 t = *reinterpret_cast<const double2*>(xs + 2 * p + 2 * q);
    x[2 * q] = t.x;
    x[2 * q + 1] = t.y;
  }
}

template <int R, int SIG, int I>
__device__ __forceinline__ void row_compute(const double (&x)[2 * R + 2], double (&acc)[2 * R + 1][2], const RdgParams& P);

template <int R, int SIG, int I>
__device__ __forceinline__ void row_body(const double* __restrict__ xs, int p, double (&acc)[2 * R + 1][2],
                                         const RdgParams& P) {
  double x[2 * R + 2];
  load_x<R>(xs, p, x);
  row_compute<R, SIG, I>(x, acc, P);
}

template <int R, int SIG, int I>
__device__ __forceinline__ void row_compute(const double (&x)[2 * R + 2], double (&acc)[2 * R + 1][2], const RdgParams& P) {
  constexpr int n = 2 * R + 1;
  if constexpr (SIG == SIG_PMA) {
    // PMA pyramid (eq. 15): term k has radius R-k; the last one is the scalar C_{h+1}.  The PMA
    // factors of a reflection-symmetric W are exactly palindromic (the planner takes the
    // PMA route only for exactly symmetric remainders), so the horizontal gather pairs the taps:
    // T = v_0 x_0 + sum_b v_b (x_{-b} + x_{+b}); the pair sums are shared by all terms.
    double sp0[R + 1], sp1[R + 1];
#pragma unroll
    for (int b = 1; b <= R; ++b) {
      sp0[b] = x[R - b] + x[R + b];
      sp1[b] = x[R - b + 1] + x[R + b + 1];
    }
#pragma unroll
    for (int k = 0; k < R; ++k) {
      const int H = R - k;
      double t0 = x[R], t1 = x[R + 1];   // v_k[R] == 1 (signature() rescales the PMA factors)
#pragma unroll
      for (int b = 1; b <= H; ++b) {
        t0 = fma(P.v[k][R + b], sp0[b], t0);
        t1 = fma(P.v[k][R + b], sp1[b], t1);
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
  } else if constexpr (SIG == SIG_ROWS) {
    // row-pair rank-1 split of a doubly reflection-symmetric W (Plan::rdg_rows): term a has
    // u_a = c_a (e_{R+a} + e_{R-a}) and v_a = W[R+a,:] / c_a with c_a = W[R+a,R] (unit centre tap),
    // so the horizontal gather is t_a = x_0 + sum_b v_a[b] (x_{-b} + x_{+b}) on the shared pair
    // sums (R DFMA, no DMUL) and the vertical gather is one DFMA c_a t_a into each of the (at most
    // two) output rows R+a, R-a away; the first term of an output row is the product c_R t_R.
    double sp0[R + 1], sp1[R + 1];
#pragma unroll
    for (int b = 1; b <= R; ++b) {
      sp0[b] = x[R - b] + x[R + b];
      sp1[b] = x[R - b + 1] + x[R + b + 1];
    }
#pragma unroll
    for (int a = 0; a <= R; ++a) {
      double t0 = x[R], t1 = x[R + 1];   // v_a[R] == 1
#pragma unroll
      for (int b = 1; b <= R; ++b) {
        t0 = fma(P.v[a][R + b], sp0[b], t0);
        t1 = fma(P.v[a][R + b], sp1[b], t1);
      }
      const double ca = P.u[a][0];
      const int s = pmod(I - R - a, n);
      acc[s][0] = fma(ca, t0, acc[s][0]);
      acc[s][1] = fma(ca, t1, acc[s][1]);
      if (a == R) {   // slot I mod n was emptied after the previous row: this is its first term
        acc[pmod(I, n)][0] = ca * t0;
        acc[pmod(I, n)][1] = ca * t1;
      } else if (a > 0) {
        const int s2 = pmod(I - R + a, n);
        acc[s2][0] = fma(ca, t0, acc[s2][0]);
        acc[s2][1] = fma(ca, t1, acc[s2][1]);
      }
    }
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
  } else if constexpr (SIG == SIG_DIRECT) {
    // the in-tree comparison (north star (c)): the unfactored (2R+1)^2 sum on the same stream —
    // input row r adds sum_b W[R+a][R+b] x[r][x+b] to output row r - R - a.
#pragma unroll
    for (int a = -R; a <= R; ++a) {
      const int s = pmod(I - R - a, n);
#pragma unroll
      for (int b = -R; b <= R; ++b) {
        acc[s][0] = fma(P.u[R + a][R + b], x[R + b], acc[s][0]);
        acc[s][1] = fma(P.u[R + a][R + b], x[R + b + 1], acc[s][1]);
      }
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

// Shift-register form of the same row update, for the runtime row loop of the fused kernels
// (RDG_LOOP): after input row r, p[j] holds output row r - R + j, so p'[j] = p[j+1] + (the
// contributions of row r with vertical offset a = R - j) and p'[2R] = the first contribution of
// row r + R; the completed row r - R is p[0].  The "shift" is only the choice of destination
// register, so the row needs no static ring index and the loop need not be unrolled by 2R + 1
// (the unrolled ring form's hot code overflows the instruction cache: ncu no_instruction stalls).
// Per output row the contributions arrive in the same order as in the ring form (first one from
// 0.0 or assigned exactly as there), so both forms give bitwise identical rows.
template <int R, int SIG>
__device__ __forceinline__ void row_shift(const double (&x)[2 * R + 2], double (&p)[2 * R + 1][2], const RdgParams& P) {
  double sp0[R + 1], sp1[R + 1];
  if constexpr (SIG == SIG_ROWS || SIG == SIG_PMA) {
#pragma unroll
    for (int b = 1; b <= R; ++b) {
      sp0[b] = x[R - b] + x[R + b];
      sp1[b] = x[R - b + 1] + x[R + b + 1];
    }
  }
  if constexpr (SIG == SIG_ROWS) {
    double t[R + 1][2];
#pragma unroll
    for (int a = 0; a <= R; ++a) {
      double t0 = x[R], t1 = x[R + 1];   // unit centre tap (row_compute SIG_ROWS)
#pragma unroll
      for (int b = 1; b <= R; ++b) {
        t0 = fma(P.v[a][R + b], sp0[b], t0);
        t1 = fma(P.v[a][R + b], sp1[b], t1);
      }
      t[a][0] = t0;
      t[a][1] = t1;
    }
#pragma unroll
    for (int j = 0; j < 2 * R; ++j) {
      const int a = j < R ? R - j : j - R;
      p[j][0] = fma(P.u[a][0], t[a][0], p[j + 1][0]);
      p[j][1] = fma(P.u[a][0], t[a][1], p[j + 1][1]);
    }
    p[2 * R][0] = P.u[R][0] * t[R][0];
    p[2 * R][1] = P.u[R][0] * t[R][1];
  } else if constexpr (SIG == SIG_PMA) {
    double t[R][2];
#pragma unroll
    for (int k = 0; k < R; ++k) {
      const int H = R - k;
      double t0 = x[R], t1 = x[R + 1];   // v_k[R] == 1 (signature() rescales the PMA factors)
#pragma unroll
      for (int b = 1; b <= H; ++b) {
        t0 = fma(P.v[k][R + b], sp0[b], t0);
        t1 = fma(P.v[k][R + b], sp1[b], t1);
      }
      t[k][0] = t0;
      t[k][1] = t1;
    }
#pragma unroll
    for (int j = 0; j <= 2 * R; ++j) {
      const int a = R - j;
      double q0 = j < 2 * R ? p[j + 1][0] : 0.0, q1 = j < 2 * R ? p[j + 1][1] : 0.0;
#pragma unroll
      for (int k = 0; k < R; ++k) {
        if (a <= R - k && -a <= R - k) {
          q0 = fma(P.u[k][R + a], t[k][0], q0);
          q1 = fma(P.u[k][R + a], t[k][1], q1);
        }
      }
      if (a == 0) {
        q0 = fma(P.c, x[R], q0);
        q1 = fma(P.c, x[R + 1], q1);
      }
      p[j][0] = q0;
      p[j][1] = q1;
    }
  } else if constexpr (SIG == SIG_STAR) {
    double t0 = 0.0, t1 = 0.0;
#pragma unroll
    for (int b = -R; b <= R; ++b) {
      t0 = fma(P.v[0][R + b], x[R + b], t0);
      t1 = fma(P.v[0][R + b], x[R + b + 1], t1);
    }
#pragma unroll
    for (int j = 0; j <= 2 * R; ++j) {
      const int a = R - j;
      double q0 = j < 2 * R ? p[j + 1][0] : 0.0, q1 = j < 2 * R ? p[j + 1][1] : 0.0;
      if (a == 0) {
        q0 += t0;
        q1 += t1;
      }
      p[j][0] = fma(P.u[1][R + a], x[R], q0);
      p[j][1] = fma(P.u[1][R + a], x[R + 1], q1);
    }
  } else {
    static_assert(SIG == SIG_ROWS || SIG == SIG_PMA || SIG == SIG_STAR, "row_shift: fused signatures only");
  }
}

// ---------------------------------------------------------------------------------------------
// Exact temporal fusion (§IV-A; reading Q5): K time steps per HBM
// round trip.  Stage 1 consumes the staged input rows; every completed step-s row is written to a
// per-warp shared row buffer (double-buffered by row parity) that stage s+1 consumes exactly like
// an input row, so the K steps form a software pipeline down the stream (stage s lags by s*R
// rows).  Each intermediate row re-imposes the fixed Dirichlet halo (rows/columns of the halo take
// the input values, P:21 Jacobi semantics), so the result equals K separate steps.  The lane
// columns lose R valid columns per fused step at each band edge: bands overlap, stride
// S = 64 - 2R(K-1) (minus 2 when R(K-1) is odd, so that the staged tile starts on an even column:
// TMA faults on a box whose innermost start is not 16-byte aligned, tools/ubench/tma_probe.cu).
// Per-stage precomputed bookkeeping (32-bit, relative to the stage's first input row) so that the
// unrolled row code carries no 64-bit index arithmetic.
template <int K>
struct StageCtx {
  int lo, hi;               // final rows: stage-local rows I with lo <= I < hi are stored
  int64_t ooff;             // element offset of (final row for I = 0, lane column c0)
  int rem_lo, rem_hi;       // device-initiated exchange: rows I < rem_lo also go to the lower
                            // neighbour's halo, rows I >= rem_hi to the upper one's
  int hlo[K], hhi[K];       // intermediate stage S: row I is halo if I < hlo or I >= hhi
  int rlo[K], rhi[K];       //                     row I is inside the array if rlo <= I < rhi
  int64_t ioff[K];          //                     element offset of (row for I = 0, column 0) in `in`
};

template <int NH>
struct LaneCtx {
  int c0;                   // padded column of the lane's first column (may be < 0); half h adds 64h
  bool inside[NH][2], colhalo[NH][2], valid[NH][2], vec[NH];
  bool edge;                // some column of the lane is a column halo or outside the array
  bool edge_any;            // ... of some lane of the warp (warp-uniform: a uniform branch)
};

// Stores the lane's column pairs of one row: a 16-byte store where the pair is valid and aligned,
// else predicated 8-byte stores (array edges, band-overlap lanes of fused bands store nothing).
// ODD (odd R): lane pairs start on odd columns, never 16-byte aligned (no vector-store code).
template <int NH, bool ODD = false>
__device__ __forceinline__ void store_pairs(double* o, const double (&v)[NH][2], const LaneCtx<NH>& lc) {
#pragma unroll
  for (int h = 0; h < NH; ++h) {
    if constexpr (ODD) {
      if (lc.valid[h][0]) o[64 * h] = v[h][0];
      if (lc.valid[h][1]) o[64 * h + 1] = v[h][1];
      continue;
    }
    const bool p0 = !lc.vec[h] && lc.valid[h][0], p1 = !lc.vec[h] && lc.valid[h][1];
    if (lc.vec[h]) *reinterpret_cast<double2*>(o + 64 * h) = make_double2(v[h][0], v[h][1]);
    if (p0) o[64 * h] = v[h][0];
    if (p1) o[64 * h + 1] = v[h][1];
  }
}

// One iteration of the fused pipeline (input row I of the staged tile), stages S = K down to 1.
// Stage S >= 2 consumes the row stage S-1 produced in the PREVIOUS iteration (row buffer of the
// other parity), so within an iteration every stage reads before any stage writes and the stages
// are independent instruction streams (ILP for the 8-cycle DFMA latency); one __syncwarp per
// iteration orders the buffer writes against the next iteration's reads.  Stage S therefore lags
// stage 1 by (S-1)(R+1) rows (StageCtx row offsets include the extra (S-1) rows).
// FULL: every row of the stage is interior for every intermediate step, every final row is stored
// and every lane stores a 16-byte pair (decided per stage, warp-uniform): no per-row checks.
// PRE: stage S's input row is already in xq (the prefetched stage-1 row); stages S down to SMIN run.
// LOOP: runtime row loop (row index Ir, shift-register row update row_shift) instead of the ring
// form unrolled over the 2R + 1 ring positions (template row index I, ring position I0).
template <int R, int SIG, int K, int NH, bool FULL, int I0, int I_, int S, bool PRE = false, int SMIN = 1, bool LOOP = false,
          bool REM = true>
__device__ __forceinline__ void fused_iter(const double* __restrict__ st_row, int p,
                                           double (&acc)[K][NH][2 * R + 1][2], const RdgParams& P,
                                           double* __restrict__ bufs, int par, const double* __restrict__ in,
                                           double* __restrict__ out, int64_t P1, const StageCtx<K>& sc,
                                           const LaneCtx<NH>& lc, const P2PArgs& dp,
                                           const double (&xq)[NH][2 * R + 2], int Ir = 0,
                                           double* __restrict__ orow = nullptr) {
  static_assert(!PRE || SMIN == S, "a preloaded stage runs alone");
  constexpr int n = 2 * R + 1;
  constexpr int BUFD = Geom<R, NH>::BUFD;
  const int I = LOOP ? Ir : I_;
  constexpr int Is = pmod(I0 - (S - 1) * (R + 1), n);   // ring index of stage S's input row (any per-stage constant)
  const double* src = S == 1 ? st_row : bufs + (2 * (S - 2) + (par ^ 1)) * BUFD;
  double v[NH][2];
  if constexpr (LOOP) {
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      if (PRE && h < RDG_PF_HALVES) {   // (RDG_PF_HALVES: only the first halves are prefetched)
        row_shift<R, SIG>(xq[h], acc[S - 1][h], P);
      } else {
        double x[2 * R + 2];
        load_x<R>(src + 64 * h, p, x);
        row_shift<R, SIG>(x, acc[S - 1][h], P);
      }
      v[h][0] = acc[S - 1][h][0][0];
      v[h][1] = acc[S - 1][h][0][1];
    }
  } else {
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      if constexpr (PRE) row_compute<R, SIG, Is>(xq[h], acc[S - 1][h], P);
      else row_body<R, SIG, Is>(src + 64 * h, p, acc[S - 1][h], P);
    }
    constexpr int cs = (Is + 1) % n;                // slot of the row this stage just completed
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      v[h][0] = acc[S - 1][h][cs][0];
      v[h][1] = acc[S - 1][h][cs][1];
      acc[S - 1][h][cs][0] = 0.0;
      acc[S - 1][h][cs][1] = 0.0;
    }
  }
  if constexpr (S < K) {
    // re-impose the fixed Dirichlet halo on the intermediate row (exact temporal blocking)
    if (FULL) {
    } else if (I < sc.hlo[S - 1] || I >= sc.hhi[S - 1]) {
      const bool row_in = I >= sc.rlo[S - 1] && I < sc.rhi[S - 1];
      const double* ir = in + sc.ioff[S - 1] + int64_t(I) * P1 + lc.c0;
#pragma unroll
      for (int h = 0; h < NH; ++h)
#pragma unroll
        for (int j = 0; j < 2; ++j) v[h][j] = (row_in && lc.inside[h][j]) ? ir[64 * h + j] : 0.0;
    } else if (lc.edge_any) {   // per-lane tests inside (lanes without edge columns keep v)
      const double* ir = in + sc.ioff[S - 1] + int64_t(I) * P1 + lc.c0;
#pragma unroll
      for (int h = 0; h < NH; ++h)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          if (lc.colhalo[h][j]) v[h][j] = ir[64 * h + j];
          if (!lc.inside[h][j]) v[h][j] = 0.0;
        }
    }
    double* b = bufs + (2 * (S - 1) + par) * BUFD;   // [stage][parity] row buffers
#pragma unroll
    for (int h = 0; h < NH; ++h) {   // 8-byte stores: R + 2p is odd for odd R
      b[R + 64 * h + 2 * p] = v[h][0];
      b[R + 64 * h + 2 * p + 1] = v[h][1];
    }
  } else if constexpr (FULL) {
    double* o = out + sc.ooff + int64_t(I) * P1;
#pragma unroll
    for (int h = 0; h < NH; ++h) {   // band-overlap lanes of a fused band store nothing
      if constexpr (R & 1) {   // odd R: lane pairs start on odd columns (8-byte stores)
        if (lc.valid[h][0]) { o[64 * h] = v[h][0]; o[64 * h + 1] = v[h][1]; }
      } else {
        if (lc.vec[h]) *reinterpret_cast<double2*>(o + 64 * h) = make_double2(v[h][0], v[h][1]);
      }
    }
  } else {
    if (I >= sc.lo && I < sc.hi) {
      if constexpr (K > 1) {
        // LOOP: orow is this row's output pointer, advanced by the loop (no 64-bit index per row)
        double* o = LOOP ? orow : out + (sc.ooff + int64_t(I) * P1);
        store_pairs<NH, (R & 1) != 0>(o, v, lc);
        if (REM && (I < sc.rem_lo || I >= sc.rem_hi)) {   // warp-uniform, rare (REM: the stage has such rows)
          const int64_t e = sc.ooff + int64_t(I) * P1;
          if (I < sc.rem_lo) store_pairs<NH>(dp.dst_lo + (e + dp.off_lo), v, lc);
          if (I >= sc.rem_hi) store_pairs<NH>(dp.dst_hi + (e + dp.off_hi), v, lc);
        }
      } else {
        const int64_t e = sc.ooff + int64_t(I) * P1;
        // the row goes to this slab and, for the first / last R interior rows of a slab with a
        // neighbour there, into that neighbour's halo as well (peer memory, csrc/dist_p2p.cu;
        // the device-initiated exchange runs unfused).  This form measured faster for K = 1
        // than store_pairs + two uniform branches (342 vs 321 GS/s, Box-2D49P).
        const int nd = 1 + (I < sc.rem_lo ? 1 : 0) + (I >= sc.rem_hi ? 1 : 0);
        for (int d = 0; d < nd; ++d) {
          double* o = d == 0 ? out + e : (I < sc.rem_lo && d == 1 ? dp.dst_lo + (e + dp.off_lo) : dp.dst_hi + (e + dp.off_hi));
#pragma unroll
          for (int h = 0; h < NH; ++h) {
            if (lc.vec[h]) {
              *reinterpret_cast<double2*>(o + 64 * h) = make_double2(v[h][0], v[h][1]);
            } else {
              if (lc.valid[h][0]) o[64 * h] = v[h][0];
              if (lc.valid[h][1]) o[64 * h + 1] = v[h][1];
            }
          }
        }
      }
    }
  }
  if constexpr (S > SMIN)
    fused_iter<R, SIG, K, NH, FULL, I0, I_, S - 1, false, SMIN, LOOP, REM>(st_row, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, xq, Ir,
                                                                      orow);
}

#ifndef RDG_PF
#define RDG_PF 0   // fused kernels of radius >= RDG_PF: prefetch the next staged input row (0: never)
#endif
#ifndef RDG_PF2
#define RDG_PF2 2  // K = 2: also load stage 2's input row before stage 1's work — 1: always, 2: star
#endif             // arms only (Star-2D13P 435 -> 451 GS/s; Box-2D49P 322 -> 290: register spills), 0: never
// Default off since the weights moved to uniform registers (r02v/r02w, same box): Box-2D49P k = 2
// 428 -> 449 GS/s without the prefetch (202 instead of 230 registers).
// Fused kernels with RDG_PF: stage 1 runs first on the row prefetched in the previous iteration,
// then the next staged row (same TMA stage) is loaded into xq, then stages K .. 2 run — their FP64
// work covers the shared-load latency of the next stage-1 row (which the per-row __syncwarp keeps
// the compiler from hoisting).  The stages of an iteration are independent, so the order is free.
// Measured (same box, short runs): Box-2D49P k = 2 312 -> 322 GS/s, Star-2D13P k = 2 unchanged;
// radius 1 (Box-2D9P k = 3) not better, so radius >= 3 only.
template <int R, int SIG, int K, int NH, bool FULL, int I>
__device__ __forceinline__ void fused_rows(const double* __restrict__ st, int p, double (&acc)[K][NH][2 * R + 1][2],
                                           const RdgParams& P, double* __restrict__ bufs,
                                           const double* __restrict__ in, double* __restrict__ out, int64_t P1,
                                           const StageCtx<K>& sc, const LaneCtx<NH>& lc, int par0, const P2PArgs& dp,
                                           double (&xq)[NH][2 * R + 2]) {
  constexpr int n = 2 * R + 1;
  constexpr int BW = Geom<R, NH>::BW;
  if constexpr (I < Geom<R, NH>::SROWS) {
    constexpr int OFF = pmod(R - K * R, n);  // q0 mod n (RC is a multiple of n)
    constexpr int I0 = pmod(I + OFF, n);
    if constexpr (K > 1 && RDG_PF > 0 && R >= RDG_PF) {
      if constexpr (I == 0) {
#pragma unroll
        for (int h = 0; h < NH; ++h) load_x<R>(st + 64 * h, p, xq[h]);
      }
      // PF2 (K = 2, light signatures): stage 2's input row (written by stage 1 in the previous
      // iteration) is loaded before stage 1's work as well
      constexpr bool PF2 = K == 2 && (RDG_PF2 == 1 || (RDG_PF2 == 2 && SIG == SIG_STAR));
      double x2[NH][2 * R + 2];
      if constexpr (PF2) {
        const double* b2 = bufs + (((par0 + I) & 1) ^ 1) * Geom<R, NH>::BUFD;
#pragma unroll
        for (int h = 0; h < NH; ++h) load_x<R>(b2 + 64 * h, p, x2[h]);
      }
      fused_iter<R, SIG, K, NH, FULL, I0, I, 1, true, 1>(st + I * BW, p, acc, P, bufs, (par0 + I) & 1, in, out, P1, sc, lc,
                                                         dp, xq);
      if constexpr (I + 1 < Geom<R, NH>::SROWS) {
#pragma unroll
        for (int h = 0; h < NH; ++h) load_x<R>(st + (I + 1) * BW + 64 * h, p, xq[h]);
      }
      if constexpr (PF2)
        fused_iter<R, SIG, K, NH, FULL, I0, I, 2, true, 2>(st + I * BW, p, acc, P, bufs, (par0 + I) & 1, in, out, P1, sc,
                                                           lc, dp, x2);
      else
        fused_iter<R, SIG, K, NH, FULL, I0, I, K, false, 2>(st + I * BW, p, acc, P, bufs, (par0 + I) & 1, in, out, P1, sc,
                                                            lc, dp, xq);
    } else {
      fused_iter<R, SIG, K, NH, FULL, I0, I, K>(st + I * BW, p, acc, P, bufs, (par0 + I) & 1, in, out, P1, sc, lc, dp, xq);
    }
    if constexpr (K > 1) __syncwarp();
    fused_rows<R, SIG, K, NH, FULL, I + 1>(st, p, acc, P, bufs, in, out, P1, sc, lc, par0, dp, xq);
  }
}

#ifndef RDG_LOOP
#define RDG_LOOP 2   // runtime row loop + row_shift — 2: fused radius >= 3 rows / PMA kernels, 1: every
#endif               // fused rows / PMA / star kernel, 0: never (ring form everywhere)
// Measured (same box, short runs; tools/gpu_variants.sh): Box-2D49P k = 2 322 -> 327 GS/s (ncu:
// no_instruction stalls 0.61 -> 0.14 per issue, 12 % more instructions), Box-2D9P k = 3 673 -> 655,
// Star-2D13P k = 2 456 -> 418 (the ring form there also loads stage 2's row early, RDG_PF2).
template <int R, int SIG, int K>
constexpr bool rdg_loop() {
  return K >= 2 && ((RDG_LOOP == 1 && (SIG == SIG_ROWS || SIG == SIG_PMA || SIG == SIG_STAR)) ||
                    (RDG_LOOP == 2 && R >= 3 && (SIG == SIG_ROWS || SIG == SIG_PMA)));
}

// The rows of one staged tile as a runtime loop (one copy of the K x NH row code; see row_shift).
template <int R, int SIG, int K, int NH, bool FULL, bool REM = true>
__device__ __forceinline__ void fused_rows_loop(const double* __restrict__ st, int p, double (&acc)[K][NH][2 * R + 1][2],
                                                const RdgParams& P, double* __restrict__ bufs,
                                                const double* __restrict__ in, double* __restrict__ out, int64_t P1,
                                                const StageCtx<K>& sc, const LaneCtx<NH>& lc, int par0,
                                                const P2PArgs& dp, double (&xq)[NH][2 * R + 2]) {
  constexpr int BW = Geom<R, NH>::BW, SROWS = Geom<R, NH>::SROWS;
  constexpr bool PF = RDG_PF > 0 && R >= RDG_PF;
  if constexpr (PF) {
#pragma unroll
    for (int h = 0; h < NH && h < RDG_PF_HALVES; ++h) load_x<R>(st + 64 * h, p, xq[h]);
  }
  double* orow = out + sc.ooff;   // output row of the final stage for I = 0 (only dereferenced when stored)
#pragma unroll kRowUnroll
  for (int I = 0; I < SROWS; ++I, orow += P1) {
    const int par = (par0 + I) & 1;
    if constexpr (PF) {
      fused_iter<R, SIG, K, NH, FULL, 0, 0, 1, true, 1, true, REM>(st + I * BW, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, xq, I,
                                                              orow);
      if (I + 1 < SROWS) {
#pragma unroll
        for (int h = 0; h < NH && h < RDG_PF_HALVES; ++h) load_x<R>(st + (I + 1) * BW + 64 * h, p, xq[h]);
      }
      fused_iter<R, SIG, K, NH, FULL, 0, 0, K, false, 2, true, REM>(st + I * BW, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, xq, I,
                                                               orow);
    } else if constexpr (RDG_S1LOAD) {   // stage 1's input row loaded first, stages K .. 2, then stage 1
      double x1[NH][2 * R + 2];
#pragma unroll
      for (int h = 0; h < NH; ++h) load_x<R>(st + I * BW + 64 * h, p, x1[h]);
      fused_iter<R, SIG, K, NH, FULL, 0, 0, K, false, 2, true, REM>(st + I * BW, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, xq, I,
                                                                    orow);
      fused_iter<R, SIG, K, NH, FULL, 0, 0, 1, true, 1, true, REM>(st + I * BW, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, x1, I,
                                                                   orow);
    } else if constexpr (RDG_S1FIRST) {   // stage 1, then stages K .. 2 (the stages of an iteration are independent)
      fused_iter<R, SIG, K, NH, FULL, 0, 0, 1, false, 1, true, REM>(st + I * BW, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, xq, I,
                                                                    orow);
      fused_iter<R, SIG, K, NH, FULL, 0, 0, K, false, 2, true, REM>(st + I * BW, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, xq, I,
                                                                    orow);
    } else {
      fused_iter<R, SIG, K, NH, FULL, 0, 0, K, false, 1, true, REM>(st + I * BW, p, acc, P, bufs, par, in, out, P1, sc, lc, dp, xq, I,
                                                               orow);
    }
    __syncwarp();
  }
}

#ifndef RDG_MINB_ALL
#define RDG_MINB_ALL 0   // experiments: force resident CTAs per SM for every instantiation
#endif
// Resident CTAs per SM (register budget 512 / minb per thread x 128 threads), measured on B200
// (profiles/r01_rdg_occupancy.txt): the heavy radius >= 3 PMA pass wants registers for ILP more
// than warps (2 CTAs: 338 GS/s vs 305 at 4 for Box-2D49P); light passes want 4; fused radius >= 2 3.
#ifndef RDG_FULL
// 2: unfused kernels get a second copy of the row loop without per-row checks for interior stages;
// the fused kernels do not (see rdg_full).  0: never, 1: always (experiments).
#define RDG_FULL 2
#endif
#ifndef RDG_NH_MINR
#define RDG_NH_MINR 1   // smallest radius with NH = 2 in the fused kernels (r02zf: Box-2D9P k = 3 730 -> 747 GS/s with 1)
#endif
#ifndef RDG_NH_FUSED
#define RDG_NH_FUSED 2   // 64-column halves per warp in the fused (K >= 2) kernels
#endif
// Check-free copy of the row loop for interior stages: unfused kernels only.  Measured on one box
// (tools/gpu_variants.sh, short runs): the fused kernels are slower with it — Box-2D49P k = 2 310 ->
// 261 GS/s, Star-2D13P k = 2 431 -> 351 — and the unfused ones gain little (Star-2D13P 311 -> 317).
template <int R, int SIG, int K>
constexpr bool rdg_full() {
  return RDG_FULL == 1 || (RDG_FULL == 2 && K == 1);
}
template <int R, int K>
constexpr int rdg_cta_smem(int nh) {   // must match rdg_launch
  return nh == 1 ? 128 + RDG_WARPS * (Geom<R, 1>::WARP_BYTES + 2 * (K - 1) * Geom<R, 1>::BUFD * 8)
                 : 128 + RDG_WARPS * (Geom<R, 2>::WARP_BYTES + 2 * (K - 1) * Geom<R, 2>::BUFD * 8);
}
// NH = 2 where two CTAs of it still fit the 228 KB of shared memory per SM (R = 3, 4)
template <int R, int SIG, int K>
// (radius 1: Box-2D9P k = 3 641 vs 630 GS/s with vector-register weights, 747 vs 730 with uniform ones)
constexpr int rdg_nh() {
  return (K >= 2 && R >= RDG_NH_MINR && RDG_NH_FUSED == 2 && 2 * (rdg_cta_smem<R, K>(2) + 1024) <= 228 * 1024) ? 2 : 1;
}

template <int R, int SIG, int K>
constexpr int rdg_minb() {
  return (RDG_MINB_ALL > 0) ? RDG_MINB_ALL
         : (rdg_nh<R, SIG, K>() == 2 ? 2
            : (((SIG == SIG_PMA || SIG == SIG_ROWS || SIG == SIG_DIRECT) && R >= 3 && K == 1) ? 2
                                                                                        : ((K == 1 || R == 1) ? 4 : 3)));
}

// P2P: the device-initiated exchange hooks (csrc/dist_p2p.cu) are compiled in.  The single-GPU
// instantiation has none: with the spin-wait code in the kernel ptxas keeps the stencil weights in
// vector registers (three vector operands per DFMA); without it they live in uniform registers
// (DFMA R, R, UR, R), which the FP64 pipe issues faster (tools/ubench/fp64_mix.cu: +20 % for this
// instruction mix) and which frees 32 vector registers per thread.
template <int R, int SIG, int K, bool TMA, bool P2P>
__global__ void __launch_bounds__(RDG_WARPS * 32, (rdg_minb<R, SIG, K>())) rdg2d_kernel(const double* __restrict__ in, double* __restrict__ out,
                                                              int64_t N0, int64_t N1, int nbands, int nitems, int RC,
                                                              int SI, const __grid_constant__ CUtensorMap tmap,
                                                              const __grid_constant__ RdgParams prm,
                                                              const __grid_constant__ P2PArgs dp) {
  constexpr int NH = rdg_nh<R, SIG, K>();
  using G = Geom<R, NH>;
  constexpr int SG = (R * (K - 1)) & 1;           // shift keeping the staged origin even (TMA: 16-B aligned start)
  constexpr int BS = 64 * NH - 2 * R * (K - 1) - 2 * SG;  // band stride (valid final columns per band)
  constexpr int BUFD = G::BUFD;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  const bool dact = P2P && dp.active;
  const int lane = threadIdx.x & 31;
  // the warp index through a shuffle from lane 0: ptxas then knows it (and all item geometry derived
  // from it) is warp-uniform — uniform branches and uniform-datapath address arithmetic
  const int wl = RDG_UNIFORM_WL ? __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0) : (int)(threadIdx.x >> 5);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw) + wl * RDG_NS;
  unsigned char* wbase = smem_raw + 128 + wl * (G::WARP_BYTES + 2 * (K - 1) * BUFD * 8);
  unsigned char* ring = wbase;
  double* bufmem = reinterpret_cast<double*>(wbase + G::WARP_BYTES);
  double* bufs = bufmem;                        // [stage][parity] rows of BUFD doubles
  for (int i = lane; i < 2 * (K - 1) * BUFD; i += 32) bufmem[i] = 0.0;  // margins stay zero
  const int64_t P1 = N1 + 2 * R;
  const int P0 = (int)(N0 + 2 * R);
  const int gw = blockIdx.x * RDG_WARPS + wl, TW = gridDim.x * RDG_WARPS;
  const int my_items = gw < nitems ? (nitems - 1 - gw) / TW + 1 : 0;
  const int nstages = my_items * SI;
  if (TMA && lane == 0) {
    for (int s = 0; s < RDG_NS; ++s) mbar_init(&bars[s], 1);
    fence_barrier_init();
  }
  __syncwarp();
  // item geometry: band b -> lane column 0 at padded column X0; chunk c -> final rows from A
  const int nch = nitems / nbands;
  auto geom = [&](int item, int& X0, int& A) {
    const int band = item % nbands;
    const int chunk = dact ? p2p_chunk_order(item / nbands, nch) : item / nbands;
    X0 = R + band * BS - R * (K - 1) - SG;
    A = R + chunk * RC;
  };
  // device-initiated exchange: the item holding the first (last) H rows of the slab touches the
  // lower (upper) neighbour — it stores them into the neighbour's halo and stages the halo the
  // neighbour wrote; the host keeps that item unique per band (RC >= 2H, last chunk >= 2H - R rows)
  auto touches = [&](int A_, bool& lo, bool& hi) {
    lo = dact && dp.dst_lo != nullptr && A_ < dp.lo_end;
    hi = dact && dp.dst_hi != nullptr && A_ + RC - 1 >= dp.hi_begin;
  };
  // producer position (next stage to stage into the ring)
  int pitem = gw, pj = 0, pX0 = 0, pA = 0;
  if (gw < nitems) geom(pitem, pX0, pA);
  auto issue_next = [&](int slot) {
    const int x = pX0 - R, y = pA - K * R + pj * G::SROWS;
    if (dact && pj == 0) {  // the halo this item stages was written by a neighbour: wait for it
      bool lo, hi;
      touches(pA, lo, hi);
      if (lo || hi) {   // warp-uniform
        const int b = pitem % nbands;
        const int u0 = dp.wait_units > 0 ? 0 : max(b - 1, 0), u1 = dp.wait_units > 0 ? dp.wait_units - 1 : min(b + 1, nbands - 1);
        if (lo) p2p_wait_units_warp(dp.wait_lo, u0, u1, dp.wait_val, dp.err);
        if (hi) p2p_wait_units_warp(dp.wait_hi, u0, u1, dp.wait_val, dp.err);
        if (lane == 0) fence_proxy_async_global();
      }
      __syncwarp();
    }
    double* dst = reinterpret_cast<double*>(ring + slot * G::STAGE);
    if constexpr (TMA) {
      if (lane == 0) {  // x is even by construction; negative origins are zero-filled by TMA
        fence_proxy_async();
        mbar_arrive_expect_tx(&bars[slot], G::SROWS * G::BW * 8);
        tma_load_2d(dst, &tmap, x, y, &bars[slot]);
      }
    } else {
      for (int i = lane; i < G::SROWS * G::BW; i += 32) {
        const int r = i / G::BW, cc = i - r * G::BW;
        const int64_t gy = y + r, gx = x + cc;
        if (gy >= 0 && gy < P0 && gx >= 0 && gx < P1) cp_async8(dst + i, in + gy * P1 + gx);
        else dst[i] = 0.0;
      }
      cp_async_commit();
    }
    if (++pj == SI) {
      pj = 0;
      pitem += TW;
      if (pitem < nitems) geom(pitem, pX0, pA);
    }
  };
  for (int q = 0; q < RDG_NS - 1; ++q) {
    if (q < nstages) issue_next(q);
    else if constexpr (!TMA) cp_async_commit();  // empty group: keeps wait_group<NS-1> exact
  }
  double acc[K][NH][2 * R + 1][2];
  LaneCtx<NH> lc{};
  StageCtx<K> sc{};
  int citem = gw, cj = 0, X0 = 0, A = 0, rows_valid_end = 0;
  bool all_fast = false;   // every lane of the item: 16-byte stores, no column halo / outside column
  bool t_lo = false, t_hi = false;   // the current item touches the lower / upper neighbour
  int slot = 0, phase = 0;
  for (int q = 0; q < nstages; ++q) {
    if (q + RDG_NS - 1 < nstages) issue_next((slot + RDG_NS - 1) % RDG_NS);
    else if constexpr (!TMA) cp_async_commit();  // keep the group count uniform
    if constexpr (TMA) {
      mbar_wait(&bars[slot], phase);
    } else {
      cp_async_wait<RDG_NS - 1>();
      __syncwarp();
    }
    if (cj == 0) {
      geom(citem, X0, A);
#pragma unroll
      for (int k = 0; k < K; ++k)
#pragma unroll
        for (int h = 0; h < NH; ++h)
#pragma unroll
          for (int s = 0; s < 2 * R + 1; ++s) { acc[k][h][s][0] = 0.0; acc[k][h][s][1] = 0.0; }
      lc.c0 = X0 + 2 * lane;
      lc.edge = false;
#pragma unroll
      for (int h = 0; h < NH; ++h) {
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const int c = lc.c0 + 64 * h + j;
          lc.inside[h][j] = c >= 0 && c < P1;
          lc.colhalo[h][j] = lc.inside[h][j] && (c < R || c >= P1 - R);
          // the band's own BS columns (even-aligned: X0 and R(K-1) + SG are even), so a lane's
          // pair is valid or invalid as a whole except at the array's right edge
          lc.valid[h][j] = c >= X0 + R * (K - 1) + SG && c < X0 + R * (K - 1) + SG + BS && c >= R && c < P1 - R;
          lc.edge = lc.edge || lc.colhalo[h][j] || !lc.inside[h][j];
        }
        lc.vec[h] = lc.valid[h][0] && lc.valid[h][1] &&
                    ((reinterpret_cast<uintptr_t>(out + lc.c0 + 64 * h) & 15) == 0) && ((P1 & 1) == 0);
      }
      rows_valid_end = min(A + RC, dact ? dp.store_hi : P0 - R);
      // FULL lanes: no halo columns; a pair is stored as a whole or not at all — one 16-byte store
      // for even R; for odd R the lane columns X0 + 2p are odd (the staged origin X0 - R is kept
      // even for TMA), so the pair is two 8-byte stores
      lc.edge_any = __any_sync(0xffffffffu, lc.edge);
      bool mine = !lc.edge;
#pragma unroll
      for (int h = 0; h < NH; ++h)
        mine = mine && lc.valid[h][0] == lc.valid[h][1] && ((R & 1) || lc.vec[h] || !lc.valid[h][0]);
      all_fast = __all_sync(0xffffffffu, mine);
      touches(A, t_lo, t_hi);
    }
    // stage bookkeeping: input row I of this stage is padded row yb + I
    const int yb = A - K * R + cj * G::SROWS;
    {
      const int yf = yb - K * R - (K - 1);  // final row produced by input row I = 0 (one-row lag per stage)
      sc.lo = (dact ? max(A, dp.store_lo) : A) - yf;
      sc.hi = rows_valid_end - yf;
      sc.ooff = int64_t(yf) * P1 + lc.c0;
      sc.rem_lo = t_lo ? dp.lo_end - yf : INT_MIN;       // rows [store_lo, lo_end)
      sc.rem_hi = t_hi ? dp.hi_begin - yf : INT_MAX;     // rows [hi_begin, store_hi)
#pragma unroll
      for (int S = 1; S < K; ++S) {
        const int ys = yb - S * R - (S - 1);  // stage-S row produced by input row I = 0
        sc.hlo[S - 1] = R - ys;
        sc.hhi[S - 1] = P0 - R - ys;
        sc.rlo[S - 1] = -ys;
        sc.rhi[S - 1] = P0 - ys;
        sc.ioff[S - 1] = int64_t(ys) * P1;
      }
    }
    const double* st = reinterpret_cast<const double*>(ring + slot * G::STAGE);
    bool full = all_fast && sc.lo <= 0 && sc.hi >= G::SROWS && sc.rem_lo <= 0 && sc.rem_hi >= G::SROWS;
#pragma unroll
    for (int S = 1; S < K; ++S) full = full && sc.hlo[S - 1] <= 0 && sc.hhi[S - 1] >= G::SROWS;
    double xq[NH][2 * R + 2];   // prefetched stage-1 input row (RDG_PF)
    if constexpr (rdg_loop<R, SIG, K>()) {
      // P2P: only the stages holding one of the slab's first / last H rows take the row code with
      // the peer stores (the others run the single-GPU row code: 931 vs 997 us per launch)
      const bool rem = P2P && (sc.rem_lo > 0 || sc.rem_hi < G::SROWS);
      if (rdg_full<R, SIG, K>() && full) fused_rows_loop<R, SIG, K, NH, true>(st, lane, acc, prm, bufs, in, out, P1, sc, lc, yb & 1, dp, xq);
      else if (rem) fused_rows_loop<R, SIG, K, NH, false, true>(st, lane, acc, prm, bufs, in, out, P1, sc, lc, yb & 1, dp, xq);
      else fused_rows_loop<R, SIG, K, NH, false, false>(st, lane, acc, prm, bufs, in, out, P1, sc, lc, yb & 1, dp, xq);
    } else {
      if (rdg_full<R, SIG, K>() && full) fused_rows<R, SIG, K, NH, true, 0>(st, lane, acc, prm, bufs, in, out, P1, sc, lc, yb & 1, dp, xq);
      else fused_rows<R, SIG, K, NH, false, 0>(st, lane, acc, prm, bufs, in, out, P1, sc, lc, yb & 1, dp, xq);
    }
    __syncwarp();  // every lane is done with this slot before it is refilled
    if (++slot == RDG_NS) { slot = 0; phase ^= 1; }
    if (++cj == SI) {
      if (t_lo) p2p_signal_warp(dp.sig_lo, citem % nbands, dp.sig_val);   // my edge rows are in its halo,
      if (t_hi) p2p_signal_warp(dp.sig_hi, citem % nbands, dp.sig_val);   // my halo reads are done
      cj = 0;
      citem += TW;
    }
  }
}

int signature(const Plan& p, RdgParams& prm) {
  std::memset(&prm, 0, sizeof(prm));
  const int R = p.R, n = 2 * R + 1;
  if (p.rdg_rows && p.ndim == 2) {
    // row pairs with a unit centre tap: v_a = W[R+a,:] / c_a, c_a = W[R+a,R] (nonzero: planner.cpp)
    prm.K = R + 1;
    for (int a = 0; a <= R; ++a) {
      const double ca = p.W[size_t(R + a) * n + R];
      for (int j = 0; j < n; ++j) prm.v[a][j] = p.W[size_t(R + a) * n + j] / ca;
      prm.v[a][R] = 1.0;
      prm.u[a][0] = ca;
    }
    return SIG_ROWS;
  }
  // PMA pyramid: chains of radius R, R-1, ..., 1 (in that order) + centre scalar
  bool pma = (int)p.terms.size() == R + 1;
  for (int k = 0; pma && k < R; ++k) pma = p.terms[k].kind == kChain && p.terms[k].r == R - k;
  if (pma) pma = p.terms[R].kind == kPoint && p.terms[R].u[R] == 1.0 && p.terms[R].r == 0;
  for (int k = 0; pma && k < R; ++k) pma = p.terms[k].v[R] != 0.0;
  if (pma) {
    // each chain rescaled so that the centre tap of v is exactly 1 (v' = v / v[R], u' = u v[R]):
    // the horizontal gather starts from x_0 itself, one DMUL less per term and element
    prm.K = R;
    for (int k = 0; k < R; ++k) {
      const double c = p.terms[k].v[R];
      for (int i = 0; i < n; ++i) { prm.u[k][i] = p.terms[k].u[i] * c; prm.v[k][i] = p.terms[k].v[i] / c; }
      prm.v[k][R] = 1.0;
    }
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

template <int R, int SIG, int K, bool TMA>
cudaError_t rdg_launch(const Plan& p, const double* src, double* dst, cudaStream_t s, const CUtensorMap& map,
                       const RdgParams& prm, const P2PArgs* d) {
  constexpr int NH = rdg_nh<R, SIG, K>();
  using G = Geom<R, NH>;
  constexpr int n = 2 * R + 1;
  constexpr int BS = 64 * NH - 2 * R * (K - 1) - 2 * ((R * (K - 1)) & 1);
  constexpr int BUFD = G::BUFD;
  const int smem = 128 + RDG_WARPS * (G::WARP_BYTES + 2 * (K - 1) * BUFD * 8);
  int max_grid = 0;
  {
    cudaError_t e = d && d->active ? kernel_setup((const void*)rdg2d_kernel<R, SIG, K, TMA, true>, RDG_WARPS * 32, smem, &max_grid)
                                   : kernel_setup((const void*)rdg2d_kernel<R, SIG, K, TMA, false>, RDG_WARPS * 32, smem, &max_grid);
    if (e != cudaSuccess) return e;
  }
  if (d && d->prepare_only) return cudaSuccess;
  // chunk rows: a multiple of 2R+1 (static ring slots), <= RDG_RC; small grids get shorter chunks
  // so that every resident warp has a stream (>= 2 items per warp slot when the grid allows it)
  const int nbands = (int)((p.N[1] + BS - 1) / BS);
  const int64_t TWmax = int64_t(max_grid) * RDG_WARPS;
  const int64_t want = TWmax * 2;
  int64_t rc = (p.N[0] * nbands + want - 1) / want;
  rc = std::max<int64_t>(rc, 4 * K * R);                      // keep the halo-row overhead bounded
  rc = std::min<int64_t>(rc, RDG_RC);
  rc = ((rc + n - 1) / n) * n;
  {  // wave balance: the fewest whole rounds of TWmax items, then the shortest chunk that fits them
    const int64_t nitems0 = nbands * ((p.N[0] + rc - 1) / rc);
    const int64_t rounds = (nitems0 + TWmax - 1) / TWmax;
    const int64_t nch = std::max<int64_t>(1, (rounds * TWmax) / nbands);
    int64_t rc2 = (p.N[0] + nch - 1) / nch;
    rc2 = ((rc2 + n - 1) / n) * n;
    if (rc2 <= RDG_RC + n && rc2 >= 4 * K * R && nbands * ((p.N[0] + rc2 - 1) / rc2) <= rounds * TWmax) rc = rc2;
  }
  if (d && d->active) {
    // device-initiated exchange: exactly one chunk per band and side may touch a neighbour: the
    // first chunk must hold rows [store_lo, lo_end) (RC >= 2H) and the last one >= 2H - R rows
    const int64_t H = std::max(d->H, R);
    rc = std::max<int64_t>(rc, ((2 * H + n - 1) / n) * n);
    if (rc < p.N[0]) {
      int64_t ok = 0;
      for (int64_t c = rc; c <= rc + 40 * n && !ok; c += n) {
        const int64_t rem = p.N[0] % c;
        if (rem == 0 || rem >= 2 * H - R) ok = c;
      }
      rc = ok ? ok : ((p.N[0] + n - 1) / n) * n;
    }
  }
  const int RC = (int)rc;
  const int SI = (RC + 2 * K * R + (K - 1) + G::SROWS - 1) / G::SROWS;
  const int nchunks = (int)((p.N[0] + RC - 1) / RC);
  const int nitems = nbands * nchunks;
  const int grid = (int)std::min<int64_t>(max_grid, (nitems + RDG_WARPS - 1) / RDG_WARPS);
  static const P2PArgs none{};
  if (d && d->active)
    rdg2d_kernel<R, SIG, K, TMA, true><<<grid, RDG_WARPS * 32, smem, s>>>(src, dst, p.N[0], p.N[1], nbands, nitems, RC, SI,
                                                                         map, prm, *d);
  else
    rdg2d_kernel<R, SIG, K, TMA, false><<<grid, RDG_WARPS * 32, smem, s>>>(src, dst, p.N[0], p.N[1], nbands, nitems, RC,
                                                                          SI, map, prm, none);
  return cudaGetLastError();
}

template <int R, int SIG, int K>
cudaError_t rdg_sig(const Plan& p, const double* src, double* dst, cudaStream_t s, const RdgParams& prm,
                    const P2PArgs* d = nullptr) {
  using G = Geom<R, rdg_nh<R, SIG, K>()>;
  CUtensorMap map;
  const int64_t padded[2] = {p.P[0], p.P[1]};
  const int box[2] = {G::SROWS, G::BW};
  if (!p.force_no_tma && encode_tmap(&map, src, 2, padded, box))
    return rdg_launch<R, SIG, K, true>(p, src, dst, s, map, prm, d);
  std::memset(&map, 0, sizeof(map));
  return rdg_launch<R, SIG, K, false>(p, src, dst, s, map, prm, d);
}

constexpr int max_fuse(int R) { return R == 1 ? 4 : (R == 2 ? 3 : 2); }

template <int R, int SIG>
cudaError_t rdg_k(const Plan& p, const double* src, double* dst, cudaStream_t s, const RdgParams& prm, int k,
                  const P2PArgs* d = nullptr) {
  if (d && (k == 1 || SIG == SIG_FULL || SIG == SIG_DIRECT)) return k == 1 ? rdg_sig<R, SIG, 1>(p, src, dst, s, prm, d) : cudaErrorNotSupported;
  if constexpr (SIG == SIG_FULL || SIG == SIG_DIRECT) {
    if (k != 1) return cudaErrorNotSupported;
    return rdg_sig<R, SIG, 1>(p, src, dst, s, prm);
  } else {
    switch (k) {
      case 1: return rdg_sig<R, SIG, 1>(p, src, dst, s, prm, d);
      case 2: return rdg_sig<R, SIG, 2>(p, src, dst, s, prm, d);
      case 3: if constexpr (max_fuse(R) >= 3) return rdg_sig<R, SIG, (max_fuse(R) >= 3 ? 3 : 1)>(p, src, dst, s, prm, d); break;
      case 4: if constexpr (max_fuse(R) >= 4) return rdg_sig<R, SIG, (max_fuse(R) >= 4 ? 4 : 1)>(p, src, dst, s, prm, d); break;
    }
    return cudaErrorNotSupported;
  }
}

template <int R>
cudaError_t rdg_r(const Plan& p, const double* src, double* dst, cudaStream_t s, int k, const P2PArgs* d = nullptr) {
  RdgParams prm;
  const int sig = signature(p, prm);
  if (sig == SIG_PMA) return rdg_k<R, SIG_PMA>(p, src, dst, s, prm, k, d);
  if constexpr (R >= 3) {
    if (sig == SIG_ROWS) return rdg_k<R, SIG_ROWS>(p, src, dst, s, prm, k, d);
  }
  if (sig == SIG_STAR) return rdg_k<R, SIG_STAR>(p, src, dst, s, prm, k, d);
  if (sig == SIG_FULL) return rdg_k<R, SIG_FULL>(p, src, dst, s, prm, k, d);
  return cudaErrorNotSupported;
}

}  // namespace

bool rdg2d_supported(const Plan& p) {
  if (p.ndim == 3) return rdg3d_supported(p);
  if (p.ndim != 2) return false;
  RdgParams prm;
  return signature(p, prm) >= 0;
}

namespace {
cudaError_t direct2d(const Plan& p, const double* src, double* dst, cudaStream_t s, const P2PArgs* d) {
  if (p.ndim != 2) return cudaErrorInvalidValue;
  RdgParams prm;
  std::memset(&prm, 0, sizeof(prm));
  const int n = 2 * p.R + 1;
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < n; ++j) prm.u[i][j] = p.W[size_t(i) * n + j];
  switch (p.R) {
    case 1: return rdg_sig<1, SIG_DIRECT, 1>(p, src, dst, s, prm, d);
    case 2: return rdg_sig<2, SIG_DIRECT, 1>(p, src, dst, s, prm, d);
    case 3: return rdg_sig<3, SIG_DIRECT, 1>(p, src, dst, s, prm, d);
    case 4: return rdg_sig<4, SIG_DIRECT, 1>(p, src, dst, s, prm, d);
  }
  return cudaErrorInvalidValue;
}
}  // namespace

cudaError_t launch_direct2d_stream(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  return direct2d(p, src, dst, s, nullptr);
}

int rdg2d_max_fuse(const Plan& p) {
  if (p.ndim == 3) return rdg3d_fused_supported(p) ? 3 : 1;
  if (p.ndim != 2) return 1;
  RdgParams prm;
  const int sig = signature(p, prm);
  if (sig < 0 || sig == SIG_FULL) return 1;
  return max_fuse(p.R);
}

// Flag units per side of the device-initiated exchange (csrc/dist_p2p.cu): the 64-column bands of
// the unfused 2D stream kernel; 3D: the 64 x BY columns of rdg3d_kernel.
int p2p_units(const Plan& p, int* nux) {
  if (nux) *nux = 0;
  if (p.ndim == 3) return rdg3d_p2p_units(p, nux);
  if (p.ndim != 2 || (p.engine != LORA_ENGINE_RDG_CUDA && p.engine != LORA_ENGINE_DIRECT)) return 0;
  if (p.engine == LORA_ENGINE_RDG_CUDA && !rdg2d_supported(p)) return 0;
  return (int)((p.N[1] + 63) / 64);
}

cudaError_t launch_step_p2p(const Plan& p, const double* src, double* dst, cudaStream_t s, const P2PArgs& d, int k) {
  if (p.ndim == 3) {
    if (k == 1) return launch_rdg3d_p2p(p, src, dst, s, d);
    return p.engine == LORA_ENGINE_RDG_CUDA ? launch_rdg3d_fused(p, src, dst, s, k, &d) : cudaErrorNotSupported;
  }
  if (p.ndim != 2) return cudaErrorNotSupported;
  if (p.engine == LORA_ENGINE_DIRECT) return k == 1 ? direct2d(p, src, dst, s, &d) : cudaErrorNotSupported;
  if (p.engine != LORA_ENGINE_RDG_CUDA) return cudaErrorNotSupported;
  switch (p.R) {
    case 1: return rdg_r<1>(p, src, dst, s, k, &d);
    case 2: return rdg_r<2>(p, src, dst, s, k, &d);
    case 3: return rdg_r<3>(p, src, dst, s, k, &d);
    case 4: return rdg_r<4>(p, src, dst, s, k, &d);
  }
  return cudaErrorInvalidValue;
}

// Band count of the 2D stream kernel at fusion depth k (the flag units of the exchange).
namespace {
template <int R>
int band_stride(int k) {
  int nh = 1;
  switch (k) {
    case 2: nh = rdg_nh<R, SIG_PMA, 2>(); break;
    case 3: nh = rdg_nh<R, SIG_PMA, 3>(); break;
    case 4: nh = rdg_nh<R, SIG_PMA, 4>(); break;
  }
  return 64 * nh - 2 * R * (k - 1) - 2 * ((R * (k - 1)) & 1);
}
}  // namespace

int p2p_units_k(const Plan& p, int k) {
  if (p.ndim == 3 && k >= 2) return rdg3d_fused_units(p, k, nullptr);
  if (p.ndim != 2 || k <= 1) return p2p_units(p, nullptr);
  const int bs = p.R == 1 ? band_stride<1>(k) : p.R == 2 ? band_stride<2>(k) : p.R == 3 ? band_stride<3>(k) : band_stride<4>(k);
  return (int)((p.N[1] + bs - 1) / bs);
}

cudaError_t launch_rdg2d(const Plan& p, const double* src, double* dst, cudaStream_t s, int k) {
  if (p.ndim == 3) return k == 1 ? launch_rdg3d(p, src, dst, s) : launch_rdg3d_fused(p, src, dst, s, k);
  switch (p.R) {
    case 1: return rdg_r<1>(p, src, dst, s, k);
    case 2: return rdg_r<2>(p, src, dst, s, k);
    case 3: return rdg_r<3>(p, src, dst, s, k);
    case 4: return rdg_r<4>(p, src, dst, s, k);
  }
  return cudaErrorInvalidValue;
}

}  // namespace lora
