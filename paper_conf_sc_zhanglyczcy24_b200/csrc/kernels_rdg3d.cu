// K2/K3 on CUDA cores — LoRAStencil-3D (§IV-C Alg. 2) with RDG per plane.
//
// Alg. 2: the (2R+1)^3 stencil is the sum over its 2R+1 z-planes W_{a0} of 2D stencils applied
// to the input planes; a plane holding a single weight is a point-wise multiply-add on CUDA cores
// (lines 3-5), any other plane is a 2D LoRAStencil (lines 7-8) — here its rank-1 terms u v^T
// (planner, eq. 8/15) evaluated as the two banded gathers of RDG (horizontal v-pass, vertical
// u-pass), or the two arms of a star plane.  Result for output plane z: sum_{a0} W_{a0} * X_{z+a0}.
//
// B200 mapping: one warp streams a 64-column x BY-row column of the domain along z through a
// chunk of ZC output planes.  Input planes arrive by TMA (3D box 1 x (BY+2R) x (64+2R), zero
// fill) into a per-warp ring; each input plane p is read from shared memory ONCE and contributes
// to the 2R+1 output planes z = p - a0 held in a register ring.  When W_{a0} == W_{2R-a0}
// (z-symmetric, e.g. Box-3D27P and Heat-3D) the plane result is computed once and added to both
// output planes.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <utility>
#include <vector>

#include "kernels.hpp"
#include "p2p.cuh"
#include "pipe.cuh"

namespace lora {
namespace {

constexpr int R3_WARPS = 4;
constexpr int R3_NS = 4;
template <int R> constexpr int BY = (R == 1 ? 4 : 2);
constexpr int R3_ZC = 64;
constexpr int R3_MAXK = 5;   // rank-1 terms per plane (<= 2R+1 for R <= 2)

enum { PM_NONE = 0, PM_POINT = 1, PM_CHAINS = 2, PM_STAR = 3, PM_PMA1 = 4, PM_DIRECT = 5, PM_SYM3 = 6 };

struct R3Params {
  int mode[5];               // per plane a0
  int K[5];                  // chain terms per plane
  int mirror[5];             // plane a0 (< R) also feeds output z = p - (2R - a0)
  double w[5];               // PM_POINT weight (centre) / PM_PMA1 scalar C_{h+1}
  double u[5][R3_MAXK][5];   // plane, term, tap (centred, length 2R+1)
  double v[5][R3_MAXK][5];
  double sym[2][3];          // PM_SYM3 (planes 0 and 1 jointly, R = 1): centre c, edge b, corner a
};

template <int R>
struct G3 {
  static constexpr int n = 2 * R + 1;
  static constexpr int ROWS = BY<R> + 2 * R;
  static constexpr int BW = 64 + 2 * R;
  static constexpr int STAGE = ((ROWS * BW * 8 + 127) / 128) * 128;
  static constexpr int WARP_BYTES = R3_NS * STAGE;
  static constexpr int SMEM = 128 + R3_WARPS * WARP_BYTES;
};

__host__ __device__ constexpr int pm(int a, int n) { return ((a % n) + n) % n; }

// Applies plane operator a0 to the staged plane (registers x) and adds into the ring slot(s).
// Mode signature of a specialised kernel: planes 0 and 1 modes (-1 = run time), plane-0/2 mirror.
template <int M0, int M1, int MIR>
struct Sig3 {
  static constexpr int m0 = M0, m1 = M1, mir = MIR;
};

template <int R, int A0, int I, int MODE = -1, int MIR = -1>
__device__ __forceinline__ void apply_plane(const double (&x)[BY<R> + 2 * R][2 * R + 2],
                                            double (&acc)[2 * R + 1][BY<R>][2], const R3Params& P) {
  constexpr int n = 2 * R + 1;
  constexpr int s1 = pm(I - A0, n);           // output plane z = p - a0
  constexpr int s2 = pm(I - (n - 1 - A0), n); // mirrored plane
  const int mode = MODE >= 0 ? MODE : P.mode[A0];
  if (mode == PM_NONE) return;
  double d[BY<R>][2];
  if (mode == PM_POINT) {
#pragma unroll
    for (int y = 0; y < BY<R>; ++y) {
      d[y][0] = P.w[A0] * x[y + R][R];
      d[y][1] = P.w[A0] * x[y + R][R + 1];
    }
  } else if (mode == PM_STAR) {
    // horizontal arm v (u = e_R) on the centre row, vertical arm u (v = e_R) on the centre column
#pragma unroll
    for (int y = 0; y < BY<R>; ++y) {
      double t0 = 0.0, t1 = 0.0;
#pragma unroll
      for (int b = -R; b <= R; ++b) {
        t0 = fma(P.v[A0][0][R + b], x[y + R][R + b], t0);
        t1 = fma(P.v[A0][0][R + b], x[y + R][R + b + 1], t1);
      }
#pragma unroll
      for (int a = -R; a <= R; ++a) {
        t0 = fma(P.u[A0][1][R + a], x[y + R + a][R], t0);
        t1 = fma(P.u[A0][1][R + a], x[y + R + a][R + 1], t1);
      }
      d[y][0] = t0;
      d[y][1] = t1;
    }
  } else if (mode == PM_DIRECT) {
    // the in-tree comparison (north star (c)): the plane's unfactored (2R+1)^2 sum, W_a0 in u[a0][][]
#pragma unroll
    for (int y = 0; y < BY<R>; ++y) {
      double t0 = 0.0, t1 = 0.0;
#pragma unroll
      for (int a = -R; a <= R; ++a)
#pragma unroll
        for (int b = -R; b <= R; ++b) {
          t0 = fma(P.u[A0][R + a][R + b], x[y + R + a][R + b], t0);
          t1 = fma(P.u[A0][R + a][R + b], x[y + R + a][R + b + 1], t1);
        }
      d[y][0] = t0;
      d[y][1] = t1;
    }
  } else if (mode == PM_PMA1) {
    // radius-1 radially symmetric plane (PMA, eq. 15): one 3x3 rank-1 chain + the centre scalar;
    // palindromic factors with the centre tap of v rescaled to 1 (pma1_unit_centre):
    // T = x0 + v1 (x_-1 + x_+1)
#pragma unroll
    for (int y = 0; y < BY<R>; ++y) {
      d[y][0] = P.w[A0] * x[y + R][R];
      d[y][1] = P.w[A0] * x[y + R][R + 1];
    }
    double T[BY<R> + 2 * R][2];
#pragma unroll
    for (int r = 0; r < BY<R> + 2 * R; ++r) {
      T[r][0] = fma(P.v[A0][0][R + 1], x[r][R - 1] + x[r][R + 1], x[r][R]);
      T[r][1] = fma(P.v[A0][0][R + 1], x[r][R] + x[r][R + 2], x[r][R + 1]);
    }
#pragma unroll
    for (int y = 0; y < BY<R>; ++y) {
      d[y][0] = fma(P.u[A0][0][R + 1], T[y + R - 1][0] + T[y + R + 1][0], fma(P.u[A0][0][R], T[y + R][0], d[y][0]));
      d[y][1] = fma(P.u[A0][0][R + 1], T[y + R - 1][1] + T[y + R + 1][1], fma(P.u[A0][0][R], T[y + R][1], d[y][1]));
    }
  } else {
#pragma unroll
    for (int y = 0; y < BY<R>; ++y) { d[y][0] = 0.0; d[y][1] = 0.0; }
#pragma unroll
    for (int k = 0; k < R3_MAXK; ++k) {
      if (k < P.K[A0]) {
        double T[BY<R> + 2 * R][2];
#pragma unroll
        for (int r = 0; r < BY<R> + 2 * R; ++r) {      // horizontal gather (v-pass)
          double t0 = 0.0, t1 = 0.0;
#pragma unroll
          for (int b = -R; b <= R; ++b) {
            t0 = fma(P.v[A0][k][R + b], x[r][R + b], t0);
            t1 = fma(P.v[A0][k][R + b], x[r][R + b + 1], t1);
          }
          T[r][0] = t0;
          T[r][1] = t1;
        }
#pragma unroll
        for (int y = 0; y < BY<R>; ++y)                 // vertical gather (u-pass)
#pragma unroll
          for (int a = -R; a <= R; ++a) {
            d[y][0] = fma(P.u[A0][k][R + a], T[y + R + a][0], d[y][0]);
            d[y][1] = fma(P.u[A0][k][R + a], T[y + R + a][1], d[y][1]);
          }
      }
    }
  }
#pragma unroll
  for (int y = 0; y < BY<R>; ++y) {
    acc[s1][y][0] += d[y][0];
    acc[s1][y][1] += d[y][1];
  }
  if (A0 < R && (MIR >= 0 ? MIR == 1 : P.mirror[A0] != 0)) {
#pragma unroll
    for (int y = 0; y < BY<R>; ++y) {
      acc[s2][y][0] += d[y][0];
      acc[s2][y][1] += d[y][1];
    }
  }
}

// PM_SYM3 (R = 1, planes 0 and 1 jointly, plane 2 = mirror of plane 0; kernels.hpp sym3_plane):
// d0 (plane 0) goes to output planes z = p and p - 2, d1 (plane 1) to z = p - 1, in the order of the
// per-plane path (plane 0 then its mirror, then plane 1).
template <int I>
__device__ __forceinline__ void apply_sym3(const double (&x)[BY<1> + 2][4], double (&acc)[3][BY<1>][2],
                                           const R3Params& P) {
  double px[BY<1> + 2][2];
#pragma unroll
  for (int r = 0; r < BY<1> + 2; ++r) {
    px[r][0] = x[r][0] + x[r][2];
    px[r][1] = x[r][1] + x[r][3];
  }
  constexpr int s0 = pm(I, 3), s2 = pm(I - 2, 3), s1 = pm(I - 1, 3);
#pragma unroll
  for (int y = 0; y < BY<1>; ++y)
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const double xc = x[y + 1][1 + e];
      const double sv = x[y][1 + e] + x[y + 2][1 + e];
      const double pc = px[y][e] + px[y + 2][e];
      const double ed = px[y + 1][e] + sv;
      const double d0 = fma(P.sym[0][2], pc, fma(P.sym[0][1], ed, P.sym[0][0] * xc));
      acc[s0][y][e] += d0;
      acc[s2][y][e] += d0;
      acc[s1][y][e] = fma(P.sym[1][2], pc, fma(P.sym[1][1], ed, fma(P.sym[1][0], xc, acc[s1][y][e])));   // plane 1 into its slot
    }
}

// Heat-3D signature (R = 1: point planes 0 / 2 mirrored, star plane 1): every contribution goes
// straight into its accumulator through FMAs (8 FP64 ops per point instead of 10 with the products
// and sums formed first); the same formula and order as kernels_rdg3df.cu's planes2.
template <int I>
__device__ __forceinline__ void apply_heat(const double (&x)[BY<1> + 2][4], double (&acc)[3][BY<1>][2],
                                           const R3Params& P) {
  constexpr int s0 = pm(I, 3), s2 = pm(I - 2, 3), s1 = pm(I - 1, 3);
#pragma unroll
  for (int y = 0; y < BY<1>; ++y)
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      acc[s0][y][e] = fma(P.w[0], x[y + 1][1 + e], acc[s0][y][e]);
      acc[s2][y][e] = fma(P.w[0], x[y + 1][1 + e], acc[s2][y][e]);
      double t = acc[s1][y][e];
#pragma unroll
      for (int b = -1; b <= 1; ++b) t = fma(P.v[1][0][1 + b], x[y + 1][1 + e + b], t);
#pragma unroll
      for (int a = -1; a <= 1; ++a) t = fma(P.u[1][1][1 + a], x[y + 1 + a][1 + e], t);
      acc[s1][y][e] = t;
    }
}

template <int R, class SG, int A0, int I>
__device__ __forceinline__ void apply_all(const double (&x)[BY<R> + 2 * R][2 * R + 2],
                                          double (&acc)[2 * R + 1][BY<R>][2], const R3Params& P) {
  if constexpr (R == 1 && SG::m0 == PM_POINT && SG::m1 == PM_STAR && SG::mir == 1) {
    if constexpr (A0 == 0) apply_heat<I>(x, acc, P);
  } else if constexpr (R == 1 && SG::m0 == PM_SYM3) {
    static_assert(SG::m1 == PM_SYM3 && SG::mir == 1, "PM_SYM3 signature");
    if constexpr (A0 == 0) apply_sym3<I>(x, acc, P);
  } else if constexpr (A0 < 2 * R + 1) {
    // specialised modes exist for R = 1 only (plane 0, plane 1, plane 2 == mirror of plane 0)
    constexpr int MODE = R != 1 ? -1 : (A0 == 0 ? SG::m0 : (A0 == 1 ? SG::m1 : (SG::mir == 1 ? SG::m0 : -1)));
    constexpr int MIR = R != 1 ? -1 : SG::mir;
    const bool skip = A0 > R && (MIR >= 0 ? MIR == 1 : P.mirror[2 * R - A0] != 0);
    if (!skip) apply_plane<R, A0, I, MODE, MIR>(x, acc, P);
    apply_all<R, SG, A0 + 1, I>(x, acc, P);
  }
}

template <int R, class SG, bool TMA>
#ifndef RDG3_MINB
#define RDG3_MINB 2   // 2 CTAs x 4 warps: registers for ILP beat occupancy (Box-3D27P 291 -> 368 GS/s)
#endif
__global__ void __launch_bounds__(R3_WARPS * 32, RDG3_MINB) rdg3d_kernel(const double* __restrict__ in, double* __restrict__ out,
                                                                 int64_t N0, int64_t N1, int64_t N2, int nbx, int nby,
                                                                 int nitems, int ZC, int SI, const __grid_constant__ CUtensorMap tmap,
                                                                 const __grid_constant__ R3Params prm,
                                                                 const __grid_constant__ P2PArgs dp) {
  using G = G3<R>;
  constexpr int n = 2 * R + 1;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw) + wl * R3_NS;
  unsigned char* ring = smem_raw + 128 + wl * G::WARP_BYTES;
  const int P0 = (int)(N0 + 2 * R);
  const int64_t P1 = N1 + 2 * R, P2 = N2 + 2 * R;
  const int gw = blockIdx.x * R3_WARPS + wl, TW = gridDim.x * R3_WARPS;
  const int my_items = gw < nitems ? (nitems - 1 - gw) / TW + 1 : 0;
  const int nstages = my_items * SI;
  if (TMA && lane == 0) {
    for (int s = 0; s < R3_NS; ++s) mbar_init(&bars[s], 1);
    fence_barrier_init();
  }
  __syncwarp();
  // item -> (x band, y block, z chunk); producer and consumer walk their stage sequences with
  // incremental counters (one division set per item, none per plane)
  const int nbz = nitems / (nbx * nby);
  auto geom = [&](int item, int& bx0, int& by0, int& bz0) {
    const int bx = item % nbx, rest = item / nbx, by = rest % nby;
    const int bz = dp.active ? p2p_chunk_order(rest / nby, nbz) : rest / nby;
    bx0 = bx * 64;           // padded column of the staged tile origin (= interior column of lane col 0)
    by0 = by * BY<R>;        // padded row of the staged tile origin (= interior row of output row 0)
    bz0 = bz * ZC;           // first padded input plane (= first interior output plane) of the chunk
  };
  int pitem = gw, pj = 0, px = 0, py = 0, pz = 0;
  if (gw < nitems) geom(pitem, px, py, pz);
  // device-initiated exchange: the z-chunk holding the first (last) R interior planes of the slab
  // touches the lower (upper) neighbour (the host keeps it unique per column)
  auto touches = [&](int bz0, bool& lo, bool& hi) {
    // (view padded planes: the chunk's outputs are planes bz0 + R .. bz0 + R + ZC - 1; with a deep-halo
    // view (fused endpoint, remainder launch) only [store_lo, store_hi) are this rank's)
    lo = dp.active && dp.dst_lo != nullptr && bz0 + R < dp.lo_end;
    hi = dp.active && dp.dst_hi != nullptr && int64_t(bz0) + R + ZC > dp.hi_begin;
  };
  auto issue_next = [&](int slot) {
    double* dst = reinterpret_cast<double*>(ring + slot * G::STAGE);
    const int z = pz + pj;
    if (dp.active && pj == 0) {  // this column's halo planes come from a neighbour: wait for them
      bool lo, hi;
      touches(pz, lo, hi);
      if (lane == 0 && (lo || hi)) {
        if (dp.wait_units > 0) {   // the neighbour's previous launch had another geometry (the fused
                                   // kernel before a remainder launch): wait on every unit it signalled
          if (lo) p2p_wait_units(dp.wait_lo, 0, dp.wait_units - 1, dp.wait_val, dp.err);
          if (hi) p2p_wait_units(dp.wait_hi, 0, dp.wait_units - 1, dp.wait_val, dp.err);
        } else {
          const int u = pitem % (nbx * nby), ux = u % nbx, uy = u / nbx;
          for (int yy = max(uy - 1, 0); yy <= min(uy + 1, nby - 1); ++yy) {
            const int u0 = yy * nbx + max(ux - 1, 0), u1 = yy * nbx + min(ux + 1, nbx - 1);
            if (lo) p2p_wait_units(dp.wait_lo, u0, u1, dp.wait_val, dp.err);
            if (hi) p2p_wait_units(dp.wait_hi, u0, u1, dp.wait_val, dp.err);
          }
        }
        fence_proxy_async_global();
      }
      __syncwarp();
    }
    if constexpr (TMA) {
      if (lane == 0) {
        fence_proxy_async();
        mbar_arrive_expect_tx(&bars[slot], G::ROWS * G::BW * 8);
        tma_load_3d(dst, &tmap, px, py, z, &bars[slot]);
      }
    } else {
      for (int i = lane; i < G::ROWS * G::BW; i += 32) {
        const int r = i / G::BW, c = i - r * G::BW;
        const int64_t gy = py + r, gx = px + c;
        if (z < P0 && gy < P1 && gx < P2) cp_async8(dst + i, in + (int64_t(z) * P1 + gy) * P2 + gx);
        else dst[i] = 0.0;
      }
      cp_async_commit();
    }
    if (++pj == SI) {
      pj = 0;
      pitem += TW;
      if (pitem < nitems) geom(pitem, px, py, pz);
    }
  };
  for (int q = 0; q < R3_NS - 1; ++q) {
    if (q < nstages) issue_next(q);
    else if constexpr (!TMA) cp_async_commit();
  }
  double acc[n][BY<R>][2];
  int citem = gw, cj = 0, slot = 0, phase = 0;
  int cz = 0, zend = 0, rowmask = 0;
  double* obase = out;
  bool c0ok = false, c1ok = false, vec = false;
  bool t_lo = false, t_hi = false;
  // consumer: stages in groups of n so that the ring slot of every plane offset is static
  for (int q0 = 0; q0 < nstages; q0 += n) {
    auto one = [&](auto Ic) {
      constexpr int I = decltype(Ic)::value;
      const int q = q0 + I;
      if (q + R3_NS - 1 < nstages) issue_next((slot + R3_NS - 1) % R3_NS);
      else if constexpr (!TMA) cp_async_commit();
      if constexpr (TMA) {
        mbar_wait(&bars[slot], phase);
      } else {
        cp_async_wait<R3_NS - 1>();
        __syncwarp();
      }
      if (cj == 0) {
        int bx0, by0, bz0;
        geom(citem, bx0, by0, bz0);
#pragma unroll
        for (int s = 0; s < n; ++s)
#pragma unroll
          for (int y = 0; y < BY<R>; ++y) { acc[s][y][0] = 0.0; acc[s][y][1] = 0.0; }
        const int col = bx0 + 2 * lane;
        c0ok = col < N2;
        c1ok = col + 1 < N2;
        cz = bz0;
        zend = (int)(int64_t(bz0) + ZC < N0 ? int64_t(bz0) + ZC : N0);
        rowmask = 0;
#pragma unroll
        for (int y = 0; y < BY<R>; ++y) rowmask |= (by0 + y < N1) ? (1 << y) : 0;
        obase = out + (int64_t(R) * P1 + by0 + R) * P2 + R + col;   // (interior z = 0, row by0, column col)
        vec = c0ok && c1ok && ((reinterpret_cast<uintptr_t>(obase) & 15) == 0) && ((P2 & 1) == 0);
        touches(bz0, t_lo, t_hi);
      }
      const double* st = reinterpret_cast<const double*>(ring + slot * G::STAGE);
      double x[BY<R> + 2 * R][2 * R + 2];
#pragma unroll
      for (int r = 0; r < BY<R> + 2 * R; ++r)
#pragma unroll
        for (int m = 0; m <= R; ++m) {
          const double2 t = *reinterpret_cast<const double2*>(st + r * G::BW + 2 * lane + 2 * m);
          x[r][2 * m] = t.x;
          x[r][2 * m + 1] = t.y;
        }
      __syncwarp();  // slot consumed
      apply_all<R, SG, 0, I>(x, acc, prm);
      // output plane zi = (input plane) - 2R is complete: slot (I - 2R) mod n == (I + 1) mod n
      constexpr int s = (I + 1) % n;
      const int zi = cz + cj - 2 * R;
      if (cj >= 2 * R && zi < zend && (!dp.active || (zi + R >= dp.store_lo && zi + R < dp.store_hi))) {
        // the plane goes to this slab and, for the first / last R interior planes of a slab with a
        // neighbour there, into that neighbour's halo as well (peer memory, csrc/dist_p2p.cu)
        const bool rlo = t_lo && zi + R < dp.lo_end, rhi = t_hi && zi + R >= dp.hi_begin;
        const int nd = 1 + (rlo ? 1 : 0) + (rhi ? 1 : 0);
        for (int d = 0; d < nd; ++d) {
          double* o = obase + int64_t(zi) * P1 * P2;
          if (d > 0) o = (rlo && d == 1) ? dp.dst_lo + ((o - out) + dp.off_lo) : dp.dst_hi + ((o - out) + dp.off_hi);
#pragma unroll
          for (int y = 0; y < BY<R>; ++y) {
            if (rowmask & (1 << y)) {
              if (vec) {
                *reinterpret_cast<double2*>(o + int64_t(y) * P2) = make_double2(acc[s][y][0], acc[s][y][1]);
              } else {
                if (c0ok) o[int64_t(y) * P2] = acc[s][y][0];
                if (c1ok) o[int64_t(y) * P2 + 1] = acc[s][y][1];
              }
            }
          }
        }
      }
#pragma unroll
      for (int y = 0; y < BY<R>; ++y) { acc[s][y][0] = 0.0; acc[s][y][1] = 0.0; }
      if (++slot == R3_NS) { slot = 0; phase ^= 1; }
      if (++cj == SI) {
        if (t_lo) p2p_signal_warp(dp.sig_lo, citem % (nbx * nby), dp.sig_val);
        if (t_hi) p2p_signal_warp(dp.sig_hi, citem % (nbx * nby), dp.sig_val);
        cj = 0;
        citem += TW;
      }
    };
    [&]<int... Is>(std::integer_sequence<int, Is...>) {
      (one(std::integral_constant<int, Is>{}), ...);
    }(std::make_integer_sequence<int, n>{});
  }
}

bool make_params3(const Plan& p, R3Params& prm, bool direct = false) {
  std::memset(&prm, 0, sizeof(prm));
  const int R = p.R, n = 2 * R + 1;
  if (p.ndim != 3 || R > 2) return false;
  if (direct) {  // every plane as its plain (2R+1)^2 sum, no plane sharing
    for (int a0 = 0; a0 < n; ++a0) {
      bool any = false;
      for (int i = 0; i < n; ++i)
        for (int j = 0; j < n; ++j) {
          prm.u[a0][i][j] = p.W[(size_t(a0) * n + i) * n + j];
          any = any || prm.u[a0][i][j] != 0.0;
        }
      prm.mode[a0] = any ? PM_DIRECT : PM_NONE;
    }
    return true;
  }
  for (int a0 = 0; a0 < n; ++a0) {
    std::vector<const Term*> ts;
    for (const Term& t : p.terms)
      if (t.plane == a0) ts.push_back(&t);
    if (ts.empty()) { prm.mode[a0] = PM_NONE; continue; }
    if (ts.size() == 1 && ts[0]->kind == kPoint && ts[0]->u[R] == 1.0 && ts[0]->v[R] != 0.0) {
      bool centre = true;
      for (int i = 0; i < n; ++i)
        if (i != R && (ts[0]->u[i] != 0.0 || ts[0]->v[i] != 0.0)) centre = false;
      if (centre) { prm.mode[a0] = PM_POINT; prm.w[a0] = ts[0]->v[R]; continue; }
    }
    if (ts.size() == 2 && ts[0]->kind == kArm && ts[1]->kind == kArm && ts[0]->u[R] == 1.0 && ts[1]->v[R] == 1.0) {
      bool ok = true;
      for (int i = 0; i < n; ++i)
        if (i != R && (ts[0]->u[i] != 0.0 || ts[1]->v[i] != 0.0)) ok = false;
      if (ok) {
        prm.mode[a0] = PM_STAR;
        for (int i = 0; i < n; ++i) { prm.v[a0][0][i] = ts[0]->v[i]; prm.u[a0][1][i] = ts[1]->u[i]; }
        continue;
      }
    }
    if (R == 1 && ts.size() == 2 && ts[0]->kind == kChain && ts[0]->r == 1 && ts[1]->kind == kPoint &&
        ts[1]->r == 0 && ts[1]->u[R] == 1.0 && ts[0]->u[0] == ts[0]->u[2] && ts[0]->v[0] == ts[0]->v[2]) {
      if (pma1_unit_centre(ts[0]->u, ts[0]->v, prm.u[a0][0], prm.v[a0][0])) {
        prm.mode[a0] = PM_PMA1;  // palindromic chain (centre tap of v rescaled to 1) + centre scalar
        prm.w[a0] = ts[1]->v[R];
        continue;
      }
    }
    if ((int)ts.size() > R3_MAXK) return false;
    prm.mode[a0] = PM_CHAINS;
    prm.K[a0] = (int)ts.size();
    for (size_t k = 0; k < ts.size(); ++k)
      for (int i = 0; i < n; ++i) { prm.u[a0][k][i] = ts[k]->u[i]; prm.v[a0][k][i] = ts[k]->v[i]; }
  }
  // z-symmetry per plane pair: identical weights => mirror
  for (int a0 = 0; a0 < R; ++a0) {
    bool same = true;
    for (int e = 0; e < n * n; ++e)
      if (p.W[size_t(a0) * n * n + e] != p.W[size_t(n - 1 - a0) * n * n + e]) { same = false; break; }
    prm.mirror[a0] = same ? 1 : 0;
  }
  if (R == 1 && prm.mode[0] == PM_PMA1 && prm.mode[1] == PM_PMA1 && prm.mirror[0] && sym3_enabled()) {
    double c0, b0, a0_, c1, b1, a1;
    if (sym3_plane(p.W.data(), 0, c0, b0, a0_) && sym3_plane(p.W.data(), 1, c1, b1, a1)) {
      prm.mode[0] = prm.mode[1] = PM_SYM3;
      prm.sym[0][0] = c0; prm.sym[0][1] = b0; prm.sym[0][2] = a0_;
      prm.sym[1][0] = c1; prm.sym[1][1] = b1; prm.sym[1][2] = a1;
    }
  }
  return true;
}

template <int R, class SG, bool TMA>
cudaError_t rdg3d_launch(const Plan& p, const double* src, double* dst, cudaStream_t s, const CUtensorMap& map,
                         const R3Params& prm, const P2PArgs* d) {
  using G = G3<R>;
  int max_grid = 0;
  {
    cudaError_t e = kernel_setup((const void*)rdg3d_kernel<R, SG, TMA>, R3_WARPS * 32, G::SMEM, &max_grid);
    if (e != cudaSuccess) return e;
  }
  if (d && d->prepare_only) return cudaSuccess;
  const int nbx = (int)((p.N[2] + 63) / 64), nby = (int)((p.N[1] + BY<R> - 1) / BY<R>);
  // z-chunk length: the fewest whole rounds of resident warps, then the shortest chunk that fits
  const int64_t TWmax = int64_t(max_grid) * R3_WARPS;
  int64_t zc = R3_ZC;
  {
    const int64_t cols = int64_t(nbx) * nby;
    const int64_t rounds = (cols * ((p.N[0] + zc - 1) / zc) + TWmax - 1) / TWmax;
    const int64_t nch = std::max<int64_t>(1, rounds * TWmax / cols);
    const int64_t zc2 = (p.N[0] + nch - 1) / nch;
    if (zc2 >= 8 && zc2 <= 2 * R3_ZC && cols * ((p.N[0] + zc2 - 1) / zc2) <= rounds * TWmax) zc = zc2;
  }
  if (d && d->active) {
    // device-initiated exchange: exactly one z-chunk per column and side may touch a neighbour — the
    // first chunk holds view planes [R, lo_end), the last one starts at or below hi_begin
    const int64_t N0v = p.N[0], need_lo = d->lo_end - R, need_hi = N0v + R - d->hi_begin;
    zc = std::max<int64_t>(zc, need_lo);
    if (zc < N0v) {
      int64_t ok = 0;
      for (int64_t c = zc; c <= zc + 64 && !ok; ++c) {
        const int64_t rem = N0v % c;
        if ((rem == 0 ? c : rem) >= need_hi) ok = c;
      }
      zc = ok ? ok : N0v;
    }
  }
  const int ZC = (int)zc;
  const int SI = (int)(((ZC + 2 * R) + G::n - 1) / G::n * G::n);
  const int nbz = (int)((p.N[0] + ZC - 1) / ZC);
  const int64_t nitems = int64_t(nbx) * nby * nbz;
  const int grid = (int)std::min<int64_t>(max_grid, (nitems + R3_WARPS - 1) / R3_WARPS);
  static const P2PArgs none{};
  rdg3d_kernel<R, SG, TMA><<<grid, R3_WARPS * 32, G::SMEM, s>>>(src, dst, p.N[0], p.N[1], p.N[2], nbx, nby, (int)nitems,
                                                           ZC, SI, map, prm, d ? *d : none);
  return cudaGetLastError();
}

template <int R>
cudaError_t rdg3d_r(const Plan& p, const double* src, double* dst, cudaStream_t s, bool direct = false,
                    const P2PArgs* d = nullptr) {
  using G = G3<R>;
  R3Params prm;
  if (!make_params3(p, prm, direct)) return cudaErrorNotSupported;
  CUtensorMap map;
  const int64_t padded[3] = {p.P[0], p.P[1], p.P[2]};
  const int box[3] = {1, G::ROWS, G::BW};
  const bool tma = !p.force_no_tma && encode_tmap(&map, src, 3, padded, box);
  if (!tma) std::memset(&map, 0, sizeof(map));
  if constexpr (R == 1) {  // Box-3D27P-like and Heat-3D-like plane signatures
    if (prm.mode[0] == PM_SYM3)
      return tma ? rdg3d_launch<R, Sig3<PM_SYM3, PM_SYM3, 1>, true>(p, src, dst, s, map, prm, d)
                 : rdg3d_launch<R, Sig3<PM_SYM3, PM_SYM3, 1>, false>(p, src, dst, s, map, prm, d);
    if (prm.mode[0] == PM_PMA1 && prm.mode[1] == PM_PMA1 && prm.mirror[0])
      return tma ? rdg3d_launch<R, Sig3<PM_PMA1, PM_PMA1, 1>, true>(p, src, dst, s, map, prm, d)
                 : rdg3d_launch<R, Sig3<PM_PMA1, PM_PMA1, 1>, false>(p, src, dst, s, map, prm, d);
    if (prm.mode[0] == PM_POINT && prm.mode[1] == PM_STAR && prm.mirror[0])
      return tma ? rdg3d_launch<R, Sig3<PM_POINT, PM_STAR, 1>, true>(p, src, dst, s, map, prm, d)
                 : rdg3d_launch<R, Sig3<PM_POINT, PM_STAR, 1>, false>(p, src, dst, s, map, prm, d);
  }
  return tma ? rdg3d_launch<R, Sig3<-1, -1, -1>, true>(p, src, dst, s, map, prm, d)
             : rdg3d_launch<R, Sig3<-1, -1, -1>, false>(p, src, dst, s, map, prm, d);
}

}  // namespace

cudaError_t launch_direct3d_stream(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  switch (p.R) {
    case 1: return rdg3d_r<1>(p, src, dst, s, true);
    case 2: return rdg3d_r<2>(p, src, dst, s, true);
  }
  return cudaErrorNotSupported;
}

int rdg3d_p2p_units(const Plan& p, int* nux) {
  R3Params prm;
  const bool direct = p.engine == LORA_ENGINE_DIRECT;
  if (p.ndim != 3 || p.R > 2 || (p.engine != LORA_ENGINE_RDG_CUDA && !direct) || !make_params3(p, prm, direct)) return 0;
  const int bx = (int)((p.N[2] + 63) / 64), by = (int)((p.N[1] + (p.R == 1 ? BY<1> : BY<2>) - 1) / (p.R == 1 ? BY<1> : BY<2>));
  if (nux) *nux = bx;
  return bx * by;
}

cudaError_t launch_rdg3d_p2p(const Plan& p, const double* src, double* dst, cudaStream_t s, const P2PArgs& d) {
  const bool direct = p.engine == LORA_ENGINE_DIRECT;
  switch (p.R) {
    case 1: return rdg3d_r<1>(p, src, dst, s, direct, &d);
    case 2: return rdg3d_r<2>(p, src, dst, s, direct, &d);
  }
  return cudaErrorNotSupported;
}

bool rdg3d_supported(const Plan& p) {
  R3Params prm;
  return make_params3(p, prm);
}

cudaError_t launch_rdg3d(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  switch (p.R) {
    case 1: return rdg3d_r<1>(p, src, dst, s);
    case 2: return rdg3d_r<2>(p, src, dst, s);
  }
  return cudaErrorNotSupported;
}

}  // namespace lora
