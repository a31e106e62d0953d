// Exact temporal fusion of K = 2 or 3 3D time steps (SURVEY NEXT-2 "2.5D blocking") for the
// radius-1 Alg. 2 CUDA-core engine.
//
// A CTA (8 warps) owns a column of the domain: 64 lane columns x 16 step-1 rows (14 final rows),
// streaming along z through a chunk of ZC final planes.  For every input plane p (TMA 3D box
// 18 x 66, 3- or 4-stage ring; zero fill outside the array):
//   stage 1: warp w applies the plane operators (Alg. 2: PMA / star / point-wise / general rank-1
//            chains per plane; the two symmetric planes of Box-3D27P jointly on shared class sums,
//            PM_SYM3, Q18) to produce step-1 rows 2w, 2w+1 and scatters them into a register
//            z-ring of 3 step-1 planes; the completed step-1 plane p-1 gets the fixed Dirichlet halo
//            re-imposed and is written to a shared plane buffer (double-buffered);
//   one __syncthreads;
//   stage 2: warps 0..6 apply the same operators to that step-1 plane (final rows 2w, 2w+1) into a
//            second z-ring; the completed final plane p-2 is stored.
// Every point goes through the same arithmetic as two unfused steps of kernels_rdg3d.cu's mode
// code (bitwise equal to two unfused steps), so the result equals two steps to rounding; halo handling makes it exact
// temporal blocking (reading Q5).  The lane columns lose one valid column per side per
// fused step: x bands overlap with stride 60 (even TMA origin).
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

#ifndef RDG3F_NS
#define RDG3F_NS 0   // TMA ring stages; 0: per signature (f_ns)
#endif
#ifndef RDG3F_LAG
#define RDG3F_LAG 0   // 1: stage S consumes the plane stage S-1 published in the PREVIOUS iteration (one
#endif                // CTA barrier at the end of the iteration, the stages of an iteration independent).
                      // Measured slower (r02m, same box): Box-3D27P k = 2 393 -> 379 GS/s, Heat-3D 449 -> 416
constexpr int F_LAG = RDG3F_LAG;
#ifndef RDG3F_DECOUPLE
#define RDG3F_DECOUPLE 0   // 1 (K = 2, TMA): mbarrier hand-offs between the stages instead of one CTA barrier
#endif                     // per plane.  Measured slower (r02ze, same box): Box-3D27P 447 -> 428, Heat-3D 483 -> 448
#ifndef RDG3F_HALO_Z
#define RDG3F_HALO_Z 1   // stage-1 Dirichlet fetch with the x/y masks precomputed per item (halo_fetch_z)
#endif
#ifndef RDG3F_WARPS
#define RDG3F_WARPS 8
#endif
constexpr int F_WARPS = RDG3F_WARPS;
constexpr int F_S1 = 2 * F_WARPS;    // stage-1 rows per CTA column (2 per warp); stage s: F_S1 - 2(s-1)
constexpr int F_IN = F_S1 + 2;       // staged input rows
constexpr int F_BW = 66;             // staged columns (64 + 2R)
constexpr int F_S1W = 72;            // step-1 plane buffer row pitch (doubles): data at [1, 65)
#ifndef RDG3F_ZC
#define RDG3F_ZC 64   // z-chunk length (final planes per work item; balanced per grid)
#endif
constexpr int F_ZC = RDG3F_ZC;

enum { PM_NONE = 0, PM_POINT = 1, PM_CHAINS = 2, PM_STAR = 3, PM_PMA1 = 4, PM_SYM3 = 6 };   // (values as in kernels_rdg3d.cu)
constexpr int F_MAXK = 3;

struct FParams {
  int mode[3], K[3], mirror[3];
  double w[3];
  double u[3][F_MAXK][3], v[3][F_MAXK][3];
  double sym[2][3];   // PM_SYM3 (planes 0 and 1 jointly): centre c, edge b, corner a (kernels.hpp sym3_plane)
};

__host__ __device__ constexpr int pm3(int a) { return ((a % 3) + 3) % 3; }

// Plane operator A0 on 2 output rows: rows 0..3 of `x` (4 consecutive input rows, 4 columns each:
// the lane's 2 columns +-1) -> d[2][2].  Same arithmetic as kernels_rdg3d.cu's apply_plane (R = 1).
template <int A0, int MODE>
__device__ __forceinline__ bool plane2(const double (&x)[4][4], const FParams& P, double (&d)[2][2]) {
  const int mode = MODE >= 0 ? MODE : P.mode[A0];  // MODE >= 0: the kernel is specialised on it
  if (mode == PM_NONE) return false;
  if (mode == PM_POINT) {
#pragma unroll
    for (int y = 0; y < 2; ++y) { d[y][0] = P.w[A0] * x[y + 1][1]; d[y][1] = P.w[A0] * x[y + 1][2]; }
  } else if (mode == PM_STAR) {
#pragma unroll
    for (int y = 0; y < 2; ++y) {
      double t0 = 0.0, t1 = 0.0;
#pragma unroll
      for (int b = -1; b <= 1; ++b) {
        t0 = fma(P.v[A0][0][1 + b], x[y + 1][1 + b], t0);
        t1 = fma(P.v[A0][0][1 + b], x[y + 1][2 + b], t1);
      }
#pragma unroll
      for (int a = -1; a <= 1; ++a) {
        t0 = fma(P.u[A0][1][1 + a], x[y + 1 + a][1], t0);
        t1 = fma(P.u[A0][1][1 + a], x[y + 1 + a][2], t1);
      }
      d[y][0] = t0; d[y][1] = t1;
    }
  } else if (mode == PM_PMA1) {
    // factors with v[1] == 1 (pma1_unit_centre): T = x_0 + v[2] (x_-1 + x_+1)
    double T[4][2];
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      T[r][0] = fma(P.v[A0][0][2], x[r][0] + x[r][2], x[r][1]);
      T[r][1] = fma(P.v[A0][0][2], x[r][1] + x[r][3], x[r][2]);
    }
#pragma unroll
    for (int y = 0; y < 2; ++y) {
      d[y][0] = fma(P.u[A0][0][2], T[y][0] + T[y + 2][0], fma(P.u[A0][0][1], T[y + 1][0], P.w[A0] * x[y + 1][1]));
      d[y][1] = fma(P.u[A0][0][2], T[y][1] + T[y + 2][1], fma(P.u[A0][0][1], T[y + 1][1], P.w[A0] * x[y + 1][2]));
    }
  } else {
#pragma unroll
    for (int y = 0; y < 2; ++y) { d[y][0] = 0.0; d[y][1] = 0.0; }
#pragma unroll
    for (int k = 0; k < F_MAXK; ++k) {
      if (k < P.K[A0]) {
        double T[4][2];
#pragma unroll
        for (int r = 0; r < 4; ++r) {
          double t0 = 0.0, t1 = 0.0;
#pragma unroll
          for (int b = -1; b <= 1; ++b) {
            t0 = fma(P.v[A0][k][1 + b], x[r][1 + b], t0);
            t1 = fma(P.v[A0][k][1 + b], x[r][2 + b], t1);
          }
          T[r][0] = t0; T[r][1] = t1;
        }
#pragma unroll
        for (int y = 0; y < 2; ++y)
#pragma unroll
          for (int a = -1; a <= 1; ++a) {
            d[y][0] = fma(P.u[A0][k][1 + a], T[y + 1 + a][0], d[y][0]);
            d[y][1] = fma(P.u[A0][k][1 + a], T[y + 1 + a][1], d[y][1]);
          }
      }
    }
  }
  return true;
}

// Mode signature of a specialised kernel: modes of planes 0 and 1 (-1 = read at run time) and
// whether plane 2 mirrors plane 0 (-1 = read at run time).
template <int M0, int M1, int MIR>
struct Sig3 {
  static constexpr int m0 = M0, m1 = M1, mir = MIR;
  // TMA ring stages: 4 for the light point + star (Heat-3D) kernel (420 -> 430 GS/s), 3 otherwise
  // (Box-3D27P: 392 with 3, 388 with 4; tools/gpu_variants.sh, same box)
  // and the joint symmetric planes (Box-3D27P: 447 with 3, 456 with 4; r02zh)
  static constexpr int ns = RDG3F_NS > 0 ? RDG3F_NS : (((M0 == 1 && M1 == 3) || M0 == PM_SYM3) ? 4 : 3);
  // plane 0 statically non-empty and its result an FMA chain: its contribution assigns (a bare
  // product, PM_POINT, would let nvcc contract it with the next addition into one FMA, which the
  // unfused kernel's 0 + w x does not: results would differ from two single steps in the last bit)
  static constexpr bool assign0 = M0 > 0 && M0 != 1 /* PM_POINT */;
};

// All plane operators of one input plane (ring position I) into a z-ring of 3 planes x 2 rows.
// PM_SYM3: both operators jointly on the shared class sums, in the order of kernels_rdg3d.cu's
// apply_sym3 (plane 0 assigned to its slot, added to the mirror slot; plane 1 added).
template <class SG, int I, int A0>
__device__ __forceinline__ void planes2(const double (&x)[4][4], const FParams& P, double (&acc)[3][2][2]) {
  if constexpr (SG::m0 == PM_POINT && SG::m1 == PM_STAR && SG::mir == 1) {
    // Heat-3D: every contribution straight into its accumulator (kernels_rdg3d.cu apply_heat)
    if constexpr (A0 == 0) {
      constexpr int s0 = pm3(I), s2 = pm3(I - 2), s1 = pm3(I - 1);
#pragma unroll
      for (int y = 0; y < 2; ++y)
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
  } else if constexpr (SG::m0 == PM_SYM3) {
    static_assert(SG::m1 == PM_SYM3 && SG::mir == 1 && SG::assign0, "PM_SYM3 signature");
    if constexpr (A0 == 0) {
      double px[4][2];
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        px[r][0] = x[r][0] + x[r][2];
        px[r][1] = x[r][1] + x[r][3];
      }
      constexpr int s0 = pm3(I), s2 = pm3(I - 2), s1 = pm3(I - 1);
#pragma unroll
      for (int y = 0; y < 2; ++y)
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const double xc = x[y + 1][1 + e];
          const double sv = x[y][1 + e] + x[y + 2][1 + e];
          const double pc = px[y][e] + px[y + 2][e];
          const double ed = px[y + 1][e] + sv;
          const double d0 = fma(P.sym[0][2], pc, fma(P.sym[0][1], ed, P.sym[0][0] * xc));
          acc[s0][y][e] = d0;
          acc[s2][y][e] += d0;
          acc[s1][y][e] = fma(P.sym[1][2], pc, fma(P.sym[1][1], ed, fma(P.sym[1][0], xc, acc[s1][y][e])));   // plane 1 into its slot
        }
    }
  } else if constexpr (A0 < 3) {
    const bool mirror = SG::mir >= 0 ? SG::mir == 1 : P.mirror[0] != 0;
    constexpr int MODE = A0 == 0 ? SG::m0 : (A0 == 1 ? SG::m1 : (SG::mir == 1 ? SG::m0 : -1));
    if (!(A0 == 2 && mirror)) {
      double d[2][2];
      if (plane2<A0, MODE>(x, P, d)) {
        constexpr int s1 = pm3(I - A0);
        if constexpr (A0 == 0 && SG::assign0) {
          // plane 0's contribution is the first one its output plane receives (the slot was
          // emitted after input plane I - 1): assigned, so emitted slots need no zeroing
#pragma unroll
          for (int y = 0; y < 2; ++y) { acc[s1][y][0] = d[y][0]; acc[s1][y][1] = d[y][1]; }
        } else {
#pragma unroll
          for (int y = 0; y < 2; ++y) { acc[s1][y][0] += d[y][0]; acc[s1][y][1] += d[y][1]; }
        }
        if (A0 == 0 && mirror) {
          constexpr int s2 = pm3(I - 2);
#pragma unroll
          for (int y = 0; y < 2; ++y) { acc[s2][y][0] += d[y][0]; acc[s2][y][1] += d[y][1]; }
        }
      }
    }
    planes2<SG, I, A0 + 1>(x, P, acc);
  }
}

__device__ __forceinline__ void load_rows(const double* __restrict__ base, int pitch, int lane, double (&x)[4][4]) {
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const double2 a = *reinterpret_cast<const double2*>(base + r * pitch + 2 * lane);
    const double2 b = *reinterpret_cast<const double2*>(base + r * pitch + 2 * lane + 2);
    x[r][0] = a.x; x[r][1] = a.y; x[r][2] = b.x; x[r][3] = b.y;
  }
}

// Intermediate stage S (1 <= S < K): the stage-S plane just completed in acc[S-1] (ring slot CS)
// gets the fixed Dirichlet halo re-imposed and is published to its shared plane buffer.
// ZERO: clear the emitted slot (not needed when plane 0's contribution assigns, Sig3::assign0).
// The Dirichlet values a slow-path publish substitutes for the lane's 4 elements of the stage-S
// row pair at plane zs: bit 2y+e of the result set = element replaced by hv[y][e] (the input's halo
// value, or 0 outside the array).  Issued at the start of the plane so the global loads overlap the
// plane's arithmetic instead of stalling the shared-memory stores of publish.
template <int K, int S>
__device__ __forceinline__ unsigned halo_fetch(int w, int lane, int Y0, int X0, int zs, int P0, int P1, int P2,
                                               const double* __restrict__ in, double (&hv)[2][2]) {
  const int c0 = 2 * lane;
  unsigned m = 0;
#pragma unroll
  for (int y = 0; y < 2; ++y) {
    const int gy = Y0 - (K - S) + 2 * w + y;  // padded row of this stage-S row
    const bool zin = zs >= 0 && zs < P0, yin = gy >= 0 && gy < P1;
    const bool zh = zs < 1 || zs >= P0 - 1, yh = gy < 1 || gy >= P1 - 1;
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const int cx = X0 + c0 + e;
      const bool xin = cx >= 0 && cx < P2, xh = cx < 1 || cx >= P2 - 1;
      const bool inside = zin && yin && xin, halo = inside && (zh || yh || xh);
      hv[y][e] = halo ? in[(int64_t(zs) * P1 + gy) * P2 + cx] : 0.0;
      if (!inside || halo) m |= 1u << (2 * y + e);
    }
  }
  return m;
}

// The same with the x/y part precomputed per item (halo_xy: in_xy = elements inside the array's
// x/y range, hal_xy = those of them on the x/y Dirichlet ring; base = the element (0, 0) offset
// gy * P2 + cx within a plane): per plane only the z tests and the loads of flagged elements.
__device__ __forceinline__ unsigned halo_fetch_z(int zs, int P0, int64_t P12, int P2, unsigned in_xy, unsigned hal_xy,
                                                 int64_t base, const double* __restrict__ in, double (&hv)[2][2]) {
  const bool zin = zs >= 0 && zs < P0, zh = zs < 1 || zs >= P0 - 1;
  const unsigned ld = zin ? (zh ? in_xy : hal_xy) : 0u;        // elements taking an input value
  const double* src = in + (int64_t(zs) * P12 + base);
#pragma unroll
  for (int y = 0; y < 2; ++y)
#pragma unroll
    for (int e = 0; e < 2; ++e) hv[y][e] = ((ld >> (2 * y + e)) & 1u) ? src[y * P2 + e] : 0.0;
  return zin ? ((~in_xy | ld) & 0xFu) : 0xFu;                  // outside the array: every element is 0
}

// fast: every element of the lane is strictly inside the array (hm == 0): plain stores; otherwise
// the elements flagged in hm take the prefetched Dirichlet values hv (halo_fetch).
template <int K, int S, int CS, bool ZERO = true>
__device__ __forceinline__ void publish(double (&acc)[K][3][2][2], double* __restrict__ buf, int w, int lane,
                                        unsigned hm, const double (&hv)[2][2]) {
  const int c0 = 2 * lane;
#pragma unroll
  for (int y = 0; y < 2; ++y) {
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const double v = acc[S - 1][CS][y][e];
      buf[(2 * w + y) * F_S1W + 1 + c0 + e] = ((hm >> (2 * y + e)) & 1u) ? hv[y][e] : v;
      if constexpr (ZERO) acc[S - 1][CS][y][e] = 0.0;
    }
  }
}

// K = 3: the Dirichlet values are loaded in place (a prefetch would cost registers the K = 3
// kernel does not have; fast: the lane's elements are strictly inside, plain stores).
template <int K, int S, int CS, bool ZERO = true>
__device__ __forceinline__ void publish_ip(double (&acc)[K][3][2][2], double* __restrict__ buf, int w, int lane,
                                        int Y0, int X0, int zs, int P0, int P1, int P2,
                                        const double* __restrict__ in, bool fast) {
  const int c0 = 2 * lane;
  if (fast) {
#pragma unroll
    for (int y = 0; y < 2; ++y) {
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        buf[(2 * w + y) * F_S1W + 1 + c0 + e] = acc[S - 1][CS][y][e];
        if constexpr (ZERO) acc[S - 1][CS][y][e] = 0.0;
      }
    }
    return;
  }
#pragma unroll
  for (int y = 0; y < 2; ++y) {
    double v[2] = {acc[S - 1][CS][y][0], acc[S - 1][CS][y][1]};
    if constexpr (ZERO) { acc[S - 1][CS][y][0] = 0.0; acc[S - 1][CS][y][1] = 0.0; }
    const int gy = Y0 - (K - S) + 2 * w + y;  // padded row of this stage-S row
    const bool zin = zs >= 0 && zs < P0, yin = gy >= 0 && gy < P1;
    const bool zh = zs < 1 || zs >= P0 - 1, yh = gy < 1 || gy >= P1 - 1;
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const int cx = X0 + c0 + e;
      const bool xin = cx >= 0 && cx < P2, xh = cx < 1 || cx >= P2 - 1;
      double t = v[e];
      if (!(zin && yin && xin)) t = 0.0;
      else if (zh || yh || xh) t = in[(int64_t(zs) * P1 + gy) * P2 + cx];
      buf[(2 * w + y) * F_S1W + 1 + c0 + e] = t;
    }
  }
}

// K fused steps (K = 2, 3).  Stage s computes 16 - 2(s-1) rows (warps w < 8 - (s-1)); final rows
// TY = 16 - 2(K-1); one __syncthreads per stage boundary per plane.
template <class SG, int K, bool TMA, bool P2P>
#ifndef RDG3F_MINB
#define RDG3F_MINB 2
#endif
__global__ void __launch_bounds__(F_WARPS * 32, RDG3F_MINB) rdg3df_kernel(const double* __restrict__ in, double* __restrict__ out,
                                                                 int64_t N0, int64_t N1, int64_t N2, int nbx, int nby,
                                                                 int nitems, int ZC, int SI,
                                                                 const __grid_constant__ CUtensorMap tmap,
                                                                 const __grid_constant__ FParams prm,
                                                                 const __grid_constant__ P2PArgs dp) {
  constexpr int STAGE = ((F_IN * F_BW * 8 + 127) / 128) * 128;
  constexpr int F_NS = SG::ns;
  constexpr int S1B = F_S1 * F_S1W;          // doubles per intermediate plane buffer
  constexpr int TY = F_S1 - 2 * (K - 1);     // final rows per CTA column
  constexpr int SG1 = (K - 1) & 1;           // keeps the staged x origin even
  constexpr int BS = 64 - 2 * (K - 1) - 2 * SG1;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem_raw);
  unsigned char* ring = smem_raw + 128;
  double* sbuf = reinterpret_cast<double*>(smem_raw + 128 + F_NS * STAGE);  // [K-1][2][F_S1][F_S1W]
  // the warp index through a shuffle: ptxas then knows it is warp-uniform (warp-0-only branches stay
  // uniform, and the weights keep their uniform registers)
  const int tid = threadIdx.x, lane = tid & 31, w = __shfl_sync(0xffffffffu, tid >> 5, 0);
  const int P0 = (int)(N0 + 2), P1 = (int)(N1 + 2), P2 = (int)(N2 + 2);
  for (int i = tid; i < 2 * (K - 1) * S1B; i += blockDim.x) sbuf[i] = 0.0;   // margins stay zero
  const int my_items = blockIdx.x < nitems ? (nitems - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const int nstages = my_items * SI;
  // DEC (K = 2, TMA): the stages hand planes over through mbarriers instead of a CTA barrier per plane
  // (ncu: 16 % of the warps' stall samples sat at that barrier; warp 7 has no stage-2 rows and the
  // stage-2 warps waited for each other): slot_free[s] — every warp has read input slot s (warp 0 then
  // refills it); pub[par] — every warp has published its stage-1 rows of the plane buffer of parity
  // par; cons[par] — the stage-2 warps have read that buffer (stage 1 may overwrite it two planes later)
  constexpr bool DEC = RDG3F_DECOUPLE && K == 2 && TMA && !F_LAG;
  static_assert(!DEC || 3 * F_NS + 4 <= 16, "mbarrier area");
  uint64_t* slot_free = bar + F_NS;
  uint64_t* pub = bar + 2 * F_NS;
  uint64_t* cons = pub + 2;
  if (TMA && tid == 0) {
    for (int s = 0; s < F_NS; ++s) mbar_init(&bar[s], 1);
    if constexpr (DEC) {
      for (int s = 0; s < F_NS; ++s) mbar_init(&slot_free[s], F_WARPS);
      for (int b = 0; b < 2; ++b) { mbar_init(&pub[b], F_WARPS); mbar_init(&cons[b], F_S1 / 2 - 1); }
    }
    fence_barrier_init();
  }
  __syncthreads();
  // item -> lane column 0 at padded X0, final rows from padded Y0, final planes from padded Z0
  const int nbz = nitems / (nbx * nby);
  // P2P: the instantiation with the exchange hooks (single-GPU launches use P2P = false: no hook code)
  const bool act = P2P && dp.active;
  auto geom = [&](int item, int& X0, int& Y0, int& Z0) {
    const int bx = item % nbx, rest = item / nbx, by = rest % nby;
    const int bz = act ? p2p_chunk_order(rest / nby, nbz) : rest / nby;
    X0 = 1 + bx * BS - (K - 1) - SG1;   // R + b*BS - R(K-1) - SG   (X0 - R even)
    Y0 = 1 + by * TY;
    Z0 = 1 + bz * ZC;
  };
  // device-initiated exchange (csrc/dist_p2p.cu; the launch sees the slab buffer as a taller "view"
  // whose deep-halo planes count as interior): the z-chunk holding the slab's first (last) H own
  // planes touches the lower (upper) neighbour — it waits for the neighbour's step counter of the
  // 3 x 3 units around its column before staging, stores those planes into the neighbour's halo as
  // well, and publishes its own counter when done.  The host keeps that chunk unique per column.
  auto touches = [&](int Z0_, bool& lo, bool& hi) {
    lo = act && dp.dst_lo != nullptr && Z0_ < dp.lo_end;
    hi = act && dp.dst_hi != nullptr && Z0_ + ZC > dp.hi_begin;
  };
  int pitem = blockIdx.x, pj = 0, pX = 0, pY = 0, pZ = 0;
  if (pitem < nitems) geom(pitem, pX, pY, pZ);
  auto issue_next = [&](int slot) {
    double* dst = reinterpret_cast<double*>(ring + slot * STAGE);
    const int x = pX - 1, y = pY - K, z = pZ - K + pj;
    if (act && pj == 0 && w == 0) {   // this column's halo planes come from a neighbour (warp 0,
      bool lo, hi;                     // warp-uniform wait: kernels.hpp / p2p.cuh p2p_wait_units_warp)
      touches(pZ, lo, hi);
      if (lo || hi) {
        if (dp.wait_units > 0) {   // the neighbour's previous launch had another geometry: every unit
          if (lo) p2p_wait_units_warp(dp.wait_lo, 0, dp.wait_units - 1, dp.wait_val, dp.err);
          if (hi) p2p_wait_units_warp(dp.wait_hi, 0, dp.wait_units - 1, dp.wait_val, dp.err);
        } else {
          const int u = pitem % (nbx * nby), ux = u % nbx, uy = u / nbx;
          for (int yy = max(uy - 1, 0); yy <= min(uy + 1, nby - 1); ++yy) {
            const int u0 = yy * nbx + max(ux - 1, 0), u1 = yy * nbx + min(ux + 1, nbx - 1);
            if (lo) p2p_wait_units_warp(dp.wait_lo, u0, u1, dp.wait_val, dp.err);
            if (hi) p2p_wait_units_warp(dp.wait_hi, u0, u1, dp.wait_val, dp.err);
          }
        }
        if (lane == 0) fence_proxy_async_global();
      }
    }
    // warp 0 reconverges here: lane 0 may have spun above, and the CTA barriers that follow are
    // .aligned (a diverged warp 0 would let lane 0 run on alone and deadlock at the next __syncwarp)
    if (act) __syncwarp();
    if constexpr (TMA) {  // x even by construction; negative origins are zero-filled by TMA
      if (tid == 0) {
        fence_proxy_async();
        mbar_arrive_expect_tx(&bar[slot], F_IN * F_BW * 8);
        tma_load_3d(dst, &tmap, x, y, z, &bar[slot]);
      }
    } else {  // no TMA (row pitch not a multiple of 16 B): the CTA fills the box itself
      if (act && pj == 0) __syncthreads();   // after tid 0's wait for the neighbour
      for (int i = tid; i < F_IN * F_BW; i += blockDim.x) {
        const int r = i / F_BW, c = i - r * F_BW;
        const int gy = y + r, gx = x + c;
        dst[i] = (z >= 0 && z < P0 && gy >= 0 && gy < P1 && gx >= 0 && gx < P2)
                     ? __ldg(in + (int64_t(z) * P1 + gy) * P2 + gx) : 0.0;
      }
      __syncthreads();
    }
    if (++pj == SI) {
      pj = 0;
      pitem += gridDim.x;
      if (pitem < nitems) geom(pitem, pX, pY, pZ);
    }
  };
  // prologue (uniform across the CTA: issue_next may contain __syncthreads)
  for (int q = 0; q < F_NS - 1; ++q)
    if (q < nstages) issue_next(q);
  __shared__ unsigned sig_count;   // warps done with the current boundary item (P2P signal)
  if (tid == 0) sig_count = 0u;
  double acc[K][3][2][2];
  int citem = blockIdx.x, cj = 0, slot = 0, phase = 0;
  int X0 = 0, Y0 = 0, Z0 = 0, zend = 0;
  bool t_lo = false, t_hi = false;   // the current item touches the lower / upper neighbour
  const int c0 = 2 * lane;  // lane's first column (relative to X0)
  // per item: intermediate stage S rows/columns of this lane strictly inside (publish fast path);
  // final elements of this lane to store (row / column validity, the z test is per plane)
  bool xy_in[K > 1 ? K - 1 : 1];
  unsigned in_xy1 = 0u, hal_xy1 = 0u;   // stage 1 (K = 2): halo_fetch_z's per-item x/y masks and offset
  int64_t base1 = 0;
  bool st_ok[2][2];
  for (int q0 = 0; q0 < nstages; q0 += 3) {
    auto one = [&](auto Ic) {
      constexpr int I = decltype(Ic)::value;
      const int q = q0 + I;
      if (TMA) mbar_wait(&bar[slot], phase);
      else __syncthreads();
      if (cj == 0) {
        geom(citem, X0, Y0, Z0);
        zend = min(Z0 + ZC, act ? dp.store_hi : P0 - 1);
        touches(Z0, t_lo, t_hi);
        const bool xs_in = X0 + c0 >= 1 && X0 + c0 + 1 < P2 - 1;
#pragma unroll
        for (int S = 1; S < K; ++S) {
          const int gy = Y0 - (K - S) + 2 * w;
          xy_in[S - 1] = xs_in && gy >= 1 && gy + 1 < P1 - 1;
        }
        if constexpr (K == 2) {
          in_xy1 = hal_xy1 = 0u;
          const int gy0 = Y0 - 1 + 2 * w;
          base1 = int64_t(gy0) * P2 + X0 + c0;
#pragma unroll
          for (int y = 0; y < 2; ++y)
#pragma unroll
            for (int e = 0; e < 2; ++e) {
              const int gy = gy0 + y, cx = X0 + c0 + e;
              const bool in_ = gy >= 0 && gy < P1 && cx >= 0 && cx < P2;
              const bool h_ = in_ && (gy < 1 || gy >= P1 - 1 || cx < 1 || cx >= P2 - 1);
              in_xy1 |= (in_ ? 1u : 0u) << (2 * y + e);
              hal_xy1 |= (h_ ? 1u : 0u) << (2 * y + e);
            }
        }
#pragma unroll
        for (int y = 0; y < 2; ++y) {
          const int gy = Y0 + 2 * w + y;
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int cx = X0 + c0 + e;
            st_ok[y][e] = gy < P1 - 1 && gy < Y0 + TY && c0 + e >= K - 1 && c0 + e < 65 - K && cx >= 1 && cx < P2 - 1;
          }
        }
#pragma unroll
        for (int k = 0; k < K; ++k)
#pragma unroll
          for (int s = 0; s < 3; ++s)
#pragma unroll
            for (int y = 0; y < 2; ++y) { acc[k][s][y][0] = 0.0; acc[k][s][y][1] = 0.0; }
      }
      const int p = Z0 - K + cj;  // padded input plane
      const int par = q & 1;
      // ---------------- stage 1: rows 2w, 2w+1 (16 rows) from input tile rows 2w .. 2w+3
      {
        const double* st = reinterpret_cast<const double*>(ring + slot * STAGE);
        // K = 2: the Dirichlet values are fetched before the plane's arithmetic (their latency hides
        // behind it: Heat-3D 431 -> 452 GS/s); K = 3 has no registers to spare (spills), fetches late
        const bool fast1 = xy_in[0] && p - 1 >= 1 && p - 1 < P0 - 1;
        double hv[2][2];
        unsigned hm = 0;
#if RDG3F_HALO_Z
        if (K == 2 && !fast1) hm = halo_fetch_z(p - 1, P0, int64_t(P1) * P2, P2, in_xy1, hal_xy1, base1, in, hv);
#else
        if (K == 2 && !fast1) hm = halo_fetch<K, 1>(w, lane, Y0, X0, p - 1, P0, P1, P2, in, hv);
#endif
        double x[4][4];
        load_rows(st + (2 * w) * F_BW, F_BW, lane, x);
        if constexpr (DEC) {   // this warp is done with the input slot
          __syncwarp();
          if (lane == 0) mbar_arrive(&slot_free[slot]);
        }
        planes2<SG, I, 0>(x, prm, acc[0]);
        if constexpr (DEC) {   // the stage-2 warps have read this parity's buffer two planes ago
          if (q >= 2) mbar_wait(&cons[par], ((q >> 1) + 1) & 1);
        }
        if constexpr (K == 2)
          publish<K, 1, (I + 1) % 3, !SG::assign0>(acc, sbuf + (0 * 2 + par) * S1B, w, lane, hm, hv);
        else
          publish_ip<K, 1, (I + 1) % 3, !SG::assign0>(acc, sbuf + (0 * 2 + par) * S1B, w, lane, Y0, X0, p - 1, P0, P1, P2, in,
                                                      fast1);
      }
      if constexpr (DEC) {
        __syncwarp();
        if (lane == 0) mbar_arrive(&pub[par]);   // my stage-1 rows of this plane are in the buffer
        if (w == 0 && q + F_NS - 1 < nstages) {  // refill the slot of plane q - 1 once every warp read it
          const int ps = (slot + F_NS - 1) % F_NS;
          if (q >= 1) mbar_wait(&slot_free[ps], ((q - 1) / F_NS) & 1);
          issue_next(ps);
        }
        mbar_wait(&pub[par], (q >> 1) & 1);      // every warp's stage-1 rows of this plane
      } else if constexpr (!F_LAG) {
        __syncthreads();  // stage-1 plane visible; every warp is done with the input slot
        if (q + F_NS - 1 < nstages) issue_next((slot + F_NS - 1) % F_NS);
      }
      // ---------------- stages 2 .. K (F_LAG: stage S runs L = S - 1 iterations behind stage 1 and
      // reads the plane stage S-1 published in the previous iteration, from the other parity buffer)
      auto stage = [&](auto Sc) {
        constexpr int S = decltype(Sc)::value;
        constexpr int LG = F_LAG ? S - 1 : 0;                  // iterations stage S lags stage 1
        constexpr int IS = pm3(I - (S - 1) - LG);              // ring position of the stage-(S-1) plane consumed
        const bool active = w < F_S1 / 2 - (S - 1) && cj >= 2 * (S - 1) + LG;
        const int rpar = F_LAG ? (par ^ 1) : par;              // parity of the buffer stage S reads
        if (active) {
          const double* Sb = sbuf + ((S - 2) * 2 + rpar) * S1B;
          double x[4][4];
          load_rows(Sb + (2 * w) * F_S1W, F_S1W, lane, x);
          if constexpr (DEC) {   // done reading the plane buffer
            __syncwarp();
            if (lane == 0) mbar_arrive(&cons[par]);
          }
          planes2<SG, IS, 0>(x, prm, acc[S - 1]);
        } else if constexpr (DEC) {
          if (w < F_S1 / 2 - (S - 1) && lane == 0) mbar_arrive(&cons[par]);   // a stage-2 warp without work
        }
        if constexpr (S < K) {
          // (S < K only for K = 3: in-place Dirichlet loads)
          if (active) publish_ip<K, S, (IS + 1) % 3, !SG::assign0>(acc, sbuf + ((S - 1) * 2 + par) * S1B, w, lane, Y0, X0,
                                                                  p - S - LG, P0, P1, P2, in,
                                                                  xy_in[S - 1] && p - S - LG >= 1 && p - S - LG < P0 - 1);
          if constexpr (!F_LAG) __syncthreads();
        } else if (active) {
          // final plane zf = p - K - LG complete: ring slot (IS + 1) % 3
          constexpr int s = (IS + 1) % 3;
          const int zf = p - K - LG;
          if (cj >= 2 * K + LG && zf >= Z0 && zf < zend && (!act || zf >= dp.store_lo)) {
            // the plane goes to this slab and, for the first / last H own planes of a slab with a
            // neighbour there, into that neighbour's halo as well (peer memory)
            const int64_t e0 = (int64_t(zf) * P1 + Y0 + 2 * w) * P2 + X0 + c0;
            auto store_to = [&](double* o) {
#pragma unroll
              for (int y = 0; y < 2; ++y)
#pragma unroll
                for (int e = 0; e < 2; ++e)
                  if (st_ok[y][e]) o[y * P2 + e] = acc[K - 1][s][y][e];
            };
            store_to(out + e0);
            if (act) {   // (uniform per CTA; rare: the slab's first / last H planes)
              if (t_lo && zf < dp.lo_end) store_to(dp.dst_lo + (e0 + dp.off_lo));
              if (t_hi && zf >= dp.hi_begin) store_to(dp.dst_hi + (e0 + dp.off_hi));
            }
          }
          if constexpr (!SG::assign0) {
#pragma unroll
            for (int y = 0; y < 2; ++y) { acc[K - 1][s][y][0] = 0.0; acc[K - 1][s][y][1] = 0.0; }
          }
        }
      };
      [&]<int... Ss>(std::integer_sequence<int, Ss...>) {
        (stage(std::integral_constant<int, Ss + 2>{}), ...);
      }(std::make_integer_sequence<int, K - 1>{});
      if constexpr (F_LAG) {
        __syncthreads();  // this iteration's planes visible, last iteration's buffers and the input slot free
        if (q + F_NS - 1 < nstages) issue_next((slot + F_NS - 1) % F_NS);
      }
      if (++slot == F_NS) { slot = 0; phase ^= 1; }
      if (++cj == SI) {
        if (t_lo || t_hi) {
          // every warp makes its item stores visible system-wide and counts itself in; the last warp
          // to arrive publishes the step counter to the neighbour(s) (no CTA-wide barrier here)
          __threadfence_system();
          __syncwarp();
          if (lane == 0) {
            const unsigned prev = atomicAdd(&sig_count, 1u);
            if (prev == F_WARPS - 1) {
              sig_count = 0u;
              __threadfence_system();
              const int u = citem % (nbx * nby);
              if (t_lo) p2p_st_release(dp.sig_lo + u, dp.sig_val);
              if (t_hi) p2p_st_release(dp.sig_hi + u, dp.sig_val);
            }
          }
          __syncwarp();
        }
        cj = 0;
        citem += gridDim.x;
      }
    };
    [&]<int... Is>(std::integer_sequence<int, Is...>) {
      (one(std::integral_constant<int, Is>{}), ...);
    }(std::make_integer_sequence<int, 3>{});
  }
}

bool make_fparams(const Plan& p, FParams& prm) {
  std::memset(&prm, 0, sizeof(prm));
  if (p.ndim != 3 || p.R != 1) return false;
  const int R = 1, n = 3;
  for (int a0 = 0; a0 < n; ++a0) {
    std::vector<const Term*> ts;
    for (const Term& t : p.terms)
      if (t.plane == a0) ts.push_back(&t);
    if (ts.empty()) { prm.mode[a0] = PM_NONE; continue; }
    if (ts.size() == 1 && ts[0]->kind == kPoint && ts[0]->u[R] == 1.0 && ts[0]->u[0] == 0.0 && ts[0]->u[2] == 0.0 &&
        ts[0]->v[0] == 0.0 && ts[0]->v[2] == 0.0) {
      prm.mode[a0] = PM_POINT; prm.w[a0] = ts[0]->v[R]; continue;
    }
    if (ts.size() == 2 && ts[0]->kind == kArm && ts[1]->kind == kArm && ts[0]->u[R] == 1.0 && ts[1]->v[R] == 1.0 &&
        ts[0]->u[0] == 0.0 && ts[0]->u[2] == 0.0 && ts[1]->v[0] == 0.0 && ts[1]->v[2] == 0.0) {
      prm.mode[a0] = PM_STAR;
      for (int i = 0; i < n; ++i) { prm.v[a0][0][i] = ts[0]->v[i]; prm.u[a0][1][i] = ts[1]->u[i]; }
      continue;
    }
    if (ts.size() == 2 && ts[0]->kind == kChain && ts[0]->r == 1 && ts[1]->kind == kPoint && ts[1]->r == 0 &&
        ts[1]->u[R] == 1.0 && ts[0]->u[0] == ts[0]->u[2] && ts[0]->v[0] == ts[0]->v[2]) {
      if (pma1_unit_centre(ts[0]->u, ts[0]->v, prm.u[a0][0], prm.v[a0][0])) {
        prm.mode[a0] = PM_PMA1;
        prm.w[a0] = ts[1]->v[R];
        continue;
      }
    }
    if ((int)ts.size() > F_MAXK) return false;
    prm.mode[a0] = PM_CHAINS;
    prm.K[a0] = (int)ts.size();
    for (size_t k = 0; k < ts.size(); ++k)
      for (int i = 0; i < n; ++i) { prm.u[a0][k][i] = ts[k]->u[i]; prm.v[a0][k][i] = ts[k]->v[i]; }
  }
  bool same = true;
  for (int e = 0; e < n * n; ++e)
    if (p.W[e] != p.W[size_t(2) * n * n + e]) { same = false; break; }
  prm.mirror[0] = same ? 1 : 0;
  if (prm.mode[0] == PM_PMA1 && prm.mode[1] == PM_PMA1 && prm.mirror[0] && sym3_enabled()) {
    double c0, b0, a0, c1, b1, a1;
    if (sym3_plane(p.W.data(), 0, c0, b0, a0) && sym3_plane(p.W.data(), 1, c1, b1, a1)) {
      prm.mode[0] = prm.mode[1] = PM_SYM3;
      prm.sym[0][0] = c0; prm.sym[0][1] = b0; prm.sym[0][2] = a0;
      prm.sym[1][0] = c1; prm.sym[1][1] = b1; prm.sym[1][2] = a1;
    }
  }
  return true;
}

template <class SG, int K, bool TMA, bool P2P>
cudaError_t launch_f(const Plan& p, const double* src, double* dst, cudaStream_t s, const CUtensorMap& map,
                     const FParams& prm, const P2PArgs* d) {
  constexpr int STAGE = ((F_IN * F_BW * 8 + 127) / 128) * 128;
  const int smem = 128 + SG::ns * STAGE + 2 * (K - 1) * F_S1 * F_S1W * 8;
  int max_grid = 0;
  {
    cudaError_t e = kernel_setup((const void*)rdg3df_kernel<SG, K, TMA, P2P>, F_WARPS * 32, smem, &max_grid);
    if (e != cudaSuccess) return e;
  }
  if (d && d->prepare_only) return cudaSuccess;
  constexpr int TY = F_S1 - 2 * (K - 1), BS = 64 - 2 * (K - 1) - 2 * ((K - 1) & 1);
  const int nbx = (int)((p.N[2] + BS - 1) / BS), nby = (int)((p.N[1] + TY - 1) / TY);
  int64_t zc = F_ZC;
  {
    const int64_t cols = int64_t(nbx) * nby;
    const int64_t rounds = (cols * ((p.N[0] + zc - 1) / zc) + max_grid - 1) / max_grid;
    const int64_t nch = std::max<int64_t>(1, rounds * max_grid / cols);
    const int64_t zc2 = (p.N[0] + nch - 1) / nch;
    if (zc2 >= 8 && zc2 <= 2 * F_ZC && cols * ((p.N[0] + zc2 - 1) / zc2) <= rounds * max_grid) zc = zc2;
  }
  if (d && d->active) {
    // device-initiated exchange: exactly one z-chunk per column and side may touch a neighbour —
    // the first chunk holds view planes [1, lo_end) (ZC >= lo_end - 1) and the last one starts at or
    // below hi_begin (it has >= P0 - 1 - hi_begin planes)
    const int64_t N0v = p.N[0], need_lo = d->lo_end - 1, need_hi = (N0v + 1) - d->hi_begin;
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
  const int SI = ((ZC + 2 * K + F_LAG * (K - 1)) + 2) / 3 * 3;   // + the lag of the last stage
  const int nbz = (int)((p.N[0] + ZC - 1) / ZC);
  const int64_t nitems = int64_t(nbx) * nby * nbz;
  const int grid = (int)std::min<int64_t>(max_grid, nitems);
  static const P2PArgs none{};
  rdg3df_kernel<SG, K, TMA, P2P><<<grid, F_WARPS * 32, smem, s>>>(src, dst, p.N[0], p.N[1], p.N[2], nbx, nby, (int)nitems, ZC, SI,
                                                     map, prm, d ? *d : none);
  return cudaGetLastError();
}

template <int K, bool P2P>
cudaError_t launch_fk(const Plan& p, const double* src, double* dst, cudaStream_t s, const FParams& prm,
                      const P2PArgs* d = nullptr) {
  CUtensorMap map;
  const int64_t padded[3] = {p.P[0], p.P[1], p.P[2]};
  const int box[3] = {1, F_IN, F_BW};
  const bool tma = !p.force_no_tma && encode_tmap(&map, src, 3, padded, box);
  if (!tma) std::memset(&map, 0, sizeof(map));
  // specialisations: Box-3D27P-like (symmetric class sums or PMA planes, z-mirrored) and Heat-3D-like
  // (point / star, mirrored)
  if (prm.mode[0] == PM_SYM3)
    return tma ? launch_f<Sig3<PM_SYM3, PM_SYM3, 1>, K, true, P2P>(p, src, dst, s, map, prm, d)
               : launch_f<Sig3<PM_SYM3, PM_SYM3, 1>, K, false, P2P>(p, src, dst, s, map, prm, d);
  if (prm.mode[0] == PM_PMA1 && prm.mode[1] == PM_PMA1 && prm.mirror[0])
    return tma ? launch_f<Sig3<PM_PMA1, PM_PMA1, 1>, K, true, P2P>(p, src, dst, s, map, prm, d)
               : launch_f<Sig3<PM_PMA1, PM_PMA1, 1>, K, false, P2P>(p, src, dst, s, map, prm, d);
  if (prm.mode[0] == PM_POINT && prm.mode[1] == PM_STAR && prm.mirror[0])
    return tma ? launch_f<Sig3<PM_POINT, PM_STAR, 1>, K, true, P2P>(p, src, dst, s, map, prm, d)
               : launch_f<Sig3<PM_POINT, PM_STAR, 1>, K, false, P2P>(p, src, dst, s, map, prm, d);
  return tma ? launch_f<Sig3<-1, -1, -1>, K, true, P2P>(p, src, dst, s, map, prm, d)
             : launch_f<Sig3<-1, -1, -1>, K, false, P2P>(p, src, dst, s, map, prm, d);
}

}  // namespace

bool rdg3d_fused_supported(const Plan& p) {
  FParams prm;
  return make_fparams(p, prm);
}

cudaError_t launch_rdg3d_fused(const Plan& p, const double* src, double* dst, cudaStream_t s, int k, const P2PArgs* d) {
  FParams prm;
  if (!make_fparams(p, prm)) return cudaErrorNotSupported;
  if (d) {
    if (k == 2) return launch_fk<2, true>(p, src, dst, s, prm, d);
    if (k == 3) return launch_fk<3, true>(p, src, dst, s, prm, d);
  } else {
    if (k == 2) return launch_fk<2, false>(p, src, dst, s, prm, nullptr);
    if (k == 3) return launch_fk<3, false>(p, src, dst, s, prm, nullptr);
  }
  return cudaErrorNotSupported;
}

int rdg3d_fused_units(const Plan& p, int k, int* nux) {
  if (k < 2 || k > 3 || !rdg3d_fused_supported(p)) return 0;
  const int TY = F_S1 - 2 * (k - 1), BS = 64 - 2 * (k - 1) - 2 * ((k - 1) & 1);
  const int bx = (int)((p.N[2] + BS - 1) / BS), by = (int)((p.N[1] + TY - 1) / TY);
  if (nux) *nux = bx;
  return bx * by;
}

}  // namespace lora
