// Small 2D grids (BASELINE configs[0], Heat-2D 256^2 x 10): ONE launch runs all T time steps.
//
// The per-step launches of the streaming engine leave a 0.5 MB problem launch- and latency-bound
// (r01: 9.7 GStencil/s with CUDA-graph replay).  Two single-launch variants:
//
// * cooperative grid (default, small2d_grid_kernel): G = N0 / rp co-resident CTAs, CTA c owns rp
//   interior rows plus a kR-deep halo on each side in two shared-memory ping-pong buffers.  A block
//   of k steps runs on a shrinking row range (step s of a block computes the rows that are still
//   valid: own rows plus (k - s) R halo rows each side).  A short run (T R <= 16) is ONE block whose
//   halo is staged from `in` (no exchange at all); longer runs exchange the first / last kR own rows
//   through a global buffer after each block, each CTA waiting only for its two neighbours' step
//   counters (release / acquire at gpu scope).
// * 2D tiles (default for short runs, small2d_tile_kernel): independent CTAs, each owning a TY x TX
//   tile and staging it with a T R-deep halo on all four sides from `in`; all T steps run on a
//   region that shrinks by R per step, with no exchange and no co-residency requirement.  Against
//   row slabs with the same T R-deep halo (below) the redundant halo work falls from about 5.5x to
//   2x for Heat-2D 256^2 x 10 (16 x 32 tiles), which is what bounded the slab form (issue-bound).
// * thread-block cluster (fallback, small2d_star_kernel): the same slab / block scheme with the whole
//   grid in the shared memory of one cluster of <= 16 CTAs and the exchange through the neighbours'
//   DSMEM mailboxes (st.shared::cluster via cluster.map_shared_rank), one cluster barrier per block.
//
// The column halo and the top / bottom halo rows of the grid are the Dirichlet values (loaded into
// both buffers, never written; Q1).
//
// Arithmetic: the two star arms of the planner (horizontal arm u = e_R, v = W[R,:]; vertical arm
// u = W[:,R] with the centre in the horizontal arm, v = e_R — planner.cpp factor_plane (i)) in
// EXACTLY the order of the streaming kernel's SIG_STAR row update (kernels_rdg.cu row_compute /
// row_shift): for output (y, x), the input rows r = y-R .. y+R in order, each adding
// fma(u[r-y+R], X[r][x], acc), with the horizontal gather t = sum_b fma(v[R+b], X[y][x+b]) added
// just before row r = y's term.  Results are therefore bitwise equal to the streaming engine
// (tests/test_gpu_parity.py::test_small_cluster_path_bitwise).
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <tuple>

#include "kernels.hpp"

namespace lora {
namespace {
namespace cg = cooperative_groups;

constexpr int SM_TX = 256, SM_TY = 4;   // 1024 threads: 256 consecutive columns x 4 rows per pass

struct StarArms {
  double h[kMaxN];   // horizontal arm, incl. the centre weight (v of term 0)
  double v[kMaxN];   // vertical arm (u of term 1; its centre is 0 when the horizontal arm has it)
};

// Buffer row j of CTA c holds padded row c*rp + R - HK + j (HK = k R: the halo depth of a block of
// k steps); own rows are j in [HK, HK + rp).  Rows outside the array are zero and never feed a
// stored value; rows of the global Dirichlet halo are loaded into both buffers and never written.
// Radius 1, even padded width: one step of rows [j0, j1) with each thread walking a strip of rows of
// one column pair (16-byte shared loads), the three rows of the vertical arm in registers and the
// horizontal neighbours from the adjacent lanes (shuffles; warp-edge lanes load theirs).  Same
// per-point arithmetic, in the same order, as the scalar loop below (and the streaming kernel).
__device__ __forceinline__ void star1_step_vec(const double* __restrict__ src, double* __restrict__ dst, int P1, int N1,
                                               int j0, int j1, const StarArms& w, double* lo_mb, double* hi_mb,
                                               int HK, int rp, bool last, size_t lo_off, size_t hi_off,
                                               int tid, int NT) {
  const int NPR = P1 / 2;                       // column pairs (2q, 2q+1), q < NPR
  const int QW = (NPR + 31) / 32 * 32;          // lanes per strip (whole warps)
  const int S = NT / QW;                        // strips
  const int q = tid % QW, sidx = tid / QW;
  if (sidx >= S) return;                        // whole warps only: shuffles stay warp-uniform
  const int lane = tid & 31;
  const int nr = j1 - j0, per = (nr + S - 1) / S;
  const int ra = j0 + sidx * per, rb = min(j1, ra + per);
  if (ra >= rb) return;                         // uniform per warp (a strip is whole warps)
  const bool act = q < NPR;
  const int x0 = act ? 2 * q : 0;               // idle lanes read column pair 0 (any row): finite values
  const bool in0 = act && x0 >= 1 && x0 <= N1, in1 = act && x0 + 1 <= N1;
  const bool ld_left = act && lane == 0 && x0 >= 1, ld_right = act && (lane == 31 || q == NPR - 1) && x0 + 2 < P1;
  const double* sp = src + ra * P1 + x0;        // row j, this pair
  double* op = dst + ra * P1 + x0;
  // mailbox rows: the block's last step stores my first / last HK own rows for the neighbours
  const bool mlo = last && lo_mb != nullptr, mhi = last && hi_mb != nullptr;
  double* lop = mlo ? lo_mb + lo_off + (ra - HK) * P1 + x0 : nullptr;
  double* hip = mhi ? hi_mb + hi_off + (ra - rp) * P1 + x0 : nullptr;
  double2 xm = *reinterpret_cast<const double2*>(sp - P1);
  double2 xc = *reinterpret_cast<const double2*>(sp);
#pragma unroll 3
  for (int j = ra; j < rb; ++j, sp += P1, op += P1, lop += P1, hip += P1) {
    const double2 xp = *reinterpret_cast<const double2*>(sp + P1);
    double left = __shfl_up_sync(0xffffffffu, xc.y, 1);
    double right = __shfl_down_sync(0xffffffffu, xc.x, 1);
    if (ld_left) left = sp[-1];
    if (ld_right) right = sp[2];
    double th = fma(w.h[0], left, 0.0);
    th = fma(w.h[1], xc.x, th);
    th = fma(w.h[2], xc.y, th);
    double a0 = fma(w.v[0], xm.x, 0.0);
    a0 += th;
    a0 = fma(w.v[1], xc.x, a0);
    a0 = fma(w.v[2], xp.x, a0);
    th = fma(w.h[0], xc.x, 0.0);
    th = fma(w.h[1], xc.y, th);
    th = fma(w.h[2], right, th);
    double a1 = fma(w.v[0], xm.y, 0.0);
    a1 += th;
    a1 = fma(w.v[1], xc.y, a1);
    a1 = fma(w.v[2], xp.y, a1);
    if (in0 && in1) {
      *reinterpret_cast<double2*>(op) = make_double2(a0, a1);
    } else {
      if (in1) op[1] = a1;
      if (in0) op[0] = a0;
    }
    if (mlo && j < 2 * HK) {
      if (in0) lop[0] = a0;
      if (in1) lop[1] = a1;
    }
    if (mhi && j >= rp) {
      if (in0) hip[0] = a0;
      if (in1) hip[1] = a1;
    }
    xm = xc;
    xc = xp;
  }
}

template <int R, bool VEC>
__global__ void __launch_bounds__(SM_TX * SM_TY, 1)
small2d_star_kernel(const double* __restrict__ in, double* __restrict__ out, int N0, int N1, int rp, int T, int kb,
                    const __grid_constant__ StarArms w) {
  cg::cluster_group cl = cg::this_cluster();
  const int c = (int)cl.block_rank(), CS = (int)cl.num_blocks();
  extern __shared__ __align__(16) double sm[];
  const int P1 = N1 + 2 * R, P0 = N0 + 2 * R, HK = kb * R, SR = rp + 2 * HK;
  double* const buf0 = sm;
  double* const buf1 = sm + size_t(SR) * P1;
  double* mbox = sm + 2 * size_t(SR) * P1;   // [parity][side 0: from c-1 (top), 1: from c+1 (bottom)][HK][P1]
  const size_t MB = size_t(HK) * P1;
  const int tid = threadIdx.y * SM_TX + threadIdx.x, NT = SM_TX * SM_TY;
  const int pr0 = c * rp + R - HK;          // padded row of buffer row 0
  for (int i = tid; i < SR * P1; i += NT) {
    const int pr = pr0 + i / P1;
    const double v = (pr >= 0 && pr < P0) ? in[int64_t(pr0) * P1 + i] : 0.0;
    buf0[i] = v;
    buf1[i] = v;
  }
  // the neighbours' mailboxes (DSMEM): my first HK own rows fill the bottom side of CTA c-1's, my
  // last HK own rows the top side of CTA c+1's
  double* lo_mb = c > 0 ? cl.map_shared_rank(mbox, c - 1) : nullptr;
  double* hi_mb = c < CS - 1 ? cl.map_shared_rank(mbox, c + 1) : nullptr;
  const int jlo = max(R, R - pr0), jhi = min(SR - R, P0 - R - pr0);   // buffer rows inside the interior
  cl.sync();   // every CTA staged its slab before any mailbox store
  int cur = 0;
  for (int t0 = 0, blk = 0; t0 < T; t0 += kb, ++blk) {
    const int ks = min(kb, T - t0);
    const int par = blk & 1;
    for (int st = 1; st <= ks; ++st) {
      const double* src = cur ? buf1 : buf0;
      double* dst = cur ? buf0 : buf1;
      const bool last = st == ks;
      // rows valid after this step: shrink by R per step from the block's HK-deep halo
      const int j0 = max(jlo, R * st + (HK - R * ks)), j1 = min(jhi, SR - R * st - (HK - R * ks));
      if constexpr (VEC) {
        star1_step_vec(src, dst, P1, N1, j0, j1, w, lo_mb, hi_mb, HK, rp, last, (2 * par + 1) * MB, (2 * par + 0) * MB,
                       tid, SM_TX * SM_TY);
      } else
      for (int j = j0 + threadIdx.y; j < j1; j += SM_TY) {
        const bool to_lo = last && lo_mb && j >= HK && j < 2 * HK;               // my first HK own rows
        const bool to_hi = last && hi_mb && j >= rp && j < rp + HK;               // my last HK own rows
        for (int x = R + threadIdx.x; x < R + N1; x += SM_TX) {
          const double* cx = src + size_t(j) * P1 + x;
          double th = 0.0;
#pragma unroll
          for (int b = -R; b <= R; ++b) th = fma(w.h[R + b], cx[b], th);
          double acc = 0.0;
#pragma unroll
          for (int a = -R; a <= R; ++a) {
            if (a == 0) acc += th;
            acc = fma(w.v[R + a], cx[a * P1], acc);
          }
          dst[size_t(j) * P1 + x] = acc;
          if (to_lo) lo_mb[(2 * par + 1) * MB + size_t(j - HK) * P1 + x] = acc;
          if (to_hi) hi_mb[(2 * par + 0) * MB + size_t(j - rp) * P1 + x] = acc;
        }
      }
      cur ^= 1;
      if (!last) __syncthreads();
    }
    cl.sync();   // release my mailbox stores, acquire the neighbours' rows of my halo
    if (t0 + ks < T) {   // unpack the mailbox into the halo rows of the block's result buffer
      // (interior columns only: the column halo of every row is the fixed Dirichlet value loaded at
      // the start, and the mailbox holds only the columns the neighbour computed)
      double* dst = cur ? buf1 : buf0;
      for (int j = threadIdx.y; j < HK; j += SM_TY)
        for (int x = R + threadIdx.x; x < R + N1; x += SM_TX) {
          if (c > 0) dst[size_t(j) * P1 + x] = mbox[(2 * par + 0) * MB + size_t(j) * P1 + x];
          if (c < CS - 1) dst[size_t(HK + rp + j) * P1 + x] = mbox[(2 * par + 1) * MB + size_t(j) * P1 + x];
        }
      __syncthreads();
    }
  }
  // write back: own rows (all columns: the column halo is the input's), plus the grid's top / bottom
  // halo rows from the first / last CTA
  const double* res = cur ? buf1 : buf0;
  const int w0 = c == 0 ? HK - R : HK, w1 = c == CS - 1 ? HK + rp + R : HK + rp;
  for (int i = w0 * P1 + tid; i < w1 * P1; i += NT) out[int64_t(pr0) * P1 + i] = res[i];
}

// Grid variant (the default when it applies): a cooperative grid of G = N0 / rp CTAs (co-resident,
// all SMs instead of one cluster's 16) with the same slab / block / shrinking-row scheme; after each
// block of k steps every CTA copies its first / last kR own rows into a global exchange buffer
// (two parities x G CTAs x 2 sides), one grid-wide barrier (cooperative groups) publishes them, and
// each CTA unpacks its neighbours' rows into its halo.  Same per-point arithmetic (bitwise equal).
#ifndef SMALL_GT_MAX
#define SMALL_GT_MAX 512
#endif
constexpr int GT_MAX = SMALL_GT_MAX;   // threads per CTA of the grid variant (whole strips of column pairs)
#ifndef SMALL_ONE_BLOCK_MAX_HALO
#define SMALL_ONE_BLOCK_MAX_HALO 16   // halo rows up to which a whole run is one block (no exchange)
#endif
#ifdef SMALL_TRACE
__device__ unsigned long long g_small_trace[64];
__device__ __forceinline__ void strace(int k) {
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_small_trace[k] = t;
  }
}
#else
__device__ __forceinline__ void strace(int) {}
#endif

template <int R, bool VEC>
__global__ void __launch_bounds__(GT_MAX)
small2d_grid_kernel(const double* __restrict__ in, double* __restrict__ out, double* __restrict__ xch,
                    unsigned long long* __restrict__ flags, unsigned long long base, int N0, int N1, int rp, int T,
                    int kb, const __grid_constant__ StarArms w) {
  const int c = blockIdx.x, G = gridDim.x;
  extern __shared__ __align__(16) double sm[];
  const int P1 = N1 + 2 * R, P0 = N0 + 2 * R, HK = kb * R, SR = rp + 2 * HK;
  double* const buf0 = sm;
  double* const buf1 = sm + size_t(SR) * P1;
  const int tid = threadIdx.x, NT = blockDim.x;
  const int pr0 = c * rp + R - HK;          // padded row of buffer row 0
  strace(0);
  {  // stage the slab: rows inside the array only (the others stay zero); all loads of a thread first
    const int r0 = max(0, -pr0), r1 = min(SR, P0 - pr0);
    for (int i = tid; i < SR * P1; i += NT) { buf0[i] = 0.0; buf1[i] = 0.0; }
    __syncthreads();
    const double* src = in + int64_t(pr0 + r0) * P1;
    const int n = (r1 - r0) * P1;
    double* d0 = buf0 + r0 * P1;
    double* d1 = buf1 + r0 * P1;
    constexpr int U = 8;
    for (int b = tid; b < n; b += NT * U) {
      double v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = b + u * NT < n ? __ldg(src + b + u * NT) : 0.0;
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (b + u * NT < n) { d0[b + u * NT] = v[u]; d1[b + u * NT] = v[u]; }
    }
  }
  const size_t XB = size_t(HK) * P1;       // one side of one CTA in the exchange buffer
  const int jlo = max(R, R - pr0), jhi = min(SR - R, P0 - R - pr0);
  __syncthreads();
  strace(1);
  int cur = 0;
  for (int t0 = 0, blk = 0; t0 < T; t0 += kb, ++blk) {
    const int ks = min(kb, T - t0);
    for (int st = 1; st <= ks; ++st) {
      const double* src = cur ? buf1 : buf0;
      double* dst = cur ? buf0 : buf1;
      const int j0 = max(jlo, R * st + (HK - R * ks)), j1 = min(jhi, SR - R * st - (HK - R * ks));
      if constexpr (VEC) {
        star1_step_vec(src, dst, P1, N1, j0, j1, w, nullptr, nullptr, HK, rp, false, 0, 0, tid, NT);
      } else {
        const int nrow = j1 - j0;
        for (int i = tid; i < nrow * N1; i += NT) {
          const int j = j0 + i / N1, x = R + i % N1;
          const double* cx = src + size_t(j) * P1 + x;
          double th = 0.0;
#pragma unroll
          for (int b = -R; b <= R; ++b) th = fma(w.h[R + b], cx[b], th);
          double acc = 0.0;
#pragma unroll
          for (int a = -R; a <= R; ++a) {
            if (a == 0) acc += th;
            acc = fma(w.v[R + a], cx[a * P1], acc);
          }
          dst[size_t(j) * P1 + x] = acc;
        }
      }
      cur ^= 1;
      __syncthreads();
      strace(2 + t0 + st);
    }
    if (t0 + ks < T) {
      double* res = cur ? buf1 : buf0;
      double* mine = xch + (size_t(blk & 1) * G + c) * 2 * XB;
      for (int i = tid; i < HK * N1; i += NT) {       // interior columns of my first / last HK own rows
        const int r = i / N1, x = R + i % N1;
        mine[size_t(r) * P1 + x] = res[size_t(HK + r) * P1 + x];
        mine[XB + size_t(r) * P1 + x] = res[size_t(rp + r) * P1 + x];
      }
      // publish my rows (release), then wait only for the two neighbours' rows of this block (acquire):
      // a CTA cannot run two blocks ahead of a neighbour, so two exchange parities suffice
      __syncthreads();
      if (tid == 0) {
        __threadfence();
        asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(flags + c), "l"(base + blk + 1) : "memory");
        for (int nb = c - 1; nb <= c + 1; nb += 2) {
          if (nb < 0 || nb >= G) continue;
          unsigned long long v;
          do {
            asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(flags + nb) : "memory");
          } while (v < base + blk + 1);
        }
      }
      __syncthreads();
      const double* lo = xch + (size_t(blk & 1) * G + (c - 1)) * 2 * XB + XB;   // c-1's last HK own rows
      const double* hi = xch + (size_t(blk & 1) * G + (c + 1)) * 2 * XB;        // c+1's first HK own rows
      for (int i = tid; i < HK * N1; i += NT) {
        const int r = i / N1, x = R + i % N1;
        if (c > 0) res[size_t(r) * P1 + x] = lo[size_t(r) * P1 + x];
        if (c < G - 1) res[size_t(HK + rp + r) * P1 + x] = hi[size_t(r) * P1 + x];
      }
      __syncthreads();
      strace(40 + blk);
    }
  }
  const double* res = cur ? buf1 : buf0;
  const int w0 = c == 0 ? HK - R : HK, w1 = c == G - 1 ? HK + rp + R : HK + rp;
  for (int i = w0 * P1 + tid; i < w1 * P1; i += NT) out[int64_t(pr0) * P1 + i] = res[i];
  strace(60);
}

// 2D-tile variant.  CTA (bx, by) owns interior rows [y0, y0 + TY) and columns [x0, x0 + TX) (padded
// coordinates, y0 = R + by TY, x0 = R + bx TX) and stages rows [y0 - H, y0 + TY + H) x columns
// [x0 - H, x0 + TX + H), H = T R, into both shared buffers (zero outside the padded array; array-halo
// cells hold the fixed Dirichlet values and are never written).  Step s computes the interior points
// within (T - s) R of the own tile; after T steps the own tile is exact.  Per-point arithmetic: the
// scalar loop of the other variants, i.e. the streaming kernel's SIG_STAR order (bitwise equal).
#ifndef SMALL_TILE_STRIPS
#define SMALL_TILE_STRIPS 1   // threads walk row strips with a register window (0: one point per iteration)
#endif
#ifndef SMALL_TILE_UNROLL
#define SMALL_TILE_UNROLL 2   // row-strip unroll of the 2D-tile kernel
#endif
constexpr int kTileUnroll = SMALL_TILE_UNROLL;   // (#pragma arguments are not macro-expanded)
#ifndef SMALL_TILE_FULL
#define SMALL_TILE_FULL 1     // every step over the whole staged interior (fixed bounds; 0: the shrinking cone)
#endif
#ifndef SMALL_TILE_TY
#define SMALL_TILE_TY 8   // 512 threads (Heat-2D 256^2 x 10: 11.7 us back to back vs 14.0 with 4, 13.4 with 2)
#endif
constexpr int TL_TX = 64, TL_TY = SMALL_TILE_TY;   // threads: 64 columns x TL_TY row groups
template <int R>
__global__ void __launch_bounds__(TL_TX * TL_TY)
small2d_tile_kernel(const double* __restrict__ in, double* __restrict__ out, int N0, int N1, int TY, int TX, int T,
                    const __grid_constant__ StarArms w) {
  extern __shared__ __align__(16) double sm[];
  const int P0 = N0 + 2 * R, P1 = N1 + 2 * R, H = T * R;
  const int y0 = R + blockIdx.y * TY, x0 = R + blockIdx.x * TX;
  const int ty1 = min(TY, N0 - (y0 - R)), tx1 = min(TX, N1 - (x0 - R));   // own extent (edge tiles are partial)
  const int SY = ty1 + 2 * H, SX = tx1 + 2 * H;                           // staged region
  const int gy0 = y0 - H, gx0 = x0 - H;                                   // padded origin of buffer cell (0, 0)
  double* const buf0 = sm;
  double* const buf1 = sm + size_t(SY) * SX;
  const int tid = threadIdx.y * TL_TX + threadIdx.x;
  constexpr int NT = TL_TX * TL_TY;
  {  // staging: thread (x, y) takes columns x, x + 64, ... of rows y, y + TL_TY, ...; all of a thread's
     // loads of a column first (one HBM / L2 latency instead of one per element), no divisions
    constexpr int U = 8;
    for (int c = (int)threadIdx.x; c < SX; c += TL_TX) {
      const int gx = gx0 + c;
      const bool cin = gx >= 0 && gx < P1;
      for (int r0 = (int)threadIdx.y; r0 < SY; r0 += TL_TY * U) {
        double v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int r = r0 + u * TL_TY, gy = gy0 + r;
          v[u] = (r < SY && cin && gy >= 0 && gy < P0) ? __ldg(in + int64_t(gy) * P1 + gx) : 0.0;
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int r = r0 + u * TL_TY;
          if (r < SY) { buf0[r * SX + c] = v[u]; buf1[r * SX + c] = v[u]; }
        }
      }
    }
  }
  __syncthreads();
  // buffer rows / columns of interior (updatable) points
  const int ilo_r = max(0, R - gy0), ihi_r = min(SY, R + N0 - gy0);
  const int ilo_c = max(0, R - gx0), ihi_c = min(SX, R + N1 - gx0);
  int cur = 0;
#if SMALL_TILE_FULL
  // every step computes the whole staged interior except its outer R ring (fixed bounds, no per-step
  // set-up): cells within s R of the staged edge are stale after step s, and s R <= T R = H never
  // reaches the own tile, whose values are exactly those of the per-step path
  const int r0 = max(ilo_r, R), r1 = min(ihi_r, SY - R), c0 = max(ilo_c, R), c1 = min(ihi_c, SX - R);
  const int per = (r1 - r0 + TL_TY - 1) / TL_TY;
  const int ra = r0 + (int)threadIdx.y * per, rb = min(r1, ra + per);
#endif
  for (int st = 1; st <= T; ++st) {
    const double* src = cur ? buf1 : buf0;
    double* dst = cur ? buf0 : buf1;
#if !SMALL_TILE_FULL
    const int m = (T - st) * R;   // distance from the own tile still computed at this step
    const int r0 = max(ilo_r, H - m), r1 = min(ihi_r, H + ty1 + m);
    const int c0 = max(ilo_c, H - m), c1 = min(ihi_c, H + tx1 + m);
#endif
#if SMALL_TILE_FULL
    for (int c = c0 + (int)threadIdx.x; c < c1 && ra < rb; c += TL_TX) {
      const double* cp = src + size_t(ra) * SX + c;
      double* op = dst + size_t(ra) * SX + c;
      double win[2 * R + 1];
#pragma unroll
      for (int a = 0; a < 2 * R; ++a) win[a] = cp[(a - R) * SX];
#pragma unroll kTileUnroll
      for (int r = ra; r < rb; ++r, cp += SX, op += SX) {
        win[2 * R] = cp[R * SX];
        double th = 0.0;
#pragma unroll
        for (int b = -R; b <= R; ++b) th = fma(w.h[R + b], b == 0 ? win[R] : cp[b], th);
        double acc = 0.0;
#pragma unroll
        for (int a = -R; a <= R; ++a) {
          if (a == 0) acc += th;
          acc = fma(w.v[R + a], win[R + a], acc);
        }
        *op = acc;
#pragma unroll
        for (int a = 0; a < 2 * R; ++a) win[a] = win[a + 1];
      }
    }
#elif SMALL_TILE_STRIPS
    // each thread walks a strip of consecutive rows of one column with the 2R + 1 rows of the
    // vertical arm in a register window (one new shared load per row for it)
    const int nr = r1 - r0, per = (nr + TL_TY - 1) / TL_TY;
    const int ra = r0 + (int)threadIdx.y * per, rb = min(r1, ra + per);
    for (int c = c0 + (int)threadIdx.x; c < c1 && ra < rb; c += TL_TX) {
      const double* cp = src + size_t(ra) * SX + c;
      double* op = dst + size_t(ra) * SX + c;
      double win[2 * R + 1];
#pragma unroll
      for (int a = 0; a < 2 * R; ++a) win[a] = cp[(a - R) * SX];
#pragma unroll 2
      for (int r = ra; r < rb; ++r, cp += SX, op += SX) {
        win[2 * R] = cp[R * SX];
        double th = 0.0;
#pragma unroll
        for (int b = -R; b <= R; ++b) th = fma(w.h[R + b], b == 0 ? win[R] : cp[b], th);
        double acc = 0.0;
#pragma unroll
        for (int a = -R; a <= R; ++a) {
          if (a == 0) acc += th;
          acc = fma(w.v[R + a], win[R + a], acc);
        }
        *op = acc;
#pragma unroll
        for (int a = 0; a < 2 * R; ++a) win[a] = win[a + 1];
      }
    }
#else
    for (int r = r0 + (int)threadIdx.y; r < r1; r += TL_TY) {
      for (int c = c0 + (int)threadIdx.x; c < c1; c += TL_TX) {
        const double* cx = src + size_t(r) * SX + c;
        double th = 0.0;
#pragma unroll
        for (int b = -R; b <= R; ++b) th = fma(w.h[R + b], cx[b], th);
        double acc = 0.0;
#pragma unroll
        for (int a = -R; a <= R; ++a) {
          if (a == 0) acc += th;
          acc = fma(w.v[R + a], cx[a * SX], acc);
        }
        dst[size_t(r) * SX + c] = acc;
      }
    }
#endif
    cur ^= 1;
    __syncthreads();
  }
  // write back the own tile, extended by R into the array halo where the tile touches the array
  // edge (those cells hold the input's Dirichlet values in both buffers)
  const double* res = cur ? buf1 : buf0;
  const int wr0 = H - (blockIdx.y == 0 ? R : 0), wr1 = H + ty1 + (y0 - R + ty1 == N0 ? R : 0);
  const int wc0 = H - (blockIdx.x == 0 ? R : 0), wc1 = H + tx1 + (x0 - R + tx1 == N1 ? R : 0);
  const int nwc = wc1 - wc0;
  for (int i = tid; i < (wr1 - wr0) * nwc; i += NT) {
    const int r = wr0 + i / nwc, c = wc0 + i % nwc;
    out[int64_t(gy0 + r) * P1 + gx0 + c] = res[size_t(r) * SX + c];
  }
}

// The two-arm star signature of the streaming engine (kernels_rdg.cu signature(), SIG_STAR).
bool star_arms(const Plan& p, StarArms& w) {
  const int R = p.R, n = 2 * R + 1;
  if (p.ndim != 2 || p.terms.size() != 2) return false;
  const Term& a = p.terms[0];
  const Term& b = p.terms[1];
  if (a.kind != kArm || b.kind != kArm || a.u[R] != 1.0 || b.v[R] != 1.0) return false;
  std::memset(&w, 0, sizeof(w));
  for (int i = 0; i < n; ++i) {
    if (i != R && (a.u[i] != 0.0 || b.v[i] != 0.0)) return false;
    w.h[i] = a.v[i];
    w.v[i] = b.u[i];
  }
  return true;
}

template <int R>
const void* kernel_of(bool vec) {
  if constexpr (R == 1) { if (vec) return (const void*)small2d_star_kernel<1, true>; }
  return (const void*)small2d_star_kernel<R, false>;
}

const void* kernel_for(int R, bool vec) {
  switch (R) {
    case 1: return kernel_of<1>(vec);
    case 2: return kernel_of<2>(vec);
    case 3: return kernel_of<3>(vec);
    case 4: return kernel_of<4>(vec);
  }
  return nullptr;
}

constexpr size_t kMaxSmem = 227 * 1024;
#ifndef SMALL_MAX_BLOCK
#define SMALL_MAX_BLOCK 4
#endif
constexpr int kMaxBlock = SMALL_MAX_BLOCK;   // steps per exchange (redundant halo rows grow with it)

// Shared memory of one CTA: two slab buffers of rp + 2kR rows plus the double-buffered two-sided
// mailbox of kR rows.
size_t smem_bytes(const Plan& p, int64_t rp, int k) {
  const size_t P1 = size_t(p.P[1]), HK = size_t(k) * p.R;
  return (2 * (size_t(rp) + 2 * HK) * P1 + 4 * HK * P1) * sizeof(double);
}

// Steps per exchange for cluster size cs: the largest k <= kMaxBlock with kR <= rp that fits.
int block_steps(const Plan& p, int cs) {
  if (p.N[0] % cs) return 0;
  const int64_t rp = p.N[0] / cs;
  for (int k = kMaxBlock; k >= 1; --k)
    if (int64_t(k) * p.R <= rp && smem_bytes(p, rp, k) <= kMaxSmem) return k;
  return 0;
}

// Cluster size for the plan: the largest CS in {16, 8, 4, 2} that divides N0 with >= R rows per CTA
// and whose buffers fit the shared memory of one CTA; 0 = the plan does not fit.
int cluster_size(const Plan& p) {
  for (int cs : {16, 8, 4, 2})
    if (block_steps(p, cs) > 0) return cs;
  return 0;
}

// Per device: attributes set once, and whether a 16-CTA (non-portable) cluster can be scheduled.
int setup(const void* k, size_t smem, int cs) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, std::pair<size_t, int>> done;   // -> (smem set, max cluster)
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  std::lock_guard<std::mutex> lock(mu);
  auto& e = done[{k, dev}];
  if (e.first < smem) {
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem) != cudaSuccess ||
        cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess) {
      cudaGetLastError();
      return 0;
    }
    e.first = kMaxSmem;
  }
  if (e.second == 0) {
    int best = 0;
    for (int c : {16, 8, 4, 2}) {
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(c, 1, 1);
      cfg.blockDim = dim3(SM_TX, SM_TY, 1);
      cfg.dynamicSmemBytes = kMaxSmem;
      cudaLaunchAttribute at;
      at.id = cudaLaunchAttributeClusterDimension;
      at.val.clusterDim.x = c; at.val.clusterDim.y = 1; at.val.clusterDim.z = 1;
      cfg.attrs = &at;
      cfg.numAttrs = 1;
      int nclusters = 0;
      if (cudaOccupancyMaxActiveClusters(&nclusters, k, &cfg) == cudaSuccess && nclusters > 0) { best = c; break; }
      cudaGetLastError();
    }
    e.second = best > 0 ? best : -1;
  }
  return e.second > 0 && cs <= e.second ? cs : 0;
}

}  // namespace

bool small2d_eligible(const Plan& p) {
  StarArms w;
  return !p.no_small && p.ndim == 2 && p.engine == LORA_ENGINE_RDG_CUDA && p.R >= 1 && p.R <= kMaxRadius &&
         star_arms(p, w) && cluster_size(p) > 0;
}

namespace {
// Grid variant: rows per CTA (a divisor of N0, >= R) and the resulting CTA count; 0 if none fits.
int grid_rows(const Plan& p, int maxG) {
  const int want = std::max(1, p.small_rp);
  int best = 0;
  for (int rp = std::max(want, p.R); rp <= 64 && !best; ++rp)
    if (p.N[0] % rp == 0 && p.N[0] / rp <= maxG && p.N[0] / rp >= 2) best = rp;
  return best;
}

template <int R, bool VEC>
cudaError_t grid_launch(const Plan& p, const double* in, double* out, double* xch, unsigned long long* flags,
                        unsigned long long base, int rp, int kb, int T, int threads, size_t smem, const StarArms& w,
                        cudaStream_t s) {
  const void* k = (const void*)small2d_grid_kernel<R, VEC>;
  const int G = (int)(p.N[0] / rp);
  {  // per (device, threads, smem): the attribute and the co-residency bound, computed once
    static std::mutex mu;
    static std::map<std::tuple<int, int, size_t>, int> cap;   // -> resident CTAs on the device (0: unusable)
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return cudaErrorNotSupported; }
    std::lock_guard<std::mutex> lock(mu);
    auto it = cap.find({dev, threads, smem});
    if (it == cap.end()) {
      int occ = 0, sms = 0, resident = 0;
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
#ifndef SMALL_ATTR_EXACT
#define SMALL_ATTR_EXACT 0
#endif
      const int attr = SMALL_ATTR_EXACT ? (int)smem : (int)kMaxSmem;
#ifdef SMALL_CARVEOUT
      cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, SMALL_CARVEOUT);
#endif
      if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, attr) == cudaSuccess &&
          cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, threads, smem) == cudaSuccess)
        resident = occ * sms;
      cudaGetLastError();
      it = cap.emplace(std::make_tuple(dev, threads, smem), resident).first;
    }
    if (it->second < G) return cudaErrorNotSupported;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(G, 1, 1);
  cfg.blockDim = dim3(threads, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at;
  at.id = cudaLaunchAttributeCooperative;
  at.val.cooperative = 1;
  cfg.attrs = &at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, small2d_grid_kernel<R, VEC>, in, out, xch, flags, base, (int)p.N[0], (int)p.N[1], rp,
                            T, kb, w);
}

cudaError_t launch_grid_variant(Plan& p, const double* in, double* out, int64_t T, cudaStream_t s,
                                const StarArms& w) {
  if (p.small_mode == 1) return cudaErrorNotSupported;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int rp = grid_rows(p, sms);
  if (rp == 0) return cudaErrorNotSupported;
  // a short run in ONE block (halo T R rows deep, all of it staged from `in`: no exchange at all, the
  // redundant halo rows are cheaper than a neighbour wait); longer runs in blocks of k <= rp / R steps
  const size_t one_block = 2 * size_t(rp + 2 * T * p.R) * size_t(p.P[1]) * sizeof(double);
  const int kb = (T * p.R <= SMALL_ONE_BLOCK_MAX_HALO && one_block <= kMaxSmem)
                     ? (int)T : (int)std::min<int64_t>(std::min(kMaxBlock, rp / p.R), T);
  const int HK = kb * p.R, G = (int)(p.N[0] / rp);
  const size_t smem = 2 * size_t(rp + 2 * HK) * size_t(p.P[1]) * sizeof(double);
  if (smem > kMaxSmem) return cudaErrorNotSupported;
  // exchange buffer [parity][CTA][side][HK][P1] followed by one 64-bit step counter per CTA
  const size_t xdata = size_t(2) * G * 2 * HK * size_t(p.P[1]);
  const size_t xelems = xdata + size_t(G);
  Plan& mp = p;
  if (mp.xbuf_elems != xelems) {   // (re)allocated per geometry: the counters start at 0 again
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone) {
      cudaGetLastError();
      return cudaErrorNotSupported;   // no allocation inside the caller's graph capture: cluster variant
    }
    if (mp.xbuf) cudaFree(mp.xbuf);
    mp.xbuf = nullptr;
    mp.xbuf_elems = 0;
    if (cudaMalloc(&mp.xbuf, xelems * sizeof(double)) != cudaSuccess) { cudaGetLastError(); mp.xbuf = nullptr; return cudaErrorNotSupported; }
    if (cudaMemsetAsync(mp.xbuf, 0, xelems * sizeof(double), s) != cudaSuccess) { cudaGetLastError(); return cudaErrorNotSupported; }
    mp.xbuf_elems = xelems;
    mp.xflag_base = 0;
  }
  // counters are monotonic across launches: this launch publishes base + 1 .. base + nblocks
  unsigned long long* flags = reinterpret_cast<unsigned long long*>(mp.xbuf + (mp.xbuf_elems - size_t(G)));
  const unsigned long long base = mp.xflag_base;
  mp.xflag_base += (unsigned long long)((T + kb - 1) / kb) + 1;
  const bool vec = p.R == 1 && (p.P[1] % 2) == 0;
  const int qw = ((int)(p.P[1] / 2) + 31) / 32 * 32;
  const int threads = vec ? std::max(1, GT_MAX / qw) * qw : 256;
  if (vec && qw > GT_MAX) return cudaErrorNotSupported;
  const int Ti = (int)T;
  switch (p.R) {
    case 1: return vec ? grid_launch<1, true>(p, in, out, mp.xbuf, flags, base, rp, kb, Ti, threads, smem, w, s)
                       : grid_launch<1, false>(p, in, out, mp.xbuf, flags, base, rp, kb, Ti, threads, smem, w, s);
    case 2: return grid_launch<2, false>(p, in, out, mp.xbuf, flags, base, rp, kb, Ti, threads, smem, w, s);
    case 3: return grid_launch<3, false>(p, in, out, mp.xbuf, flags, base, rp, kb, Ti, threads, smem, w, s);
    case 4: return grid_launch<4, false>(p, in, out, mp.xbuf, flags, base, rp, kb, Ti, threads, smem, w, s);
  }
  return cudaErrorNotSupported;
}

// Tile shape for the 2D-tile variant: the (TY, TX) in {8, 16, 32, 64}^2 with the least work per SM
// (CTA rounds over the SMs x the CTA's points over the T steps); 0 if the halo'd tile
// does not fit the shared memory.
bool tile_shape(const Plan& p, int64_t T, int sms, int& TY, int& TX, size_t& smem) {
  const int64_t H = T * p.R;
  double best = 0.0;
  TY = TX = 0;
  for (int ty : {8, 16, 32, 64})
    for (int tx : {8, 16, 32, 64}) {
      const int ey = (int)std::min<int64_t>(ty, p.N[0]), ex = (int)std::min<int64_t>(tx, p.N[1]);
      const size_t sb = 2 * size_t(ey + 2 * H) * size_t(ex + 2 * H) * sizeof(double);
      if (sb > kMaxSmem) continue;
      const int64_t G = ((p.N[0] + ty - 1) / ty) * ((p.N[1] + tx - 1) / tx);
      double work = 0.0;
      for (int64_t s = 1; s <= T; ++s) {   // points computed per step (SMALL_TILE_FULL: the staged interior)
        const int64_t m = SMALL_TILE_FULL ? H - p.R : (T - s) * p.R;
        work += double(std::min<int64_t>(ey + 2 * m, p.N[0])) * double(std::min<int64_t>(ex + 2 * m, p.N[1]));
      }
      const double cost = double((G + sms - 1) / sms) * work;   // CTAs on the busiest SM x points per CTA
      if (TY == 0 || cost < best) { best = cost; TY = ty; TX = tx; smem = sb; }
    }
  return TY > 0;
}

cudaError_t launch_tile_variant(const Plan& p, const double* in, double* out, int64_t T, cudaStream_t s,
                                const StarArms& w) {
  if (p.small_mode != 0 || T * p.R > SMALL_ONE_BLOCK_MAX_HALO) return cudaErrorNotSupported;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int TY = 0, TX = 0;
  size_t smem = 0;
  if (!tile_shape(p, T, sms, TY, TX, smem)) return cudaErrorNotSupported;
  const void* k = nullptr;
  switch (p.R) {
    case 1: k = (const void*)small2d_tile_kernel<1>; break;
    case 2: k = (const void*)small2d_tile_kernel<2>; break;
    case 3: k = (const void*)small2d_tile_kernel<3>; break;
    case 4: k = (const void*)small2d_tile_kernel<4>; break;
    default: return cudaErrorNotSupported;
  }
  {  // the dynamic shared memory attribute, once per (kernel, device)
    static std::mutex mu;
    static std::map<std::pair<const void*, int>, bool> done;
    std::lock_guard<std::mutex> lock(mu);
    bool& d = done[{k, dev}];
    if (!d) {
      if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem) != cudaSuccess) {
        cudaGetLastError();
        return cudaErrorNotSupported;
      }
      d = true;
    }
  }
  const dim3 grid((unsigned)((p.N[1] + TX - 1) / TX), (unsigned)((p.N[0] + TY - 1) / TY), 1);
  const dim3 block(TL_TX, TL_TY, 1);
  const int N0 = (int)p.N[0], N1 = (int)p.N[1], Ti = (int)T;
  switch (p.R) {
    case 1: small2d_tile_kernel<1><<<grid, block, smem, s>>>(in, out, N0, N1, TY, TX, Ti, w); break;
    case 2: small2d_tile_kernel<2><<<grid, block, smem, s>>>(in, out, N0, N1, TY, TX, Ti, w); break;
    case 3: small2d_tile_kernel<3><<<grid, block, smem, s>>>(in, out, N0, N1, TY, TX, Ti, w); break;
    case 4: small2d_tile_kernel<4><<<grid, block, smem, s>>>(in, out, N0, N1, TY, TX, Ti, w); break;
  }
  return cudaGetLastError();
}
}  // namespace

#ifdef SMALL_TRACE
extern "C" int lora_small_trace(unsigned long long* h) { return (int)cudaMemcpyFromSymbol(h, g_small_trace, sizeof(unsigned long long) * 64); }
#endif
cudaError_t launch_small2d(Plan& p, const double* in, double* out, int64_t T, cudaStream_t s) {
  StarArms w;
  if (!star_arms(p, w) || T < 1) return cudaErrorInvalidValue;
  if (T > (int64_t(1) << 30)) return cudaErrorNotSupported;   // (int step counts) the per-step path runs it
  {
    const cudaError_t et = launch_tile_variant(p, in, out, T, s, w);
    if (et != cudaErrorNotSupported) return et;
    const cudaError_t eg = launch_grid_variant(p, in, out, T, s, w);
    if (eg != cudaErrorNotSupported) return eg;
  }
  int cs = cluster_size(p);
  if (cs == 0) return cudaErrorInvalidValue;
  const bool vec = p.R == 1 && (p.P[1] % 2) == 0;   // 16-byte rows: the register-walking R = 1 step
  const void* k = kernel_for(p.R, vec);
  // fall back to smaller clusters if the device cannot schedule this one
  while (cs >= 2 && (block_steps(p, cs) == 0 || setup(k, kMaxSmem, cs) == 0)) cs /= 2;
  if (cs < 2) return cudaErrorNotSupported;
  const int rp = (int)(p.N[0] / cs);
  const int kb = (int)std::min<int64_t>(block_steps(p, cs), T);
  const size_t smem = smem_bytes(p, rp, kb);
  if (smem > kMaxSmem) return cudaErrorNotSupported;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(cs, 1, 1);
  cfg.blockDim = dim3(SM_TX, SM_TY, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at;
  at.id = cudaLaunchAttributeClusterDimension;
  at.val.clusterDim.x = cs; at.val.clusterDim.y = 1; at.val.clusterDim.z = 1;
  cfg.attrs = &at;
  cfg.numAttrs = 1;
  const int N0 = (int)p.N[0], N1 = (int)p.N[1], Ti = (int)T;
  switch (p.R) {
    case 1: return vec ? cudaLaunchKernelEx(&cfg, small2d_star_kernel<1, true>, in, out, N0, N1, rp, Ti, kb, w)
                       : cudaLaunchKernelEx(&cfg, small2d_star_kernel<1, false>, in, out, N0, N1, rp, Ti, kb, w);
    case 2: return cudaLaunchKernelEx(&cfg, small2d_star_kernel<2, false>, in, out, N0, N1, rp, Ti, kb, w);
    case 3: return cudaLaunchKernelEx(&cfg, small2d_star_kernel<3, false>, in, out, N0, N1, rp, Ti, kb, w);
    case 4: return cudaLaunchKernelEx(&cfg, small2d_star_kernel<4, false>, in, out, N0, N1, rp, Ti, kb, w);
  }
  return cudaErrorInvalidValue;
}

}  // namespace lora
