// Small 2D grids (BASELINE configs[0], Heat-2D 256^2 x 10): ONE launch runs all T time steps.
//
// The per-step launches of the streaming engine leave a 0.5 MB problem launch- and latency-bound
// (r01: 9.7 GStencil/s with CUDA-graph replay).  Here the whole padded grid lives in the shared
// memory of one thread-block cluster (the B200 rules: distributed shared memory
// between the CTAs of a cluster): CTA c of CS owns rp = N0 / CS interior rows plus an R-row halo on
// each side, in two ping-pong buffers.  A step computes the CTA's own rows from buffer `cur` into
// `nxt`; the first / last R of them are also stored straight into the neighbour CTA's halo rows of
// `nxt` through DSMEM (st.shared::cluster via cluster.map_shared_rank); one cluster barrier per
// step (release/acquire) publishes them.  The column halo and the top / bottom halo rows of the
// grid are the Dirichlet values (loaded into both buffers, never written; Q1).
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
                                               int HK, int rp, bool last, size_t lo_off, size_t hi_off) {
  constexpr int NT = SM_TX * SM_TY;
  const int tid = threadIdx.y * SM_TX + threadIdx.x;
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
    if (in0 && in1) *reinterpret_cast<double2*>(op) = make_double2(a0, a1);
    else if (in1) op[1] = a1;
    else if (in0) op[0] = a0;
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
        star1_step_vec(src, dst, P1, N1, j0, j1, w, lo_mb, hi_mb, HK, rp, last, (2 * par + 1) * MB, (2 * par + 0) * MB);
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

cudaError_t launch_small2d(const Plan& p, const double* in, double* out, int64_t T, cudaStream_t s) {
  StarArms w;
  if (!star_arms(p, w) || T < 1 || T > (int64_t(1) << 30)) return cudaErrorInvalidValue;
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
