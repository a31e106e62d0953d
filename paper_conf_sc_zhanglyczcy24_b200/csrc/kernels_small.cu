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

template <int R>
__global__ void __launch_bounds__(SM_TX * SM_TY, 1)
small2d_star_kernel(const double* __restrict__ in, double* __restrict__ out, int N0, int N1, int rp, int T,
                    const __grid_constant__ StarArms w) {
  cg::cluster_group cl = cg::this_cluster();
  const int c = (int)cl.block_rank(), CS = (int)cl.num_blocks();
  extern __shared__ __align__(16) double sm[];
  const int P1 = N1 + 2 * R, SR = rp + 2 * R;
  double* buf0 = sm;
  double* buf1 = sm + size_t(SR) * P1;
  const int tid = threadIdx.y * SM_TX + threadIdx.x;
  const int64_t g0 = int64_t(c) * rp;   // padded row of buffer row 0 (own rows are buffer rows R .. R+rp-1)
  // stage the slab (own rows + R halo rows each side, all columns) into both buffers
  const double* src = in + g0 * P1;
  for (int i = tid; i < SR * P1; i += SM_TX * SM_TY) {
    const double v = src[i];
    buf0[i] = v;
    buf1[i] = v;
  }
  // neighbours' buffers (DSMEM): my first R own rows are rows rp+R.. of CTA c-1, my last R own
  // rows are rows 0..R-1 of CTA c+1
  double* lo0 = c > 0 ? cl.map_shared_rank(buf0, c - 1) : nullptr;
  double* lo1 = c > 0 ? cl.map_shared_rank(buf1, c - 1) : nullptr;
  double* hi0 = c < CS - 1 ? cl.map_shared_rank(buf0, c + 1) : nullptr;
  double* hi1 = c < CS - 1 ? cl.map_shared_rank(buf1, c + 1) : nullptr;
  cl.sync();   // every CTA staged its slab before anyone stores into a neighbour's halo
  for (int t = 0; t < T; ++t) {
    const double* cur = (t & 1) ? buf1 : buf0;
    double* nxt = (t & 1) ? buf0 : buf1;
    double* lo = (t & 1) ? lo0 : lo1;
    double* hi = (t & 1) ? hi0 : hi1;
    for (int j = R + threadIdx.y; j < R + rp; j += SM_TY) {
      for (int x = R + threadIdx.x; x < R + N1; x += SM_TX) {
        const double* cx = cur + size_t(j) * P1 + x;
        double th = 0.0;
#pragma unroll
        for (int b = -R; b <= R; ++b) th = fma(w.h[R + b], cx[b], th);
        double acc = 0.0;
#pragma unroll
        for (int a = -R; a <= R; ++a) {
          if (a == 0) acc += th;
          acc = fma(w.v[R + a], cx[a * P1], acc);
        }
        nxt[size_t(j) * P1 + x] = acc;
        if (lo && j < 2 * R) lo[size_t(rp + j) * P1 + x] = acc;
        if (hi && j >= rp) hi[size_t(j - rp) * P1 + x] = acc;
      }
    }
    cl.sync();   // release my rows (local and remote), acquire the neighbours' rows of my halo
  }
  // write back: own rows (all columns: the column halo is the input's), plus the grid's top / bottom
  // halo rows from the first / last CTA
  const double* res = (T & 1) ? buf1 : buf0;
  const int j0 = c == 0 ? 0 : R, j1 = c == CS - 1 ? SR : R + rp;
  double* dst = out + g0 * P1;
  for (int i = j0 * P1 + tid; i < j1 * P1; i += SM_TX * SM_TY) dst[i] = res[i];
  (void)N0;
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
const void* kernel_of() { return (const void*)small2d_star_kernel<R>; }

const void* kernel_for(int R) {
  switch (R) {
    case 1: return kernel_of<1>();
    case 2: return kernel_of<2>();
    case 3: return kernel_of<3>();
    case 4: return kernel_of<4>();
  }
  return nullptr;
}

constexpr size_t kMaxSmem = 227 * 1024;

// Cluster size for the plan: the largest CS in {16, 8, 4, 2} that divides N0 with >= R rows per CTA
// and whose slab pair fits the shared memory of one CTA; 0 = the plan does not fit.
int cluster_size(const Plan& p) {
  for (int cs : {16, 8, 4, 2}) {
    if (p.N[0] % cs) continue;
    const int64_t rp = p.N[0] / cs;
    if (rp < p.R) continue;
    const size_t smem = 2 * size_t(rp + 2 * p.R) * size_t(p.P[1]) * sizeof(double);
    if (smem <= kMaxSmem) return cs;
  }
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
  const void* k = kernel_for(p.R);
  // fall back to smaller clusters if the device cannot schedule this one
  while (cs >= 2 && setup(k, 2 * size_t(p.N[0] / cs + 2 * p.R) * size_t(p.P[1]) * 8, cs) == 0) {
    do { cs /= 2; } while (cs >= 2 && p.N[0] % cs);
  }
  if (cs < 2) return cudaErrorNotSupported;
  const int rp = (int)(p.N[0] / cs);
  const size_t smem = 2 * size_t(rp + 2 * p.R) * size_t(p.P[1]) * sizeof(double);
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
    case 1: return cudaLaunchKernelEx(&cfg, small2d_star_kernel<1>, in, out, N0, N1, rp, Ti, w);
    case 2: return cudaLaunchKernelEx(&cfg, small2d_star_kernel<2>, in, out, N0, N1, rp, Ti, w);
    case 3: return cudaLaunchKernelEx(&cfg, small2d_star_kernel<3>, in, out, N0, N1, rp, Ti, w);
    case 4: return cudaLaunchKernelEx(&cfg, small2d_star_kernel<4>, in, out, N0, N1, rp, Ti, w);
  }
  return cudaErrorInvalidValue;
}

}  // namespace lora
