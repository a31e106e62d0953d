// 1D stencils (§IV-C P:354 "for 1D stencil ... one MM suffices"; Table II Heat-1D, 1D5P).
//
// A 1D stencil is a single banded gather (the horizontal RDG pass alone).  On B200 it is plainly
// HBM-bound, so the kernel is a CUDA-core banded pass with exact temporal fusion: a CTA stages a
// segment of S + 2KR points in shared memory (16-byte cp.async when aligned), advances it K time
// steps in shared memory (ping-pong, the region shrinking by R per step, the fixed Dirichlet halo
// re-imposed every step) and writes S points: 16/K bytes of HBM traffic per point-step.
// Consecutive lanes own consecutive points (bank-conflict-free shared-memory taps).
#include <cuda_runtime.h>

#include <algorithm>

#include "kernels.hpp"
#include "pipe.cuh"

namespace lora {
namespace {

constexpr int S1_THREADS = 256;
constexpr int S1_SEG = S1_THREADS * 8;              // final points per CTA item

struct W1 { double w[kMaxN]; };

template <int R, int K>
__global__ void __launch_bounds__(S1_THREADS) stencil1d_kernel(const double* __restrict__ in, double* __restrict__ out,
                                                             int64_t N0, int64_t nitems, const __grid_constant__ W1 W) {
  constexpr int n = 2 * R + 1;
  constexpr int HALO = K * R;
  constexpr int LEN = S1_SEG + 2 * HALO + 8;  // staged points (+ 8 of slack, never stored)
  extern __shared__ __align__(16) double sm1[];
  double* buf[2] = {sm1, sm1 + LEN};
  const int64_t P0 = N0 + 2 * R;
  const int tid = threadIdx.x;
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t x0 = R + item * S1_SEG;          // first final point (padded index)
    const int64_t g0 = x0 - HALO;                  // padded index of smem element 0
    // stage [g0, g0 + LEN) (zero outside the array)
    {
      double* b = buf[0];
      const bool vec = ((g0 & 1) == 0) && ((reinterpret_cast<uintptr_t>(in) & 15) == 0) && g0 >= 0 && g0 + LEN <= P0;
      if (vec) {
        for (int i = 2 * tid; i < LEN; i += 2 * S1_THREADS) cp_async16(b + i, in + g0 + i);
        cp_async_commit();
        cp_async_wait<0>();
      } else {
        for (int i = tid; i < LEN; i += S1_THREADS) {
          const int64_t g = g0 + i;
          b[i] = (g >= 0 && g < P0) ? __ldg(in + g) : 0.0;
        }
      }
      __syncthreads();
    }
    int cur = 0;
#pragma unroll
    for (int k = 1; k <= K; ++k) {
      // step k is computed on smem positions [k R, LEN - 8 - k R)
      const double* a = buf[cur];
      double* b = buf[cur ^ 1];
      const int lo = k * R, hi = LEN - 8 - k * R;
      // lane-consecutive points: a warp reads 32 consecutive doubles per tap (conflict-free)
      for (int pos = lo + tid; pos < hi; pos += S1_THREADS) {
        double s = 0.0;
#pragma unroll
        for (int t = 0; t < n; ++t) s = fma(W.w[t], a[pos - R + t], s);
        const int64_t g = g0 + pos;
        // the Dirichlet halo keeps its input value; points outside the array stay zero
        if (g < R || g >= P0 - R) s = (g >= 0 && g < P0) ? in[g] : 0.0;
        if (k == K) {
          if (pos >= HALO && pos < HALO + S1_SEG && g < P0 - R) out[g] = s;
        } else {
          b[pos] = s;
        }
      }
      __syncthreads();
      cur ^= 1;
    }
  }
}

template <int R, int K>
cudaError_t launch_k(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  constexpr int LEN = S1_SEG + 2 * K * R + 8;
  const int smem = 2 * LEN * 8;
  int max_grid = 0;
  {
    cudaError_t e = kernel_setup((const void*)stencil1d_kernel<R, K>, S1_THREADS, smem, &max_grid);
    if (e != cudaSuccess) return e;
  }
  W1 w{};
  for (int i = 0; i < 2 * R + 1; ++i) w.w[i] = p.W[i];
  const int64_t nitems = (p.N[0] + S1_SEG - 1) / S1_SEG;
  const int grid = (int)std::min<int64_t>(max_grid, nitems);
  stencil1d_kernel<R, K><<<grid, S1_THREADS, smem, s>>>(src, dst, p.N[0], nitems, w);
  return cudaGetLastError();
}

template <int R>
cudaError_t launch_r(const Plan& p, const double* src, double* dst, cudaStream_t s, int k) {
  switch (k) {
    case 1: return launch_k<R, 1>(p, src, dst, s);
    case 2: return launch_k<R, 2>(p, src, dst, s);
    case 3: return launch_k<R, 3>(p, src, dst, s);
    case 4: return launch_k<R, 4>(p, src, dst, s);
    case 5: return launch_k<R, 5>(p, src, dst, s);
    case 6: return launch_k<R, 6>(p, src, dst, s);
    case 7: return launch_k<R, 7>(p, src, dst, s);
    case 8: return launch_k<R, 8>(p, src, dst, s);
  }
  return cudaErrorNotSupported;
}

}  // namespace

cudaError_t launch_1d(const Plan& p, const double* src, double* dst, cudaStream_t s, int k) {
  if (p.ndim != 1) return cudaErrorInvalidValue;
  switch (p.R) {
    case 1: return launch_r<1>(p, src, dst, s, k);
    case 2: return launch_r<2>(p, src, dst, s, k);
    case 3: return launch_r<3>(p, src, dst, s, k);
    case 4: return launch_r<4>(p, src, dst, s, k);
  }
  return cudaErrorNotSupported;
}

}  // namespace lora
