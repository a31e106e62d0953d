// K11 — CUDA-core FP64 direct stencil (the in-tree comparison kernel, north star (c)), and the
// halo-copy helper.  out(x) = sum_a W[a] in(x + a - R) (eq. 2), interior only.
// 1D, 2D and 3D with R <= 2 run the direct sum on the same warp-streaming machinery as the RDG
// engines (kernels_1d.cu, kernels_rdg.cu SIG_DIRECT, kernels_rdg3d.cu PM_DIRECT) so that the
// comparison is like for like; this file keeps the 3D R = 3, 4 tile kernel and the halo copy.
//
// Weights travel as kernel parameters (constant bank 0), so every DFMA takes its weight as a
// c[0x0][..] operand: no load instruction per weight.
#include <cuda_runtime.h>

#include "kernels.hpp"

namespace lora {
namespace {

template <int R> struct W3 { double w[(2 * R + 1) * (2 * R + 1) * (2 * R + 1)]; };

// ---------------------------------------------------------------- 3D
// z-streaming: CTA = 32 x 8 threads owns a 32 x 8 (x, y) column of outputs over a z-chunk.
// Each input plane p is staged once in smem ((8+2R) x (32+2R)); every thread reads its
// (2R+1)^2 window of it once and adds the contribution of plane p to the 2R+1 outputs
// z = p - a0 + R in a rolling register accumulator ring.
constexpr int D3_BX = 32, D3_BY = 8, D3_ZC = 64;

template <int R>
__global__ void __launch_bounds__(256) direct3d(const double* __restrict__ in, double* __restrict__ out,
                                                int64_t N0, int64_t N1, int64_t N2, const W3<R> W) {
  constexpr int n = 2 * R + 1;
  constexpr int SH = D3_BY + 2 * R, SW = D3_BX + 2 * R;
  __shared__ double pl[2][SH][SW + 1];
  const int64_t P1 = N1 + 2 * R, P2 = N2 + 2 * R;
  const int64_t x0 = int64_t(blockIdx.x) * D3_BX, y0 = int64_t(blockIdx.y) * D3_BY;
  const int64_t z0 = int64_t(blockIdx.z) * D3_ZC;                   // first output (interior z)
  const int64_t z1 = (z0 + D3_ZC < N0) ? z0 + D3_ZC : N0;
  const int tid = threadIdx.y * D3_BX + threadIdx.x, tx = threadIdx.x, ty = threadIdx.y;
  double acc[n];
#pragma unroll
  for (int k = 0; k < n; ++k) acc[k] = 0.0;
  // input planes (padded z) p = z0 .. z1 + 2R - 1; output (interior z) zo = p - a0 uses plane p with weight a0.
  const int64_t pz_end = z1 + 2 * R;
  int buf = 0;
  for (int64_t p = z0; p < pz_end; ++p, buf ^= 1) {
    for (int i = tid; i < SH * SW; i += 256) {
      int r = i / SW, c = i % SW;
      int64_t gy = y0 + r, gx = x0 + c;
      pl[buf][r][c] = (gy < P1 && gx < P2) ? in[(p * P1 + gy) * P2 + gx] : 0.0;
    }
    __syncthreads();
    double x[n][n];
#pragma unroll
    for (int a1 = 0; a1 < n; ++a1)
#pragma unroll
      for (int a2 = 0; a2 < n; ++a2) x[a1][a2] = pl[buf][ty + a1][tx + a2];
    // ring: acc[k] accumulates output zo = p - (2R - k)... shift after each plane.
    // output zo receives planes zo .. zo + 2R (padded), plane p contributes with a0 = p - zo.
#pragma unroll
    for (int k = 0; k < n; ++k) {
      // acc[k] holds output zo = p - k  (a0 = k)
#pragma unroll
      for (int a1 = 0; a1 < n; ++a1)
#pragma unroll
        for (int a2 = 0; a2 < n; ++a2) acc[k] = fma(W.w[(k * n + a1) * n + a2], x[a1][a2], acc[k]);
    }
    // acc[2R] (output zo = p - 2R) is complete
    const int64_t zo = p - 2 * R;
    const int64_t gx = x0 + tx, gy = y0 + ty;
    if (zo >= z0 && gx < N2 && gy < N1) out[((zo + R) * P1 + gy + R) * P2 + gx + R] = acc[2 * R];
#pragma unroll
    for (int k = 2 * R; k > 0; --k) acc[k] = acc[k - 1];
    acc[0] = 0.0;
  }
}

// ---------------------------------------------------------------- halo copy
// One CTA per padded row (2D) or per padded (z, y) row (3D): halo rows are copied whole,
// interior rows only their 2R edge cells.
__global__ void copy_halo_kernel(const double* __restrict__ in, double* __restrict__ dst, int ndim, int R,
                                 int64_t P0, int64_t P1, int64_t P2) {
  const int64_t row = blockIdx.x + int64_t(blockIdx.y) * gridDim.x;
  const int64_t W = ndim == 2 ? P1 : P2;
  int64_t nrows = ndim == 2 ? P0 : P0 * P1;
  if (row >= nrows) return;
  bool halo_row;
  if (ndim == 2) halo_row = row < R || row >= P0 - R;
  else {
    int64_t z = row / P1, y = row % P1;
    halo_row = z < R || z >= P0 - R || y < R || y >= P1 - R;
  }
  const double* s = in + row * W;
  double* d = dst + row * W;
  if (halo_row) {
    for (int64_t i = threadIdx.x; i < W; i += blockDim.x) d[i] = s[i];
  } else if (threadIdx.x < 2 * R) {
    int64_t i = threadIdx.x < R ? threadIdx.x : W - 2 * R + threadIdx.x;
    d[i] = s[i];
  }
}

}  // namespace

__global__ void copy_halo_1d(const double* __restrict__ in, double* __restrict__ dst, int R, int64_t P0) {
  const int i = threadIdx.x;
  if (i < R) dst[i] = in[i];
  else if (i < 2 * R) dst[P0 - 2 * R + i] = in[P0 - 2 * R + i];
}

cudaError_t launch_copy_halo(const Plan& p, const double* in, double* dst, cudaStream_t s) {
  if (p.ndim == 1) {
    copy_halo_1d<<<1, 32, 0, s>>>(in, dst, p.R, p.P[0]);
    return cudaGetLastError();
  }
  int64_t rows = p.ndim == 2 ? p.P[0] : p.P[0] * p.P[1];
  dim3 grid((unsigned)std::min<int64_t>(rows, 65535), (unsigned)((rows + 65534) / 65535));
  copy_halo_kernel<<<grid, 128, 0, s>>>(in, dst, p.ndim, p.R, p.P[0], p.P[1], p.P[2]);
  return cudaGetLastError();
}

template <int R>
static cudaError_t direct_r(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  constexpr int n = 2 * R + 1;
  {
    W3<R> w{};
    for (int i = 0; i < n * n * n; ++i) w.w[i] = p.W[i];
    dim3 grid((unsigned)((p.N[2] + D3_BX - 1) / D3_BX), (unsigned)((p.N[1] + D3_BY - 1) / D3_BY),
              (unsigned)((p.N[0] + D3_ZC - 1) / D3_ZC));
    direct3d<R><<<grid, dim3(D3_BX, D3_BY), 0, s>>>(src, dst, p.N[0], p.N[1], p.N[2], w);
  }
  return cudaGetLastError();
}

cudaError_t launch_direct(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  if (p.ndim == 1) return launch_1d(p, src, dst, s, 1);
  if (p.ndim == 2) return launch_direct2d_stream(p, src, dst, s);
  if (p.ndim == 3 && p.R <= 2) return launch_direct3d_stream(p, src, dst, s);
  switch (p.R) {
    case 1: return direct_r<1>(p, src, dst, s);
    case 2: return direct_r<2>(p, src, dst, s);
    case 3: return direct_r<3>(p, src, dst, s);
    case 4: return direct_r<4>(p, src, dst, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace lora
