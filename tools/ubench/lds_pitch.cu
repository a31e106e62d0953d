// LDS.64 throughput for the DMMA fragment access patterns vs shared-memory row pitch (sm_100a).
// pattern 0: B fragment, lane (g,t) reads [t][g]            (t = lane&3, g = lane>>2)
// pattern 1: A fragment, lane (g,t) reads [g][t]
// pattern 2: point term, lane (g,t) reads [g][2t]
// pattern 3: grouped B, lane (g,t) reads [t][gc(g)]
// Reports cycles per LDS.64 per warp with 16 warps/SM saturating the shared-memory pipe.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(double* out, int pitch, int pattern, int iters, long long* cyc, int shift) {
  extern __shared__ double sm[];
  for (int i = threadIdx.x; i < 80 * 96; i += blockDim.x) sm[i] = i * 1e-3;
  __syncthreads();
  const int lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  int off;
  if (pattern == 0) off = t * pitch + g;
  else if (pattern == 1) off = g * pitch + t;
  else if (pattern == 2) off = g * pitch + 2 * t;
  else off = t * pitch + ((g & 1) ? 4 + (((g >> 1) + 2) & 3) : (g >> 1));
  const double* p = sm + off + shift;
  double s = 0;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      double v;
      const unsigned a = (unsigned)__cvta_generic_to_shared(p + (j & 3) * 4 * pitch + 8 * (j >> 2));
      asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
      s += v;
    }
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
  double* o; long long* c; cudaMalloc(&o, 148 * 512 * 8); cudaMalloc(&c, 148 * 8);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 80 * 96 * 8);
  for (int pattern = 0; pattern < 4; ++pattern)
    for (int pitch = 76; pitch <= 76; ++pitch)
    for (int shift = 0; shift < 16; ++shift) {
      const int iters = 20, warps = 16;
      k<<<148, warps * 32, 80 * 96 * 8>>>(o, pitch, pattern, iters, c, shift);
      cudaDeviceSynchronize();
      long long h; cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
      // per SM: warps * iters * 16 LDS.64; cycles per LDS per SM
      printf("{\"pattern\":%d,\"pitch\":%d,\"pitch_mod16\":%d,\"cyc_per_lds_per_sm\":%.3f}\n", pattern, pitch, pitch % 16,
             double(h) / (double(warps) * iters * 16));
    }
}
