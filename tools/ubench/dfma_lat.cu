// DFMA / DADD latency and throughput vs ILP and warps per SM (sm_100a).
#include <cstdio>
#include <cuda_runtime.h>
template <int ILP>
__global__ void chain(double* out, long long* cyc, int iters, double a, double b) {
  double d[ILP];
#pragma unroll
  for (int i = 0; i < ILP; ++i) d[i] = threadIdx.x * 1e-9 + i;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
      for (int i = 0; i < ILP; ++i) d[i] = fma(d[i], a, b);
  }
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int i = 0; i < ILP; ++i) s += d[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int ILP>
void run(int warps_per_sm, int nsm) {
  double* o; long long* c;
  int threads = 32 * warps_per_sm;  // one CTA per SM
  cudaMalloc(&o, sizeof(double) * threads * nsm); cudaMalloc(&c, sizeof(long long) * nsm);
  int iters = 2000;
  chain<ILP><<<nsm, threads>>>(o, c, iters, 1.0000001, 1e-7);
  cudaDeviceSynchronize();
  chain<ILP><<<nsm, threads>>>(o, c, iters, 1.0000001, 1e-7);
  cudaDeviceSynchronize();
  long long h; cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
  double fmas_per_warp = double(iters) * 8 * ILP;        // warp-instructions per warp
  double cyc_per_dfma_per_warp = double(h) / fmas_per_warp;
  double fma_per_clk_sm = fmas_per_warp * warps_per_sm * 32 / double(h);
  printf("{\"ilp\":%d,\"warps_per_sm\":%d,\"cycles_per_dependent_step\":%.2f,\"fma_per_clk_per_sm\":%.1f}\n", ILP, warps_per_sm,
         cyc_per_dfma_per_warp * ILP, fma_per_clk_sm);
  cudaFree(o); cudaFree(c);
}
int main() {
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  run<1>(1, nsm); run<1>(4, nsm);                    // latency
  for (int w : {4, 8, 12, 16, 32}) { run<2>(w, nsm); run<4>(w, nsm); run<8>(w, nsm); }
  return 0;
}
