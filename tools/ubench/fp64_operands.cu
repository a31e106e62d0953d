// FP64 pipe throughput vs operand pattern (B200): is ~56 % FP64-pipe activity (ncu) the ceiling of a
// DFMA/DADD/DMUL stream whose three operands are distinct registers, as in the stencil kernels?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_operands fp64_operands.cu
#include <cstdio>
#include <cuda_runtime.h>
// MODE 0: d = fma(d, a, b) (a, b shared: operand reuse); 1: d = fma(w_i, x_i, d) (distinct regs);
// 2: d = d + x_i (DADD); 3: mix 2 DFMA : 1 DADD : 1 DMUL with distinct regs; 4: as 1 + 1 INT op per FP64
struct WU { double w[16]; };
template <int MODE>
__global__ void k(double* out, int iters, double seed, const __grid_constant__ WU wp) {
  const double* wu = wp.w;
  double d[16], w[16], x[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) { d[i] = i * 1e-3 + threadIdx.x; w[i] = seed + i * 1e-7; x[i] = 1.0 - i * 1e-6; }
  const double a = seed, b = seed * 0.5;
  int acc = threadIdx.x;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      if (MODE == 0) d[i] = fma(d[i], a, b);
      if (MODE == 1) d[i] = fma(w[i], x[(i + 5) & 15], d[i]);
      if (MODE == 2) d[i] = d[i] + x[(i + 3) & 15];
      if (MODE == 3) {
        if ((i & 3) < 2) d[i] = fma(w[i], x[(i + 5) & 15], d[i]);
        else if ((i & 3) == 2) d[i] = d[i] + x[(i + 3) & 15];
        else d[i] = w[(i + 7) & 15] * x[i];
      }
      if (MODE == 4) { d[i] = fma(w[i], x[(i + 5) & 15], d[i]); acc = acc * 3 + i; }
      if (MODE == 5) d[i] = d[i] * x[(i + 5) & 15];                       // DMUL, 2 distinct regs
      if (MODE == 6) d[i] = fma(wu[i], x[(i + 5) & 15], d[i]);            // DFMA, weight from a kernel param (uniform)
    }
#pragma unroll
    for (int i = 0; i < 16; ++i) x[i] = d[(i + 1) & 15] * 1e-30 + x[i];   // keep x live / varying (1/16 extra)
  }
  double s = acc;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += d[i] + x[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int MODE>
void run(const char* name, int ctas_per_sm, int threads) {
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  int blocks = nsm * ctas_per_sm, iters = 20000;
  double* out; cudaMalloc(&out, sizeof(double) * blocks * threads);
  WU wu; for (int i = 0; i < 16; ++i) wu.w[i] = 1.0 - i * 1e-9;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k<MODE><<<blocks, threads>>>(out, iters, 1.0000001, wu);
  cudaDeviceSynchronize();
  cudaEventRecord(e0);
  k<MODE><<<blocks, threads>>>(out, iters, 1.0000001, wu);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double inst = 32.0 * iters * (double)blocks * threads;   // FP64 lane-ops (16 + 16 x-updates)
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double peak = 64.0 * nsm * clk * 1e3;                    // lane-ops/s at the max clock
  printf("{\"mode\":\"%s\",\"warps_per_sm\":%d,\"ms\":%.3f,\"Gops\":%.1f,\"frac_of_64lane_peak_at_max_clock\":%.3f}\n", name,
         ctas_per_sm * threads / 32, ms, inst / ms / 1e6, inst / (ms * 1e-3) / peak);
  cudaFree(out);
}
int main() {
  for (int c : {2, 4}) {
    run<0>("fma_shared_operands", c, 128);
    run<1>("fma_distinct_regs", c, 128);
    run<2>("dadd_distinct", c, 128);
    run<3>("mix_2fma_1add_1mul", c, 128);
    run<4>("fma_plus_int", c, 128);
    run<5>("dmul_distinct", c, 128);
    run<6>("fma_uniform_weight", c, 128);
  }
  return 0;
}
