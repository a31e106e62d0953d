// FP64 pipe throughput of the row-pair stencil's instruction mix (B200), weights in VECTOR registers
// vs UNIFORM registers (kernel parameters).  Question: does moving the stencil weights out of vector
// registers (three distinct vector operands per DFMA) raise the FP64 issue rate of the Box-2D49P
// kernel's arithmetic?  Check the SASS (cuobjdump -sass) for "DFMA R, R, UR, R" in the UNI variants.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_mix fp64_mix.cu
#include <cstdio>
#include <cuda_runtime.h>

struct W16 { double v[4][4]; double c[4]; };

// One "row" of the row-pair form (R = 3) for NC independent column pairs: 3 DADD pair sums,
// 4 x 3 DFMA horizontal gathers, 7 vertical DFMA (one DMUL) into a 7-deep shift ring.
template <bool UNI, int NC>
__global__ void __launch_bounds__(128) k(double* out, const double* __restrict__ wg, int iters, const __grid_constant__ W16 wp) {
  double v[4][4], c[4];
  if (UNI) {
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      c[a] = wp.c[a];
#pragma unroll
      for (int b = 0; b < 4; ++b) v[a][b] = wp.v[a][b];
    }
  } else {   // per-thread loads: ptxas cannot prove them uniform -> vector registers
    const double* w = wg + (threadIdx.x & 31) * 0;
    const double* wt = wg + ((threadIdx.x * 7) & 1) * 20;   // 0 for every thread, not provable
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      c[a] = wt[16 + a];
#pragma unroll
      for (int b = 0; b < 4; ++b) v[a][b] = wt[4 * a + b];
    }
    (void)w;
  }
  double x[NC][8], p[NC][7];
#pragma unroll
  for (int q = 0; q < NC; ++q) {
#pragma unroll
    for (int i = 0; i < 8; ++i) x[q][i] = 1.0 + 1e-3 * i + q + threadIdx.x;
#pragma unroll
    for (int j = 0; j < 7; ++j) p[q][j] = 0.0;
  }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int q = 0; q < NC; ++q) {
      double sp[4];
#pragma unroll
      for (int b = 1; b <= 3; ++b) sp[b] = x[q][3 - b] + x[q][3 + b];
      double t[4];
#pragma unroll
      for (int a = 0; a <= 3; ++a) {
        double ta = x[q][3];
#pragma unroll
        for (int b = 1; b <= 3; ++b) ta = fma(v[a][b], sp[b], ta);
        t[a] = ta;
      }
#pragma unroll
      for (int j = 0; j < 6; ++j) {
        const int a = j < 3 ? 3 - j : j - 3;
        p[q][j] = fma(c[a], t[a], p[q][j + 1]);
      }
      p[q][6] = c[3] * t[3];
      // next "row": rotate inputs through the outputs (keeps values bounded and live)
#pragma unroll
      for (int i = 0; i < 7; ++i) x[q][i] = x[q][i + 1];
      x[q][7] = p[q][0];
    }
  }
  double s = 0.0;
#pragma unroll
  for (int q = 0; q < NC; ++q)
#pragma unroll
    for (int j = 0; j < 7; ++j) s += p[q][j] + x[q][j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <bool UNI, int NC>
void run(const char* name, int ctas_per_sm) {
  int nsm;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int threads = 128, blocks = nsm * ctas_per_sm, iters = 4000;
  double* out;
  double* wg;
  cudaMalloc(&out, sizeof(double) * blocks * threads);
  cudaMalloc(&wg, sizeof(double) * 64);
  W16 w;
  double hw[64];
  for (int a = 0; a < 4; ++a) {
    w.c[a] = 0.25 - 0.01 * a;
    hw[16 + a] = w.c[a];
    for (int b = 0; b < 4; ++b) w.v[a][b] = hw[4 * a + b] = 0.1 / (1 + a + b);
  }
  cudaMemcpy(wg, hw, sizeof(hw), cudaMemcpyHostToDevice);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  k<UNI, NC><<<blocks, threads>>>(out, wg, iters, w);
  cudaDeviceSynchronize();
  cudaEventRecord(e0);
  k<UNI, NC><<<blocks, threads>>>(out, wg, iters, w);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double ops = 22.0 * NC * iters * (double)blocks * threads;   // FP64 lane-ops
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const double peak = 64.0 * nsm * clk * 1e3;
  printf("{\"mode\":\"%s\",\"nc\":%d,\"warps_per_sm\":%d,\"ms\":%.3f,\"Gops\":%.1f,\"frac_of_64lane_peak_at_max_clock\":%.3f,\"err\":\"%s\"}\n",
         name, NC, ctas_per_sm * threads / 32, ms, ops / ms / 1e6, ops / (ms * 1e-3) / peak,
         cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
  cudaFree(wg);
}

int main() {
  for (int c : {1, 2, 3, 4}) {
    run<false, 4>("rowpair_vector_weights", c);
    run<true, 4>("rowpair_uniform_weights", c);
    run<false, 2>("rowpair_vector_weights", c);
    run<true, 2>("rowpair_uniform_weights", c);
  }
  return 0;
}
