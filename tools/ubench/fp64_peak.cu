// FP64 pipe peak on sm_100a, for the roofline denominator of the FP64-issue-bound stencil kernels
// (bench.py roofline "alu" view).  Each thread runs 16 independent dependency chains (DFMA latency
// 8 cycles x 2-cycle issue per warp instruction: 16 chains per warp keep the pipe busy at >= 4 warps
// per scheduler) for `iters` iterations; every SM holds 2 CTAs x 512 threads.  Ops:
//   dfma_u : d = fma(d, a, b) with a, b kernel parameters (uniform operands: the stencil weights)
//   dfma_v : d = fma(d, x, y) with x, y per-thread registers (three vector operands)
//   dadd   : d = d + a ;  dmul : d = d * a
// Prints one JSON line per op: FP64 lane-ops/s (one DFMA = one lane-op = 2 flops), elapsed ms
// (CUDA events).  The SM clock comes from NVML in tools/fp64_peak.py (clock64 on B200 does not tick at
// the SM clock: cycles / elapsed time gives ~1.47 GHz while NVML reports 1965 MHz under load).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_peak fp64_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("{\"error\":\"%s\",\"line\":%d}\n", cudaGetErrorString(e_), __LINE__); return 1; } } while (0)

template <int OP>
__global__ void __launch_bounds__(512, 2) fp64_kernel(double* out, long long* cyc, int iters, double a, double b) {
  double d[16];
  const double x = 1.0 + threadIdx.x * 1e-12, y = 1e-9 * blockIdx.x;
#pragma unroll
  for (int i = 0; i < 16; ++i) d[i] = 1.0 + i * 1e-7;
  const long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      if (OP == 0) d[i] = fma(d[i], a, b);
      if (OP == 1) d[i] = fma(d[i], x, y);
      if (OP == 2) d[i] = d[i] + a;
      if (OP == 3) d[i] = d[i] * a;
    }
  }
  const long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += d[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int OP>
int run(const char* name, int nsm, int iters) {
  const int blocks = 2 * nsm, threads = 512;
  double* out; long long* cyc;
  CK(cudaMalloc(&out, sizeof(double) * blocks * threads));
  CK(cudaMalloc(&cyc, sizeof(long long) * blocks));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  fp64_kernel<OP><<<blocks, threads>>>(out, cyc, iters / 10, 1.0000000001, 1e-12);   // warm-up (clocks ramp)
  CK(cudaDeviceSynchronize());
  cudaEventRecord(e0);
  fp64_kernel<OP><<<blocks, threads>>>(out, cyc, iters, 1.0000000001, 1e-12);
  cudaEventRecord(e1);
  CK(cudaDeviceSynchronize());
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  long long* h = new long long[blocks];
  CK(cudaMemcpy(h, cyc, sizeof(long long) * blocks, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (int i = 0; i < blocks; ++i) avg += (double)h[i];
  avg /= blocks;
  const double lane_ops = 16.0 * iters * (double)blocks * threads;
  const double rate = lane_ops / (ms * 1e-3);
  printf("{\"op\":\"%s\",\"ms\":%.3f,\"lane_ops_per_s\":%.6e,\"tflops\":%.3f,\"clock64_per_us\":%.0f}\n",
         name, ms, rate, (OP <= 1 ? 2.0 : 1.0) * rate / 1e12, avg / (ms * 1e3));
  fflush(stdout);
  delete[] h;
  cudaFree(out); cudaFree(cyc);
  return 0;
}

int main(int argc, char** argv) {
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  cudaDeviceProp p;
  CK(cudaGetDeviceProperties(&p, 0));
  printf("{\"device\":\"%s\",\"sms\":%d,\"cc\":\"%d.%d\"}\n", p.name, nsm, p.major, p.minor);
  const int iters = argc > 1 ? atoi(argv[1]) : 200000;   // ~2-3 s per op at full clock
  for (int rep = 0; rep < 2; ++rep) {
    run<0>("dfma_uniform", nsm, iters);
    run<1>("dfma_vector", nsm, iters);
    run<2>("dadd", nsm, iters);
    run<3>("dmul", nsm, iters);
  }
  return 0;
}
