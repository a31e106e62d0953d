// Step-0 microbenchmark: FP64 DMMA (mma.sync.m8n8k4.f64) vs DFMA
// throughput on sm_100a, alone and co-issued, plus an FP64 copy for HBM bandwidth.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_pipes fp64_pipes.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}

// mode 0: DFMA only, mode 1: DMMA only, mode 2: both in every warp (ratio r DFMA per DMMA),
// mode 3: even warps DMMA, odd warps DFMA
template <int MODE>
__global__ void pipes(double* out, long long* cyc, int iters, double seed) {
  double a = seed + threadIdx.x * 1e-9, b = seed * 0.5;
  double c[16], d[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) { c[i] = i * 1e-3; d[i] = i * 2e-3; }
  long long t0 = clock64();
  int warp = threadIdx.x >> 5;
  for (int it = 0; it < iters; ++it) {
    if (MODE == 0 || (MODE == 3 && (warp & 1))) {
#pragma unroll
      for (int i = 0; i < 16; ++i) d[i] = fma(d[i], a, b);
    }
    if (MODE == 1 || (MODE == 3 && !(warp & 1))) {
#pragma unroll
      for (int i = 0; i < 8; ++i) dmma(c[2 * i], c[2 * i + 1], a, b);
    }
    if (MODE == 2) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        dmma(c[2 * i], c[2 * i + 1], a, b);
        d[2 * i] = fma(d[2 * i], a, b);
        d[2 * i + 1] = fma(d[2 * i + 1], a, b);
      }
    }
  }
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += c[i] + d[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

__global__ void copy2(const double2* __restrict__ in, double2* __restrict__ out, size_t n) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += stride) out[i] = in[i];
}

template <int MODE>
int run(const char* name, int blocks, int threads, int iters) {
  double* out; long long* cyc;
  CK(cudaMalloc(&out, sizeof(double) * blocks * threads));
  CK(cudaMalloc(&cyc, sizeof(long long) * blocks));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  pipes<MODE><<<blocks, threads>>>(out, cyc, iters, 1.0000001);
  CK(cudaDeviceSynchronize());
  cudaEventRecord(e0);
  pipes<MODE><<<blocks, threads>>>(out, cyc, iters, 1.0000001);
  cudaEventRecord(e1);
  CK(cudaDeviceSynchronize());
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  long long* h = new long long[blocks];
  cudaMemcpy(h, cyc, sizeof(long long) * blocks, cudaMemcpyDeviceToHost);
  double avgcyc = 0; for (int i = 0; i < blocks; ++i) avgcyc += h[i]; avgcyc /= blocks;
  int warps = blocks * threads / 32;
  // FMAs: DFMA = 16 per thread per iter (mode0), DMMA = 8*256 per warp per iter
  double dfma = 0, dmmaf = 0;
  if (MODE == 0) dfma = 16.0 * threads * blocks * (double)iters;
  if (MODE == 1) dmmaf = 8.0 * 256 * warps * (double)iters;
  if (MODE == 2) { dfma = 16.0 * threads * blocks * (double)iters; dmmaf = 8.0 * 256 * warps * (double)iters; }
  if (MODE == 3) { dfma = 16.0 * threads * blocks * (double)iters / 2; dmmaf = 8.0 * 256 * warps * (double)iters / 2; }
  double tot = dfma + dmmaf;
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  double resident_blocks_per_sm = (double)blocks / nsm;
  double fma_per_clk_sm = tot / nsm / avgcyc;  // assumes all blocks co-resident
  double implied_mhz = avgcyc / (ms * 1e3);
  printf("{\"bench\":\"%s\",\"blocks\":%d,\"threads\":%d,\"ms\":%.3f,\"TFLOPS\":%.2f,\"dfma_TF\":%.2f,\"dmma_TF\":%.2f,"
         "\"fma_per_clk_per_sm\":%.2f,\"avg_block_cycles\":%.0f,\"implied_mhz\":%.0f,\"blocks_per_sm\":%.2f}\n",
         name, blocks, threads, ms, 2 * tot / ms / 1e9, 2 * dfma / ms / 1e9, 2 * dmmaf / ms / 1e9, fma_per_clk_sm, avgcyc,
         implied_mhz, resident_blocks_per_sm);
  cudaFree(out); cudaFree(cyc); delete[] h;
  return 0;
}

int main() {
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  printf("{\"device\":\"%s\",\"sms\":%d,\"cc\":\"%d.%d\"}\n", p.name, nsm, p.major, p.minor);
  for (int t : {128, 256, 512}) {
    run<0>("dfma", nsm * 2, t, 20000);
    run<1>("dmma", nsm * 2, t, 20000);
    run<2>("dmma+dfma_same_warp", nsm * 2, t, 20000);
    run<3>("dmma|dfma_split_warps", nsm * 2, t, 20000);
  }
  // long run for clocks under sustained load
  run<1>("dmma_long", nsm * 2, 256, 400000);
  run<0>("dfma_long", nsm * 2, 256, 400000);
  // HBM copy
  size_t n = (size_t)1 << 27;  // 2^27 double2 = 2 GiB per buffer
  double2 *a, *b; CK(cudaMalloc(&a, n * 16)); CK(cudaMalloc(&b, n * 16));
  cudaMemset(a, 0, n * 16);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int blocksPerSm : {2, 4, 8}) {
    float best = 1e9;
    for (int r = 0; r < 5; ++r) {
      cudaEventRecord(e0); copy2<<<nsm * blocksPerSm, 512>>>(a, b, n); cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1)); float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    printf("{\"bench\":\"copy_fp64x2\",\"blocks_per_sm\":%d,\"GBps\":%.1f}\n", blocksPerSm, 2.0 * n * 16 / best / 1e6);
  }
  return 0;
}
