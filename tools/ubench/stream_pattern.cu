// Is the per-warp 64-column streaming pattern (TMA ring per warp, STG.128 rows) DRAM-efficient?
// Copies a 10246 x 10246 FP64 array interior through each pattern and reports GB/s (read+write).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)
__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, int c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(c)); }
__device__ __forceinline__ void expect(uint64_t* b, int bytes) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes) : "memory"); }
__device__ __forceinline__ void arrive(uint64_t* b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(b)) : "memory"); }
__device__ __forceinline__ void wait(uint64_t* b, int ph) {
  asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W;\n}\n" ::"r"(sa(b)), "r"(ph) : "memory"); }
__device__ __forceinline__ void tma2d(void* dst, const CUtensorMap* m, int x, int y, uint64_t* b) {
  asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
               ::"r"(sa(dst)), "l"(m), "r"(x), "r"(y), "r"(sa(b)) : "memory"); }
constexpr int R = 3, NS = 3, RC = 140;
// W warps per CTA; each warp a 64-col band (BAND = 64) or the CTA a 64*W band read with boxes of width BW
template <int W, bool COOP, int SROWS, bool TST = false>
__global__ void __launch_bounds__(W * 32) pat(const __grid_constant__ CUtensorMap map, double* out, int P1, int N0, int nbands, int nitems, const __grid_constant__ CUtensorMap omap) {
  extern __shared__ __align__(128) unsigned char sm[];
  constexpr int BW = COOP ? 136 : 70;        // box width (doubles)
  constexpr int NB = COOP ? W / 2 : 1;       // boxes per stage (coop: one per warp pair)
  constexpr int BOXB = ((SROWS * BW * 8 + 127) / 128) * 128;
  constexpr int STAGE = BOXB * NB;
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  uint64_t* full = reinterpret_cast<uint64_t*>(sm) + (COOP ? 0 : wl * NS);
  uint64_t* empty = reinterpret_cast<uint64_t*>(sm) + 64;
  unsigned char* ring = sm + 1024 + (COOP ? 0 : wl * NS * STAGE);
  const int unit = COOP ? blockIdx.x : blockIdx.x * W + wl;         // stream id
  const int TU = COOP ? gridDim.x : gridDim.x * W;
  const int SI = (RC + 2 * R + SROWS - 1) / SROWS;
  const int my = unit < nitems ? (nitems - 1 - unit) / TU + 1 : 0;
  const int nst = my * SI;
  const bool leader = COOP ? threadIdx.x == 0 : lane == 0;
  if (leader) { for (int s = 0; s < NS; ++s) { mbar_init(&full[s], 1); if (COOP) mbar_init(&empty[s], W); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  if (COOP) __syncthreads(); else __syncwarp();
  auto issue = [&](int q) {
    const int item = unit + (q / SI) * TU, j = q % SI;
    const int band = item % nbands, chunk = item / nbands;
    const int y = chunk * RC + j * SROWS;
    const int x = band * (COOP ? 64 * W : 64);
    unsigned char* dst = ring + (q % NS) * STAGE;
    if (leader) {
      expect(&full[q % NS], SROWS * BW * 8 * NB);
      for (int b = 0; b < NB; ++b) tma2d(dst + b * BOXB, &map, x + b * 128, y, &full[q % NS]);
    }
  };
  for (int q = 0; q < NS - 1 && q < nst; ++q) issue(q);
  for (int q = 0; q < nst; ++q) {
    if (q + NS - 1 < nst) {
      if (COOP && q >= 1) { if (threadIdx.x == 0) wait(&empty[(q - 1) % NS], ((q - 1) / NS) & 1); }
      issue(q + NS - 1);
    }
    wait(&full[q % NS], (q / NS) & 1);
    const int item = unit + (q / SI) * TU, j = q % SI;
    const int band = item % nbands, chunk = item / nbands;
    const double* st = reinterpret_cast<const double*>(ring + (q % NS) * STAGE);
    int sub = COOP ? wl : 0;
    const double* sb = st + (COOP ? (sub / 2) * BOXB / 8 : 0);
    const int cofs = COOP ? (sub % 2) * 64 : 0;
    const int col = (COOP ? band * 64 * W + sub * 64 : band * 64) + 2 * lane;
    if constexpr (TST) {
      // stage the 7 output rows (64 cols) in a per-warp smem buffer, then one TMA store
      double* ob = reinterpret_cast<double*>(sm + 1024 + W * NS * STAGE) + wl * 2 * SROWS * 64 + (q & 1) * SROWS * 64;
      if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      __syncwarp();
      for (int i = 0; i < SROWS; ++i) {
        double2 v = *reinterpret_cast<const double2*>(sb + i * BW + cofs + 2 * lane + 2);
        *reinterpret_cast<double2*>(ob + i * 64 + 2 * lane) = v;
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      const int y = chunk * RC + j * SROWS;
      if (lane == 0) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                     ::"l"(&omap), "r"(col + R + 1), "r"(y), "r"(sa(ob)) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    } else {
    for (int i = 0; i < SROWS; ++i) {
      const int y = chunk * RC + j * SROWS + i - R;   // "output" row
      double2 v = *reinterpret_cast<const double2*>(sb + i * BW + cofs + 2 * lane + 2);
      if (y >= chunk * RC && y < chunk * RC + RC && y < N0)
        *reinterpret_cast<double2*>(out + int64_t(y + R) * P1 + R + col + 1) = v;
    }
    }
    __syncwarp();
    if (COOP && lane == 0) arrive(&empty[q % NS]);
  }
  if constexpr (TST) { if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
}
__global__ void plain_copy(const double2* __restrict__ a, double2* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}
using EncodeFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                              const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                              CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
template <int W, bool COOP, int SROWS, bool TST = false>
int run(EncodeFn enc, double* a, double* b, int P, const char* name) {
  constexpr int BW = COOP ? 136 : 70;
  CUtensorMap map;
  cuuint64_t dims[2] = {(cuuint64_t)P, (cuuint64_t)P}, str[1] = {(cuuint64_t)P * 8};
  cuuint32_t box[2] = {BW, SROWS}, es[2] = {1, 1};
  enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, a, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  CUtensorMap omap;
  cuuint32_t obox[2] = {64, SROWS};
  enc(&omap, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, b, dims, str, obox, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  const int N = P - 2 * R;
  const int nbands = (N + (COOP ? 64 * W : 64) - 1) / (COOP ? 64 * W : 64);
  const int nitems = nbands * ((N + RC - 1) / RC);
  constexpr int STAGE = ((SROWS * BW * 8 + 127) / 128) * 128 * (COOP ? W / 2 : 1);
  const int smem = 1024 + (COOP ? 1 : W) * NS * STAGE + (TST ? W * 2 * SROWS * 64 * 8 : 0);
  CK(cudaFuncSetAttribute(pat<W, COOP, SROWS, TST>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, pat<W, COOP, SROWS, TST>, W * 32, smem);
  const int units = COOP ? nitems : (nitems + W - 1) / W;
  const int grid = std::min(148 * occ, units);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  pat<W, COOP, SROWS, TST><<<grid, W * 32, smem>>>(map, b, P, N, nbands, nitems, omap);
  CK(cudaDeviceSynchronize());
  float best = 1e9;
  for (int r = 0; r < 5; ++r) { cudaEventRecord(e0); pat<W, COOP, SROWS, TST><<<grid, W * 32, smem>>>(map, b, P, N, nbands, nitems, omap); cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1)); float ms; cudaEventElapsedTime(&ms, e0, e1); best = std::min(best, ms); }
  printf("{\"pattern\":\"%s\",\"srows\":%d,\"occ\":%d,\"grid\":%d,\"GBps\":%.0f}\n", name, SROWS, occ, grid, 2.0 * double(N) * N * 8 / best / 1e6);
  return 0;
}
#include <algorithm>
int main() {
  void* p; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  EncodeFn enc = (EncodeFn)p;
  const int P = 10246;
  double *a, *b; CK(cudaMalloc(&a, (size_t)P * P * 8)); CK(cudaMalloc(&b, (size_t)P * P * 8));
  cudaMemset(a, 0, (size_t)P * P * 8);
  run<4, false, 7>(enc, a, b, P, "warp64_x4");
  run<4, false, 7, true>(enc, a, b, P, "warp64_x4_tmastore");
  run<4, false, 14, true>(enc, a, b, P, "warp64_x4_tmastore");
  run<8, false, 7, true>(enc, a, b, P, "warp64_x8_tmastore");
  size_t n = (size_t)P * P / 2;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) { cudaEventRecord(e0); plain_copy<<<148 * 8, 512>>>((double2*)a, (double2*)b, n); cudaEventRecord(e1);
    cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1); best = std::min(best, ms); }
  printf("{\"pattern\":\"plain_copy\",\"GBps\":%.0f}\n", 2.0 * n * 16 / best / 1e6);
}
