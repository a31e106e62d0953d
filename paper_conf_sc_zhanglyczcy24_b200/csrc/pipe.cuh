// Tile staging for the persistent stencil kernels: TMA (cp.async.bulk.tensor) + mbarrier double
// buffering, with an LDGSTS (cp.async) fallback for arrays whose row pitch is not a multiple of
// 16 bytes (TMA's global-stride rule, cuda.h cuTensorMapEncodeTiled).
//
// Both paths fill a box of `rows x cols` doubles (row pitch = cols) starting at a padded-array
// coordinate; elements outside the array are ZERO (CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE / explicit
// st.shared 0): zero band weights multiply every staged element, and 0 * NaN would be NaN.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

namespace lora {

// ------------------------------------------------------------------ device side
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Orders this thread's earlier generic-proxy shared-memory accesses before later async-proxy
// (TMA) accesses to the same buffer.
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra LAB_WAIT;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int x, int y, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(dst)),
      "l"(map), "r"(x), "r"(y), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, int x, int y, int z, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
          smem_u32(dst)),
      "l"(map), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}

__device__ __forceinline__ void cp_async8(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// TMA tile loads fault ("illegal instruction") when the innermost box start is not 16-byte aligned
// (an odd FP64 column); negative and out-of-range origins are fine and zero-filled
// (tools/ubench/tma_probe.cu).  Every caller keeps the innermost coordinate even.

// Fallback fill of a rows x cols box at padded coordinate (y, x) of a P0 x P1 array (2D) by all
// threads of the CTA with LDGSTS; zero outside the array.  Completion: cp_async_wait + barrier.
__device__ __forceinline__ void box_fill_cpasync(double* dst, const double* __restrict__ src, int64_t P0, int64_t P1,
                                                 int64_t y, int64_t x, int rows, int cols) {
  for (int i = threadIdx.x; i < rows * cols; i += blockDim.x) {
    const int r = i / cols, c = i - r * cols;
    const int64_t gy = y + r, gx = x + c;
    if (gy < P0 && gx < P1) cp_async8(dst + i, src + gy * P1 + gx);
    else dst[i] = 0.0;
  }
}

// ------------------------------------------------------------------ host side
// Encodes a 2D (rank = 2) or 3D (rank = 3) FP64 tensor map over a padded array with box
// {box_cols, box_rows[, box_planes]}.  Returns false when TMA's rules are not met (base not
// 16-byte aligned, row pitch not a multiple of 16 bytes) or the driver entry point is missing.
bool encode_tmap(CUtensorMap* map, const double* base, int rank, const int64_t* padded /*slowest first*/,
                 const int* box /*slowest first*/);

int persistent_grid(const void* kernel, int threads, size_t smem, int64_t ntiles);

// Per-device, thread-safe kernel preparation: sets the kernel's dynamic shared-memory limit on the
// CURRENT device (function attributes are per device context) the first time this (kernel, device)
// pair is seen, and returns the persistent grid size (SMs x resident CTAs) for it in *max_grid.
cudaError_t kernel_setup(const void* kernel, int threads, size_t smem, int* max_grid);

}  // namespace lora
