// Host helpers for pipe.cuh: tensor-map encoding through the driver entry point (no -lcuda)
// and the persistent grid size (SM count x resident CTAs per SM).
#include <cuda.h>
#include <cuda_runtime.h>

#include <map>
#include <mutex>
#include <utility>

#include "pipe.cuh"

namespace lora {
namespace {
using EncodeFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                              const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                              CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeFn get_encode() {
  static EncodeFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeFn>(p);
    cudaGetLastError();
  });
  return fn;
}
}  // namespace

bool encode_tmap(CUtensorMap* map, const double* base, int rank, const int64_t* padded, const int* box) {
  EncodeFn fn = get_encode();
  if (!fn) return false;
  if (reinterpret_cast<uintptr_t>(base) & 15) return false;
  cuuint64_t dims[3], strides[2];
  cuuint32_t bdim[3], estr[3] = {1, 1, 1};
  for (int i = 0; i < rank; ++i) {
    dims[i] = (cuuint64_t)padded[rank - 1 - i];  // innermost first
    bdim[i] = (cuuint32_t)box[rank - 1 - i];
    if (bdim[i] == 0 || bdim[i] > 256) return false;
  }
  if ((bdim[0] * 8) % 16) return false;
  cuuint64_t s = 8;
  for (int i = 0; i < rank - 1; ++i) {
    s *= dims[i];
    if (s % 16) return false;
    strides[i] = s;
  }
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, (cuuint32_t)rank, const_cast<double*>(base), dims, strides,
                  bdim, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

int persistent_grid(const void* kernel, int threads, size_t smem, int64_t ntiles) {
  int dev = 0, sms = 148, occ = 1;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, smem) != cudaSuccess || occ < 1) {
    cudaGetLastError();
    occ = 1;
  }
  int64_t g = int64_t(sms) * occ;
  if (g > ntiles) g = ntiles;
  return (int)(g < 1 ? 1 : g);
}

cudaError_t kernel_setup(const void* kernel, int threads, size_t smem, int* max_grid) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, int> cache;   // (kernel, device) -> persistent grid
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lock(mu);
  auto it = cache.find({kernel, dev});
  if (it != cache.end()) { *max_grid = it->second; return cudaSuccess; }
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int g = persistent_grid(kernel, threads, smem, int64_t(1) << 40);
  cache[{kernel, dev}] = g;
  *max_grid = g;
  return cudaSuccess;
}

}  // namespace lora
