// Device side of the device-initiated halo exchange (host side csrc/dist_p2p.cu,
// argument block P2PArgs in kernels.hpp).
//
// Memory-model recipe (PTX ISA memory consistency model, system scope because the peer is another
// GPU reached over NVLink, or another process's IPC mapping):
//   producer: each lane st.global its rows into the peer's halo; each lane fence.sc.sys
//             (__threadfence_system); __syncwarp; lane 0 st.release.sys flag = step value.
//   consumer: lane 0 ld.acquire.sys flag until >= expected; fence.proxy.async.global so that the
//             TMA (async proxy) reads issued afterwards observe the peer's generic-proxy stores;
//             __syncwarp before the LDGSTS path's lanes read.
// Flags are monotonic 64-bit step counters, so no reset is ever needed between steps or runs.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.hpp"

namespace lora {

__device__ __forceinline__ unsigned long long p2p_ld_acquire(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void p2p_st_release(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

__device__ __forceinline__ unsigned long long p2p_clock_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Spin (one thread) until flags[u] >= val for u in [u0, u1].  Gives up after kP2PTimeoutNs and
// raises the device error word instead of hanging the GPU (the result is then invalid and
// lora_stencil_p2p_status reports it).
#ifndef LORA_P2P_TIMEOUT_S
#define LORA_P2P_TIMEOUT_S 20
#endif
constexpr unsigned long long kP2PTimeoutNs = LORA_P2P_TIMEOUT_S * 1000ull * 1000 * 1000;

__device__ __forceinline__ void p2p_wait_units(const unsigned long long* flags, int u0, int u1,
                                               unsigned long long val, int* err) {
  unsigned long long t0 = 0;
  for (int u = u0; u <= u1; ++u) {
    while (p2p_ld_acquire(flags + u) < val) {
      // once any wait of this endpoint has timed out the run is void: fail fast instead of paying
      // the timeout again in every later wait
      if (*reinterpret_cast<volatile int*>(err)) return;
      const unsigned long long now = p2p_clock_ns();
      if (t0 == 0) t0 = now;
      else if (now - t0 > kP2PTimeoutNs) { atomicExch(err, 1); return; }
      __nanosleep(128);
    }
  }
}

// Warp-uniform form of p2p_wait_units, called by EVERY lane of a warp: lane 0 does the acquire
// loads and the timeout bookkeeping, the loop decisions are broadcast by shuffles, so the loop
// exits are warp-uniform.  (A spin loop of lane 0 alone inside the 2D stream kernel made ptxas keep
// the stencil weights in vector registers for the whole kernel: 364 vs 429 GS/s single-GPU.)
__device__ __forceinline__ void p2p_wait_units_warp(const unsigned long long* flags, int u0, int u1,
                                                    unsigned long long val, int* err) {
  const bool l0 = (threadIdx.x & 31) == 0;
  unsigned long long t0 = 0;
  for (int u = u0; u <= u1; ++u) {
    for (;;) {
      int st = 0;   // 0: wait, 1: ready, 2: give up
      if (l0) {
        if (p2p_ld_acquire(flags + u) >= val) st = 1;
        else if (*reinterpret_cast<volatile int*>(err)) st = 2;
        else {
          const unsigned long long now = p2p_clock_ns();
          if (t0 == 0) t0 = now;
          else if (now - t0 > kP2PTimeoutNs) { atomicExch(err, 1); st = 2; }
        }
      }
      st = __shfl_sync(0xffffffffu, st, 0);
      if (st == 2) return;
      if (st == 1) break;
      __nanosleep(128);
    }
  }
}

// Called by every lane of the warp after its last store of a boundary item: publishes `val` in the
// peer's flag `u` once every lane's stores are visible system-wide.
__device__ __forceinline__ void p2p_signal_warp(unsigned long long* peer_flags, int u, unsigned long long val) {
  __threadfence_system();
  __syncwarp();
  if ((threadIdx.x & 31) == 0) p2p_st_release(peer_flags + u, val);
  __syncwarp();
}

// Chunk order of a slab's stream items when the exchange is on: the two boundary chunks first
// (0, then nch-1), so that their signals go out early in every step, then the interior chunks.
__device__ __forceinline__ int p2p_chunk_order(int c, int nch) {
  if (nch < 3) return c;
  return c == 0 ? 0 : (c == 1 ? nch - 1 : c - 1);
}

}  // namespace lora
