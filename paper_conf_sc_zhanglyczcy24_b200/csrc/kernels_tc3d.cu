// K2 on tensor cores — LoRAStencil-3D, §IV-C Alg. 2 as published:
// the (2R+1)^3 stencil is the sum over its z-planes W_{a0}; a plane with a single weight is a
// point-wise multiply-add on CUDA cores (Alg. 2 lines 3-5: DFMA), every other plane is a 2D
// LoRAStencil on tensor cores (lines 7-8): its rank-1 terms as RDG chains U X V on DMMA m8n8k4
// with Butterfly Vector Swapping (tc_terms.cuh), star planes as single-stage arms.
//
// B200 mapping: a persistent CTA (8 warps) owns a 64x64 (y, x) column of the domain and streams
// a chunk of ZC output planes along z.  Each input plane arrives once through a 3-stage TMA ring
// (3D box 1 x (64+2R+4) x 76, zero fill); for every plane operator a0 the warp computes the 8x64
// result P and adds it into the accumulator fragments of output plane z = p - a0 (a register ring
// of 2R+1 planes); z-symmetric plane pairs (W_a0 == W_{2R-a0}) are computed once and added twice.
// Radius 1 only (the accumulator ring of larger radii does not fit the register file).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <utility>

#include "kernels.hpp"
#include "pipe.cuh"
#include "tc_terms.cuh"

namespace lora {
namespace {
using namespace tc;

constexpr int T3_NS = 3;
constexpr int T3_ZC = 32;

struct Tc3Planes {
  int k0[kMaxN], k1[kMaxN];  // term range of plane a0 in TcParams (terms sorted by plane)
  int mirror[kMaxN];         // plane a0 < R also feeds output z = p - (2R - a0)
};

template <int R>
struct T3G {
  static constexpr int n = 2 * R + 1;
  static constexpr int SH = tc_rows<R>();
  static constexpr int BUF = ((SH * TC_PITCH * 8 + 127) / 128) * 128;  // bytes per stage
  static constexpr int SI = ((T3_ZC + 2 * R + n - 1) / n) * n;          // planes per item (multiple of n)
  static constexpr int SMEM = 128 + T3_NS * BUF;
};

template <int R, int A0, int I>
__device__ __forceinline__ void plane_op(const double* __restrict__ X, int w, int g, int t, const TcParams& prm,
                                         const Tc3Planes& pl, double (&acc)[2 * R + 1][8][2]) {
  constexpr int n = 2 * R + 1;
  if constexpr (A0 < n) {
    const bool skip = pl.k0[A0] == pl.k1[A0] || (A0 > R && pl.mirror[2 * R - A0]);
    if (!skip) {
      constexpr int s1 = (((I - A0) % n) + n) % n;
      constexpr int s2 = (((I - (n - 1 - A0)) % n) + n) % n;
      double P[8][2];
#pragma unroll
      for (int ob = 0; ob < 8; ++ob) { P[ob][0] = 0.0; P[ob][1] = 0.0; }
      apply_terms<R>(X, w, g, t, prm, pl.k0[A0], pl.k1[A0], P);
#pragma unroll
      for (int ob = 0; ob < 8; ++ob) { acc[s1][ob][0] += P[ob][0]; acc[s1][ob][1] += P[ob][1]; }
      if (A0 < R && pl.mirror[A0]) {
#pragma unroll
        for (int ob = 0; ob < 8; ++ob) { acc[s2][ob][0] += P[ob][0]; acc[s2][ob][1] += P[ob][1]; }
      }
    }
    plane_op<R, A0 + 1, I>(X, w, g, t, prm, pl, acc);
  }
}

template <int R, bool TMA>
__global__ void __launch_bounds__(256, 1) tc3d_kernel(const double* __restrict__ in, double* __restrict__ out,
                                                      int64_t N0, int64_t N1, int64_t N2, int ntx, int nty, int nitems,
                                                      const __grid_constant__ CUtensorMap tmap,
                                                      const __grid_constant__ TcParams prm,
                                                      const __grid_constant__ Tc3Planes pl) {
  using G = T3G<R>;
  constexpr int n = G::n;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem_raw);
  unsigned char* ring = smem_raw + 128;
  const int64_t P1 = N1 + 2 * R, P2 = N2 + 2 * R;
  const int P0 = (int)(N0 + 2 * R);
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5, g = lane >> 2, t = lane & 3;
  const int my_items = blockIdx.x < nitems ? (nitems - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const int nstages = my_items * G::SI;
  if (TMA && tid == 0) {
    for (int s = 0; s < T3_NS; ++s) mbar_init(&bar[s], 1);
    fence_barrier_init();
  }
  __syncthreads();
  auto geom = [&](int item, int& x0, int& y0, int& z0) {
    const int tx = item % ntx, rest = item / ntx, ty = rest % nty, tz = rest / nty;
    x0 = tx * TC_BN;
    y0 = ty * TC_BM;
    z0 = tz * T3_ZC;
  };
  int pitem = blockIdx.x, pj = 0, px = 0, py = 0, pz = 0;
  if (pitem < nitems) geom(pitem, px, py, pz);
  auto issue_next = [&](int slot) {
    double* dst = reinterpret_cast<double*>(ring + slot * G::BUF);
    const int z = pz + pj;
    if constexpr (TMA) {
      if (tid == 0) {
        fence_proxy_async();
        mbar_arrive_expect_tx(&bar[slot], G::SH * TC_PITCH * 8);
        tma_load_3d(dst, &tmap, px, py, z, &bar[slot]);
      }
    } else {
      for (int i = tid; i < G::SH * TC_PITCH; i += blockDim.x) {
        const int r = i / TC_PITCH, c = i - r * TC_PITCH;
        const int64_t gy = py + r, gx = px + c;
        if (z < P0 && gy < P1 && gx < P2) cp_async8(dst + i, in + (int64_t(z) * P1 + gy) * P2 + gx);
        else dst[i] = 0.0;
      }
      cp_async_commit();
    }
    if (++pj == G::SI) {
      pj = 0;
      pitem += gridDim.x;
      if (pitem < nitems) geom(pitem, px, py, pz);
    }
  };
  for (int q = 0; q < T3_NS - 1; ++q) {
    if (q < nstages) issue_next(q);
    else if constexpr (!TMA) cp_async_commit();
  }
  double acc[n][8][2];
  int citem = blockIdx.x, cj = 0, slot = 0, phase = 0, cz = 0, zend = 0;
  int x0 = 0, y0 = 0;
  for (int q0 = 0; q0 < nstages; q0 += n) {
    auto one = [&](auto Ic) {
      constexpr int I = decltype(Ic)::value;
      const int q = q0 + I;
      if (q + T3_NS - 1 < nstages) issue_next((slot + T3_NS - 1) % T3_NS);
      else if constexpr (!TMA) cp_async_commit();
      if constexpr (TMA) {
        mbar_wait(&bar[slot], phase);
      } else {
        cp_async_wait<T3_NS - 1>();
        __syncthreads();
      }
      if (cj == 0) {
        int z0;
        geom(citem, x0, y0, z0);
        cz = z0;
        zend = (int)(int64_t(z0) + T3_ZC < N0 ? int64_t(z0) + T3_ZC : N0);
#pragma unroll
        for (int s = 0; s < n; ++s)
#pragma unroll
          for (int ob = 0; ob < 8; ++ob) { acc[s][ob][0] = 0.0; acc[s][ob][1] = 0.0; }
      }
      const double* X = reinterpret_cast<const double*>(ring + slot * G::BUF);
      plane_op<R, 0, I>(X, w, g, t, prm, pl, acc);
      // output plane zi = (input plane) - 2R is complete: ring slot (I - 2R) mod n == (I + 1) mod n
      constexpr int s = (I + 1) % n;
      const int zi = cz + cj - 2 * R;
      const int64_t gy = int64_t(y0) + 8 * w + g;
      if (cj >= 2 * R && zi < zend && gy < N1) {
        double* orow = out + ((int64_t(zi) + R) * P1 + gy + R) * P2 + R;
#pragma unroll
        for (int ob = 0; ob < 8; ++ob) {
          const int64_t gx = int64_t(x0) + 8 * ob + 2 * t;
          if (gx < N2) orow[gx] = acc[s][ob][0];
          if (gx + 1 < N2) orow[gx + 1] = acc[s][ob][1];
        }
      }
#pragma unroll
      for (int ob = 0; ob < 8; ++ob) { acc[s][ob][0] = 0.0; acc[s][ob][1] = 0.0; }
      __syncthreads();  // every warp is done with this slot before it is refilled
      if (++slot == T3_NS) { slot = 0; phase ^= 1; }
      if (++cj == G::SI) { cj = 0; citem += gridDim.x; }
    };
    [&]<int... Is>(std::integer_sequence<int, Is...>) {
      (one(std::integral_constant<int, Is>{}), ...);
    }(std::make_integer_sequence<int, n>{});
  }
}

bool make_params_tc3(const Plan& p, TcParams& prm, Tc3Planes& pl) {
  std::memset(&prm, 0, sizeof(prm));
  std::memset(&pl, 0, sizeof(pl));
  const int R = p.R, n = 2 * R + 1;
  if (p.ndim != 3 || R != 1) return false;
  int k = 0;
  for (int a0 = 0; a0 < n; ++a0) {
    pl.k0[a0] = k;
    for (const Term& t : p.terms) {
      if (t.plane != a0) continue;
      if (k >= TC_MAXT) return false;
      TcTerm& d = prm.t[k++];
      d.r = t.r < 1 ? 1 : t.r;
      for (int i = 0; i < n; ++i) { d.u[i] = t.u[i]; d.v[i] = t.v[i]; }
      d.ic = R; d.jc = R;
      if (t.kind == kChain) d.kind = 0;
      else if (t.kind == kArm) {
        bool u_unit = true;
        for (int i = 0; i < n; ++i) if (t.u[i] != (i == R ? 1.0 : 0.0)) u_unit = false;
        d.kind = u_unit ? 1 : 2;
      } else {
        d.kind = 3;
        for (int i = 0; i < n; ++i) if (t.u[i] != 0.0) d.ic = i;
        for (int j = 0; j < n; ++j) if (t.v[j] != 0.0) d.jc = j;
      }
    }
    pl.k1[a0] = k;
  }
  prm.nterms = k;
  for (int a0 = 0; a0 < R; ++a0) {
    bool same = true;
    for (int e = 0; e < n * n; ++e)
      if (p.W[size_t(a0) * n * n + e] != p.W[size_t(n - 1 - a0) * n * n + e]) { same = false; break; }
    pl.mirror[a0] = same ? 1 : 0;
  }
  return true;
}

template <int R, bool TMA>
cudaError_t tc3d_launch(const Plan& p, const double* src, double* dst, cudaStream_t s, const CUtensorMap& map,
                        const TcParams& prm, const Tc3Planes& pl) {
  using G = T3G<R>;
  int max_grid = 0;
  {
    cudaError_t e = kernel_setup((const void*)tc3d_kernel<R, TMA>, 256, G::SMEM, &max_grid);
    if (e != cudaSuccess) return e;
  }
  const int ntx = (int)((p.N[2] + TC_BN - 1) / TC_BN), nty = (int)((p.N[1] + TC_BM - 1) / TC_BM);
  const int ntz = (int)((p.N[0] + T3_ZC - 1) / T3_ZC);
  const int64_t nitems = int64_t(ntx) * nty * ntz;
  const int grid = (int)std::min<int64_t>(max_grid, nitems);
  tc3d_kernel<R, TMA><<<grid, 256, G::SMEM, s>>>(src, dst, p.N[0], p.N[1], p.N[2], ntx, nty, (int)nitems, map, prm, pl);
  return cudaGetLastError();
}

}  // namespace

bool tc3d_supported(const Plan& p) {
  TcParams prm;
  Tc3Planes pl;
  return make_params_tc3(p, prm, pl);
}

cudaError_t launch_tc3d(const Plan& p, const double* src, double* dst, cudaStream_t s) {
  TcParams prm;
  Tc3Planes pl;
  if (!make_params_tc3(p, prm, pl)) return cudaErrorNotSupported;
  using G = T3G<1>;
  CUtensorMap map;
  const int64_t padded[3] = {p.P[0], p.P[1], p.P[2]};
  const int box[3] = {1, G::SH, TC_PITCH};
  if (!p.force_no_tma && encode_tmap(&map, src, 3, padded, box)) return tc3d_launch<1, true>(p, src, dst, s, map, prm, pl);
  std::memset(&map, 0, sizeof(map));
  return tc3d_launch<1, false>(p, src, dst, s, map, prm, pl);
}

}  // namespace lora
