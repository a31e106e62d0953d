// Multi-GPU slab decomposition with a DEVICE-INITIATED halo exchange (
// include/lora_stencil.h "lora_stencil_p2p_*").  The paper is single-GPU; the exchange
// step is the north star's (d).
//
// Layout.  A launch advances k steps (k = the plan's fusion depth for the 2D CUDA-core engine, else
// 1).  Each internal slab edge carries a halo of H = k R rows (physical edges keep R): the slab
// buffer has hl + n0 + hh rows (hl, hh = H or R).  The kernel sees it as a taller padded array (the
// "view"): the deep-halo rows beyond R are interior rows of the view, recomputed redundantly for the
// intermediate fused steps, and only the rank's own rows [hl, hl + n0) are stored.  Every stored row
// is computed exactly as in a single-GPU run: after j fused steps the rows within jR of the view's
// R-deep edge are wrong, and jR <= kR = H never reaches the stored rows.
//
// Protocol (per run, `base` = the endpoint's epoch, identical on every rank because every rank runs
// the same sequence of collective calls; L launches):
//   init      copy `in` into buffer 0 (rows [hl-R, hl+n0+R)), the Dirichlet ring of `in` into
//             buffer 1, publish base + 1 ("my buffers are ready"); wait for the neighbours' base + 1;
//             push my first / last H rows (full width, step 0) into both of their buffers' deep
//             halo; publish base + 2 in every flag unit.
//   launch j  buf[(j-1)%2] -> buf[j%2]: boundary items wait until the neighbour's flags of the units
//             around them reach base + 1 + j (the neighbour finished launch j-1: its edge rows are in
//             my halo, and its own launch j-1 halo reads are done, so I may overwrite its buf[j%2]
//             halo), stage, compute, store their edge rows locally AND into the neighbour's buf[j%2]
//             deep halo, then publish base + 2 + j in the neighbour's flag of their unit.
//   final     wait until my flags reach base + 2 + L, copy buf[L%2] out; epoch = base + L + 3.
// Flags are monotonic, so no reset is ever needed.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "kernels.hpp"
#include "lora_stencil.h"
#include "p2p.cuh"
#include "plan.hpp"

namespace {

constexpr uint32_t kMagic = 0x4c503250u;  // "LP2P"
constexpr uint32_t kVersion = 2;

struct Blob {                     // the 128-byte exchange handle
  uint32_t magic, version;
  cudaIpcMemHandle_t ipc;         // 64 bytes
  int64_t n0, row;                // local interior extent along the slab axis, elements per padded row/plane
  int32_t nunits, R, k, hl;       // flag units, radius, fusion depth, depth of the lower halo
  uint64_t off_buf0, off_buf1, off_flags;   // byte offsets inside the allocation
};
static_assert(sizeof(Blob) <= 128, "exchange handle must fit 128 bytes");

struct Peer {
  bool present = false;
  double* buf[2] = {nullptr, nullptr};
  unsigned long long* flags = nullptr;   // the peer's flag array [2][nunits]
  int64_t n0 = 0;
  int hl = 0;
  void* ipc_base = nullptr;              // cudaIpcOpenMemHandle mapping to close
};

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

__global__ void p2p_publish_kernel(unsigned long long* flags, int n, unsigned long long val) {
  __threadfence_system();
  for (int i = threadIdx.x; i < n; i += blockDim.x) lora::p2p_st_release(flags + i, val);
}

__global__ void p2p_wait_kernel(const unsigned long long* flags, int n, unsigned long long val, int* err) {
  if (threadIdx.x == 0) lora::p2p_wait_units(flags, 0, n - 1, val, err);
  __syncthreads();
}

// n doubles from src into two peer destinations (init push of the step-0 edge rows).
__global__ void p2p_push_kernel(const double* __restrict__ src, double* d0, double* d1, int64_t n) {
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const double v = src[i];
    d0[i] = v;
    d1[i] = v;
  }
}

}  // namespace

struct lora_p2p {
  int rank = 0, nranks = 1, device = -1;
  int ndim = 2, R = 1, engine = 0;
  int k = 1, H = 1, hl = 1, hh = 1;     // fusion depth per launch, deep-halo depth, my halo depths
  int64_t N[3] = {1, 1, 1};
  int64_t row = 0;                 // elements per padded row (2D) / plane (3D)
  size_t elems = 0;                // elements per slab buffer (hl + n0 + hh rows)
  int nunits = 0, nux = 0;         // flag units per side (max over the launch geometries)
  char* mem = nullptr;
  size_t bytes = 0;
  uint64_t off_buf[2] = {0, 0}, off_flags = 0, off_err = 0;
  double* buf[2] = {nullptr, nullptr};
  unsigned long long* flags = nullptr;   // [0][u]: written by rank-1, [1][u]: written by rank+1
  int* err = nullptr;
  Peer lo, hi;
  unsigned long long epoch = 0;
  bool poisoned = false;           // a spin-wait timed out: the flag protocol is out of step for good
};

namespace {

Peer local_peer(const lora_p2p* o) {
  Peer q;
  q.present = true;
  q.buf[0] = o->buf[0];
  q.buf[1] = o->buf[1];
  q.flags = o->flags;
  q.n0 = o->N[0];
  q.hl = o->hl;
  return q;
}

int check_layout(const lora_p2p* c, int64_t row, int nunits, int R, int k, const char* who) {
  if (row != c->row || nunits != c->nunits || R != c->R || k != c->k)
    return lora::fail(LORA_ERR_INVALID_ARG,
                      std::string(who) + " neighbour's slab layout (trailing extents / radius / fusion depth) differs");
  return LORA_OK;
}

// The kernel's view of the slab buffer: a padded array of hl + n0 + hh rows with an R-deep halo.
lora::Plan view_of(const lora::Plan& p, const lora_p2p* c) {
  lora::Plan v = p;
  v.N[0] = p.N[0] + (c->hl - p.R) + (c->hh - p.R);
  v.P[0] = v.N[0] + 2 * p.R;
  v.elems = size_t(v.P[0]) * size_t(c->row);
  v.graph_exec = nullptr;
  v.scratch = nullptr;
  v.dev_in = v.dev_out = nullptr;
  v.xbuf = nullptr;
  v.xbuf_elems = 0;
  return v;
}

}  // namespace

extern "C" {

size_t lora_stencil_p2p_handle_size(void) { return 128; }

int lora_stencil_p2p_create(lora_p2p** out, const lora_plan* p, int nranks, int rank) {
  using namespace lora;
  if (!out || !p || nranks < 1 || rank < 0 || rank >= nranks) return fail(LORA_ERR_INVALID_ARG, "bad p2p arguments");
  *out = nullptr;
  int nux = 0;
  const int nunits1 = p2p_units(*p, &nux);
  if (nunits1 <= 0)
    return fail(LORA_ERR_UNSUPPORTED, "device-initiated exchange: needs the CUDA-core engine (2D, 3D radius <= 2) or the direct kernel");
  if (nranks > 1 && p->N[0] < p->R) return fail(LORA_ERR_INVALID_ARG, "each slab needs >= radius rows/planes");
  lora_p2p* c = new (std::nothrow) lora_p2p();
  if (!c) return fail(LORA_ERR_OOM, "out of host memory");
  c->rank = rank;
  c->nranks = nranks;
  c->ndim = p->ndim;
  c->R = p->R;
  c->engine = p->engine;
  // fused launches: the CUDA-core engine keeps the plan's fusion depth (2D stream kernel, 3D radius-1
  // fused kernel); the direct comparison kernel steps unfused
  c->k = (p->engine == LORA_ENGINE_RDG_CUDA && (p->ndim == 2 || (p->ndim == 3 && rdg3d_fused_supported(*p))))
             ? std::max(1, p->fuse_k) : 1;
  c->H = c->k * p->R;
  if (nranks > 1 && p->N[0] < c->H) {
    delete c;
    return fail(LORA_ERR_INVALID_ARG, "each slab needs >= fuse_k * radius rows (the deep halo its neighbours read); plan with a smaller fuse_k");
  }
  c->hl = rank > 0 ? c->H : p->R;
  c->hh = rank < nranks - 1 ? c->H : p->R;
  for (int i = 0; i < 3; ++i) c->N[i] = p->N[i];
  c->row = p->ndim == 2 ? p->P[1] : p->P[1] * p->P[2];
  c->elems = size_t(c->hl + p->N[0] + c->hh) * size_t(c->row);
  c->nux = nux;
  {
    const lora::Plan v = view_of(*p, c);
    int nu = nunits1;
    for (int kk = 2; kk <= c->k; ++kk) nu = std::max(nu, p2p_units_k(v, kk));
    c->nunits = nu;
  }
  const size_t bb = align_up(c->elems * sizeof(double), 256);
  c->off_buf[0] = 0;
  c->off_buf[1] = bb;
  c->off_flags = 2 * bb;
  c->off_err = c->off_flags + align_up(2 * size_t(c->nunits) * sizeof(unsigned long long), 256);
  c->bytes = c->off_err + 256;
  cudaGetDevice(&c->device);
  cudaError_t e = cudaMalloc(&c->mem, c->bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    delete c;
    return fail(LORA_ERR_OOM, "cudaMalloc(p2p exchange buffers) failed");
  }
  c->buf[0] = reinterpret_cast<double*>(c->mem + c->off_buf[0]);
  c->buf[1] = reinterpret_cast<double*>(c->mem + c->off_buf[1]);
  c->flags = reinterpret_cast<unsigned long long*>(c->mem + c->off_flags);
  c->err = reinterpret_cast<int*>(c->mem + c->off_err);
  {  // load the helper kernels now: with lazy module loading a first launch while a neighbour's
     // kernel spins on this process's signals could otherwise wait on a context-wide load
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, p2p_publish_kernel);
    cudaFuncGetAttributes(&fa, p2p_wait_kernel);
    cudaFuncGetAttributes(&fa, p2p_push_kernel);
  }
  e = cudaMemset(c->mem, 0, c->bytes);   // finite values everywhere (the view's outermost rows are staged)
  if (e == cudaSuccess) {
    // Load every kernel a run launches now.  With lazy module loading (the CUDA 12 default) the
    // first launch of a kernel while a spin-waiting kernel of this process is running would wait
    // for the device, i.e. for a neighbour that in turn waits for this rank: a deadlock that only
    // the 20 s guard breaks.
    const lora::Plan v = view_of(*p, c);
    P2PArgs d;
    d.active = 1;
    d.prepare_only = 1;
    d.H = c->H;
    for (int kk = 1; kk <= c->k && e == cudaSuccess; ++kk) e = launch_step_p2p(v, c->buf[0], c->buf[1], nullptr, d, kk);
    if (e == cudaSuccess) e = launch_copy_halo(v, c->buf[0], c->buf[1], nullptr);
  }
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    cudaFree(c->mem);
    delete c;
    return cuda_fail(e, "p2p buffer initialisation");
  }
  *out = c;
  return LORA_OK;
}

int lora_stencil_p2p_get_handle(const lora_p2p* c, void* handle_out) {
  using namespace lora;
  if (!c || !handle_out) return fail(LORA_ERR_INVALID_ARG, "NULL endpoint or handle buffer");
  Blob b;
  std::memset(&b, 0, sizeof(b));
  b.magic = kMagic;
  b.version = kVersion;
  cudaError_t e = cudaIpcGetMemHandle(&b.ipc, c->mem);
  if (e != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle");
  b.n0 = c->N[0];
  b.row = c->row;
  b.nunits = c->nunits;
  b.R = c->R;
  b.k = c->k;
  b.hl = c->hl;
  b.off_buf0 = c->off_buf[0];
  b.off_buf1 = c->off_buf[1];
  b.off_flags = c->off_flags;
  std::memset(handle_out, 0, 128);
  std::memcpy(handle_out, &b, sizeof(b));
  return LORA_OK;
}

int lora_stencil_p2p_connect(lora_p2p* c, const void* lo_handle, const void* hi_handle) {
  using namespace lora;
  if (!c) return fail(LORA_ERR_INVALID_ARG, "NULL endpoint");
  if ((c->rank > 0) != (lo_handle != nullptr) || (c->rank < c->nranks - 1) != (hi_handle != nullptr))
    return fail(LORA_ERR_INVALID_ARG, "a handle is needed exactly for each existing neighbour (rank-1, rank+1)");
  const void* hs[2] = {lo_handle, hi_handle};
  Peer* ps[2] = {&c->lo, &c->hi};
  for (int k = 0; k < 2; ++k) {
    if (!hs[k]) continue;
    Blob b;
    std::memcpy(&b, hs[k], sizeof(b));
    if (b.magic != kMagic || b.version != kVersion) return fail(LORA_ERR_INVALID_ARG, "not a lora p2p handle");
    int rc = check_layout(c, b.row, b.nunits, b.R, b.k, k == 0 ? "lower" : "upper");
    if (rc) return rc;
    void* base = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&base, b.ipc, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle (neighbour in this process? use p2p_connect_local)");
    Peer& q = *ps[k];
    if (q.ipc_base) cudaIpcCloseMemHandle(q.ipc_base);
    q.present = true;
    q.ipc_base = base;
    q.buf[0] = reinterpret_cast<double*>(static_cast<char*>(base) + b.off_buf0);
    q.buf[1] = reinterpret_cast<double*>(static_cast<char*>(base) + b.off_buf1);
    q.flags = reinterpret_cast<unsigned long long*>(static_cast<char*>(base) + b.off_flags);
    q.n0 = b.n0;
    q.hl = b.hl;
  }
  return LORA_OK;
}

int lora_stencil_p2p_connect_local(lora_p2p* c, const lora_p2p* lo, const lora_p2p* hi) {
  using namespace lora;
  if (!c) return fail(LORA_ERR_INVALID_ARG, "NULL endpoint");
  const lora_p2p* os[2] = {lo, hi};
  Peer* ps[2] = {&c->lo, &c->hi};
  for (int k = 0; k < 2; ++k) {
    if (!os[k]) { *ps[k] = Peer(); continue; }
    int rc = check_layout(c, os[k]->row, os[k]->nunits, os[k]->R, os[k]->k, k == 0 ? "lower" : "upper");
    if (rc) return rc;
    if (os[k]->device != c->device) {
      int ok = 0;
      cudaDeviceCanAccessPeer(&ok, c->device, os[k]->device);
      if (!ok) return fail(LORA_ERR_UNSUPPORTED, "no peer access between the two devices");
      cudaError_t e = cudaDeviceEnablePeerAccess(os[k]->device, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_fail(e, "cudaDeviceEnablePeerAccess");
      cudaGetLastError();
    }
    *ps[k] = local_peer(os[k]);
  }
  return LORA_OK;
}

double* lora_stencil_p2p_buffer(const lora_p2p* c, int i) {
  if (!c || i < 0 || i > 1) return nullptr;
  return c->buf[i];
}

double* lora_stencil_p2p_view(const lora_p2p* c, int i) {
  if (!c || i < 0 || i > 1) return nullptr;
  return c->buf[i] + int64_t(c->hl - c->R) * c->row;   // caller row 0 = buffer row hl - R
}

int lora_stencil_run_dist_p2p(lora_plan* p, lora_p2p* c, const double* in_local, double* out_local,
                              int64_t timesteps, void* stream) {
  using namespace lora;
  if (!p || !c || !in_local || !out_local) return fail(LORA_ERR_INVALID_ARG, "NULL plan, endpoint, in or out");
  if (timesteps < 0) return fail(LORA_ERR_INVALID_ARG, "timesteps must be >= 0");
  if (p->ndim != c->ndim || p->R != c->R || p->engine != c->engine || p->N[0] != c->N[0] || p->N[1] != c->N[1] ||
      p->N[2] != c->N[2])
    return fail(LORA_ERR_INVALID_ARG, "plan does not match the endpoint's slab");
  if ((c->rank > 0 && !c->lo.present) || (c->rank < c->nranks - 1 && !c->hi.present))
    return fail(LORA_ERR_INVALID_ARG, "endpoint is not connected to its neighbours");
  if (c->poisoned)
    return fail(LORA_ERR_INVALID_ARG, "endpoint is poisoned by an earlier exchange timeout: destroy it and create a new one");
  const int R = p->R;
  const size_t bytes = p->elems * sizeof(double);          // the caller's layout (R-deep halos)
  // launches: ceil(T / k) of k steps, the last one taking the remainder
  std::vector<int> steps;
  for (int64_t done = 0; done < timesteps;) {
    const int64_t st = std::min<int64_t>(c->k, timesteps - done);
    steps.push_back((int)st);
    done += st;
  }
  const int64_t L = (int64_t)steps.size();
  // zero-copy use of the exchange buffers: in = the caller-layout view of buffer 0 and out = that of
  // buffer L%2 (lora_stencil_p2p_view; the buffers themselves for R-deep halos) may coincide (L even):
  // `in` is fully consumed by the first launch and its halo is buffer 0's own
  const int64_t vshift = int64_t(c->hl - R) * c->row;
  const bool zero_copy = in_local == c->buf[0] + vshift && out_local == c->buf[L % 2] + vshift;
  const char* a = reinterpret_cast<const char*>(in_local);
  const char* b = reinterpret_cast<const char*>(out_local);
  if (!zero_copy && a < b + bytes && b < a + bytes) return fail(LORA_ERR_ALIAS, "in and out overlap");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  int dev = -1;
  cudaGetDevice(&dev);
  if (dev != c->device) return fail(LORA_ERR_INVALID_ARG, "endpoint is bound to another CUDA device");
  int rc = ensure_device(*p, false);
  if (rc) return rc;
  if (timesteps == 0) {
    cudaError_t e = cudaMemcpyAsync(out_local, in_local, bytes, cudaMemcpyDeviceToDevice, s);
    return e == cudaSuccess ? LORA_OK : cuda_fail(e, "cudaMemcpyAsync");
  }
  const unsigned long long base = c->epoch;
  const int64_t row = c->row, n0 = c->N[0];
  const int64_t shift = int64_t(c->hl - R) * row;   // caller row 0 -> buffer row hl - R
  const lora::Plan v = view_of(*p, c);
  cudaError_t e = cudaSuccess;
  if (in_local != c->buf[0] + shift) e = cudaMemcpyAsync(c->buf[0] + shift, in_local, bytes, cudaMemcpyDeviceToDevice, s);
  if (e != cudaSuccess) return cuda_fail(e, "copy-in");
  if ((e = launch_copy_halo(*p, in_local, c->buf[1] + shift, s)) != cudaSuccess) return cuda_fail(e, "copy_halo launch");
  // init: my buffers are ready; once the neighbours' are, push my step-0 edge rows into their deep halos
  const int U = c->nunits;
  if (c->lo.present) p2p_publish_kernel<<<1, 256, 0, s>>>(c->lo.flags + U, U, base + 1);
  if (c->hi.present) p2p_publish_kernel<<<1, 256, 0, s>>>(c->hi.flags, U, base + 1);
  if (c->lo.present) p2p_wait_kernel<<<1, 32, 0, s>>>(c->flags, U, base + 1, c->err);
  if (c->hi.present) p2p_wait_kernel<<<1, 32, 0, s>>>(c->flags + U, U, base + 1, c->err);
  const int64_t H = c->H;
  if (c->lo.present) {   // my rows [hl, hl + H) -> its rows [hl_lo + n0_lo, +H)
    const int64_t to = (int64_t(c->lo.hl) + c->lo.n0) * row;
    p2p_push_kernel<<<148, 256, 0, s>>>(c->buf[0] + int64_t(c->hl) * row, c->lo.buf[0] + to, c->lo.buf[1] + to, H * row);
  }
  if (c->hi.present) {   // my rows [hl + n0 - H, hl + n0) -> its rows [0, H)
    p2p_push_kernel<<<148, 256, 0, s>>>(c->buf[0] + (int64_t(c->hl) + n0 - H) * row, c->hi.buf[0], c->hi.buf[1], H * row);
  }
  if (c->lo.present) p2p_publish_kernel<<<1, 256, 0, s>>>(c->lo.flags + U, U, base + 2);
  if (c->hi.present) p2p_publish_kernel<<<1, 256, 0, s>>>(c->hi.flags, U, base + 2);
  if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e, "p2p init launches");
  P2PArgs d;
  d.active = 1;
  d.nunits = U;
  d.nux = c->nux;
  d.wait_lo = c->lo.present ? c->flags : nullptr;
  d.wait_hi = c->hi.present ? c->flags + U : nullptr;
  d.sig_lo = c->lo.present ? c->lo.flags + U : nullptr;   // I am the lower neighbour's upper side
  d.sig_hi = c->hi.present ? c->hi.flags : nullptr;       // ... and the upper neighbour's lower side
  d.off_lo = c->lo.present ? (long long)((int64_t(c->lo.hl) + c->lo.n0 - c->hl) * row) : 0;
  d.off_hi = -(long long)((int64_t(c->hl) + n0 - H) * row);
  d.err = c->err;
  d.H = (int)H;
  d.store_lo = c->hl;
  d.store_hi = (int)(c->hl + n0);
  d.lo_end = (int)(c->hl + H);
  d.hi_begin = (int)(c->hl + n0 - H);
  auto units_of = [&](int kk) { return p2p_units_k(v, kk); };
  for (int64_t j = 1; j <= L; ++j) {
    const int kk = steps[j - 1];
    d.dst_lo = c->lo.present ? c->lo.buf[j % 2] : nullptr;
    d.dst_hi = c->hi.present ? c->hi.buf[j % 2] : nullptr;
    d.wait_val = base + 1 + (unsigned long long)j;
    d.sig_val = base + 2 + (unsigned long long)j;
    // after a launch of another band geometry (the remainder launch) wait on every unit it signalled
    d.wait_units = (j >= 2 && steps[j - 2] != kk) ? units_of(steps[j - 2]) : 0;
    e = launch_step_p2p(v, c->buf[(j - 1) % 2], c->buf[j % 2], s, d, kk);
    if (e != cudaSuccess) return cuda_fail(e, "stencil kernel launch (p2p)");
  }
  const unsigned long long fin = base + 2 + (unsigned long long)L;
  const int ulast = units_of(steps[L - 1]);
  if (c->lo.present) p2p_wait_kernel<<<1, 32, 0, s>>>(c->flags, ulast, fin, c->err);
  if (c->hi.present) p2p_wait_kernel<<<1, 32, 0, s>>>(c->flags + U, ulast, fin, c->err);
  if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e, "p2p wait launch");
  double* last = c->buf[L % 2] + shift;
  if (out_local != last) {
    e = cudaMemcpyAsync(out_local, last, bytes, cudaMemcpyDeviceToDevice, s);
    if (e != cudaSuccess) return cuda_fail(e, "copy-out");
  }
  c->epoch = base + (unsigned long long)L + 3;
  if (sync_check()) {
    cudaError_t ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "LORA_SYNC_CHECK stream sync");
    return lora_stencil_p2p_status(c);
  }
  return LORA_OK;
}

int lora_stencil_p2p_status(lora_p2p* c) {
  using namespace lora;
  if (!c) return fail(LORA_ERR_INVALID_ARG, "NULL endpoint");
  int h = 0;
  cudaError_t e = cudaMemcpy(&h, c->err, sizeof(int), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return cuda_fail(e, "p2p status read");
  if (h) {
    c->poisoned = true;   // every later run_dist_p2p on this endpoint is refused
    return fail(LORA_ERR_CUDA, "device-initiated halo exchange: a neighbour's step counter did not advance for 20 s "
                               "(endpoint poisoned: destroy and re-create it)");
  }
  return LORA_OK;
}

void lora_stencil_p2p_destroy(lora_p2p* c) {
  if (!c) return;
  if (c->lo.ipc_base) cudaIpcCloseMemHandle(c->lo.ipc_base);
  if (c->hi.ipc_base) cudaIpcCloseMemHandle(c->hi.ipc_base);
  if (c->mem) cudaFree(c->mem);
  delete c;
}

}  // extern "C"
