// Multi-GPU: slab decomposition along the slowest axis with a per-step halo exchange over NCCL
// (north star (d); the paper itself is single-GPU).
//
// Rank q owns interior rows (2D) or planes (3D) [s_q, s_q + n_q) of the global grid and a padded
// local array of n_q + 2R rows/planes.  Halo rows/planes are contiguous, so ncclSend/ncclRecv move
// them in place (no pack kernel).  Per time step t: step src -> dst on this rank's slab, then a
// grouped exchange fills dst's slab-edge halos with the neighbours' step-t edge rows (rank 0's low
// halo and rank n-1's high halo are the physical Dirichlet boundary and are never exchanged).
// Every point is computed with the single-GPU kernels, so the result is bitwise equal to a
// single-GPU run of the global grid (pin P10).
//
// Overlap (boundary first): each step computes the two edge strips of the slab first, the exchange
// of their edge rows then runs on the comm's own stream while the interior strip is computed; the
// next step waits for the exchange.  A strip is launched as the same kernel on a row-range view of
// the arrays (rows [r0, r1) with the rows around them as its halo), so no kernel needs a row-range
// argument and every point is computed exactly as in the full launch.
//
// NCCL is loaded at run time (dlopen of the libnccl.so.2 the process already has — torch's — or
// the system one), so the library has no link-time NCCL dependency.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>

#include "lora_stencil.h"
#include "plan.hpp"

namespace {
using ncclComm_t = struct ncclComm*;
struct ncclUniqueId { char internal[128]; };
using ncclResult_t = int;
constexpr int kNcclFloat64 = 8;

struct Nccl {
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  bool ok = false;
};

Nccl& nccl() {
  static Nccl n;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    n.GetUniqueId = (decltype(n.GetUniqueId))dlsym(h, "ncclGetUniqueId");
    n.CommInitRank = (decltype(n.CommInitRank))dlsym(h, "ncclCommInitRank");
    n.CommDestroy = (decltype(n.CommDestroy))dlsym(h, "ncclCommDestroy");
    n.Send = (decltype(n.Send))dlsym(h, "ncclSend");
    n.Recv = (decltype(n.Recv))dlsym(h, "ncclRecv");
    n.GroupStart = (decltype(n.GroupStart))dlsym(h, "ncclGroupStart");
    n.GroupEnd = (decltype(n.GroupEnd))dlsym(h, "ncclGroupEnd");
    n.GetErrorString = (decltype(n.GetErrorString))dlsym(h, "ncclGetErrorString");
    n.ok = n.GetUniqueId && n.CommInitRank && n.CommDestroy && n.Send && n.Recv && n.GroupStart && n.GroupEnd;
  });
  return n;
}

int nccl_fail(ncclResult_t r, const char* what) {
  std::string m = std::string(what) + ": NCCL error " + std::to_string(r);
  if (nccl().GetErrorString) m += std::string(" (") + nccl().GetErrorString(r) + ")";
  return lora::fail(LORA_ERR_NCCL, m);
}
}  // namespace

struct lora_comm {
  ncclComm_t comm = nullptr;
  int rank = 0, nranks = 1, device = -1;
  cudaStream_t comm_stream = nullptr;   // halo exchange runs here, overlapped with interior compute
  cudaEvent_t ev_edge = nullptr, ev_comm = nullptr;
  double* dbuf[2] = {nullptr, nullptr}; // fused runs: deep-halo slab buffers (hl + n0 + hh rows)
  size_t dbuf_elems = 0;
};

namespace {
// The halo exchange of a slab buffer whose internal edges carry H-deep halos (H = R: the caller's
// layout; H = k R: the fused path's deep-halo buffers).  Buffer rows: [0, hl) low halo, [hl, hl + n0)
// own rows, [hl + n0, hl + n0 + hh) high halo, with hl = H below a neighbour (R at the physical
// boundary), likewise hh.  My first H own rows go to rank - 1's high halo, my last H to rank + 1's
// low halo; the neighbours' rows fill mine.  All transfers are whole contiguous rows / planes.
int exchange_plan(const lora_plan* p, int rank, int nranks, int64_t H, int64_t* kind, int64_t* peer, int64_t* off,
                  int64_t* cnt) {
  const int64_t row = p->ndim == 2 ? p->P[1] : p->P[1] * p->P[2];   // elements per padded row/plane
  const int64_t n0 = p->N[0];
  const int64_t hl = rank > 0 ? H : p->R;
  int k = 0;
  if (rank > 0) {  // my first H own rows go down; the neighbour's last H fill my low halo
    kind[k] = 0; peer[k] = rank - 1; off[k] = hl * row; cnt[k] = H * row; ++k;
    kind[k] = 1; peer[k] = rank - 1; off[k] = 0; cnt[k] = H * row; ++k;
  }
  if (rank < nranks - 1) {  // my last H own rows go up; the neighbour's first H fill my high halo
    kind[k] = 0; peer[k] = rank + 1; off[k] = (hl + n0 - H) * row; cnt[k] = H * row; ++k;
    kind[k] = 1; peer[k] = rank + 1; off[k] = (hl + n0) * row; cnt[k] = H * row; ++k;
  }
  return k;
}

// Fills buf's slab-edge halos (depth H) from the neighbours (one NCCL group, stream-ordered).
int exchange(const lora_plan* p, lora_comm* c, double* buf, cudaStream_t s, int64_t H = 0) {
  if (c->nranks == 1) return LORA_OK;
  int64_t kind[4], peer[4], off[4], cnt[4];
  const int m = exchange_plan(p, c->rank, c->nranks, H > 0 ? H : p->R, kind, peer, off, cnt);
  Nccl& n = nccl();
  ncclResult_t r = n.GroupStart();
  if (r) return nccl_fail(r, "ncclGroupStart");
  for (int i = 0; i < m; ++i) {
    r = kind[i] == 0 ? n.Send(buf + off[i], size_t(cnt[i]), kNcclFloat64, (int)peer[i], c->comm, s)
                     : n.Recv(buf + off[i], size_t(cnt[i]), kNcclFloat64, (int)peer[i], c->comm, s);
    if (r) { n.GroupEnd(); return nccl_fail(r, kind[i] == 0 ? "ncclSend" : "ncclRecv"); }
  }
  if ((r = n.GroupEnd())) return nccl_fail(r, "ncclGroupEnd");
  return LORA_OK;
}
}  // namespace

extern "C" {

size_t lora_stencil_comm_id_size(void) { return sizeof(ncclUniqueId); }

int lora_stencil_dist_exchange_plan(const lora_plan* p, int rank, int nranks, int64_t* kind, int64_t* peer,
                                    int64_t* offset, int64_t* count) {
  if (!p || !kind || !peer || !offset || !count || nranks < 1 || rank < 0 || rank >= nranks)
    return lora::fail(LORA_ERR_INVALID_ARG, "bad exchange-plan arguments");
  if (nranks > 1 && p->N[0] < p->R) return lora::fail(LORA_ERR_INVALID_ARG, "each slab needs >= radius rows/planes");
  return exchange_plan(p, rank, nranks, p->R, kind, peer, offset, count);
}

int lora_stencil_dist_exchange_plan_ex(const lora_plan* p, int rank, int nranks, int64_t halo_depth, int64_t* kind,
                                       int64_t* peer, int64_t* offset, int64_t* count) {
  if (!p || !kind || !peer || !offset || !count || nranks < 1 || rank < 0 || rank >= nranks || halo_depth < p->R)
    return lora::fail(LORA_ERR_INVALID_ARG, "bad exchange-plan arguments (halo_depth must be >= radius)");
  if (nranks > 1 && p->N[0] < halo_depth)
    return lora::fail(LORA_ERR_INVALID_ARG, "each slab needs >= halo_depth rows/planes");
  return exchange_plan(p, rank, nranks, halo_depth, kind, peer, offset, count);
}

int lora_stencil_comm_get_id(void* id_out) {
  if (!id_out) return lora::fail(LORA_ERR_INVALID_ARG, "NULL id buffer");
  if (!nccl().ok) return lora::fail(LORA_ERR_NCCL, "libnccl.so.2 could not be loaded");
  ncclUniqueId id;
  ncclResult_t r = nccl().GetUniqueId(&id);
  if (r) return nccl_fail(r, "ncclGetUniqueId");
  std::memcpy(id_out, &id, sizeof(id));
  return LORA_OK;
}

int lora_stencil_comm_init(lora_comm** c, int nranks, int rank, const void* nccl_unique_id) {
  if (!c || !nccl_unique_id || nranks < 1 || rank < 0 || rank >= nranks)
    return lora::fail(LORA_ERR_INVALID_ARG, "bad comm arguments");
  *c = nullptr;
  lora_comm* cc = new (std::nothrow) lora_comm();
  if (!cc) return lora::fail(LORA_ERR_OOM, "out of host memory");
  cc->rank = rank;
  cc->nranks = nranks;
  cudaGetDevice(&cc->device);
  if (cudaStreamCreateWithFlags(&cc->comm_stream, cudaStreamNonBlocking) != cudaSuccess ||
      cudaEventCreateWithFlags(&cc->ev_edge, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&cc->ev_comm, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    lora_stencil_comm_destroy(cc);
    return lora::fail(LORA_ERR_CUDA, "stream/event creation failed");
  }
  const char* fn = std::getenv("LORA_FORCE_NCCL");  // tests: build a real (1-rank) NCCL communicator
  if (nranks > 1 || (fn && fn[0] == '1')) {
    if (!nccl().ok) { lora_stencil_comm_destroy(cc); return lora::fail(LORA_ERR_NCCL, "libnccl.so.2 could not be loaded"); }
    ncclUniqueId id;
    std::memcpy(&id, nccl_unique_id, sizeof(id));
    ncclResult_t r = nccl().CommInitRank(&cc->comm, nranks, id, rank);
    if (r) { lora_stencil_comm_destroy(cc); return nccl_fail(r, "ncclCommInitRank"); }
  }
  *c = cc;
  return LORA_OK;
}

}  // extern "C"

namespace {
// Fused run (the plan's fusion depth k > 1, CUDA-core engine): the slab lives in two comm-owned
// buffers with H = k R deep halos at internal edges, presented to the plan's own fused kernels as a
// taller padded array (the "view": its deep-halo rows count as interior and are recomputed
// redundantly; after j fused sub-steps only rows within jR of the view's R-deep edge are wrong, and
// jR <= H never reaches an own row).  Per launch: k steps on the view, then one NCCL group refills
// the H-deep halos of the result with the neighbours' rows (what the kernel wrote there is
// discarded).  Every own point is computed exactly as in a single-GPU run (pin P10).
int run_fused(lora_plan* p, lora_comm* c, const double* in_local, double* out_local, int64_t T, cudaStream_t s) {
  using namespace lora;
  const int R = p->R, k = p->fuse_k;
  const int64_t H = int64_t(k) * R, n0 = p->N[0];
  if (c->nranks > 1 && n0 < H)
    return fail(LORA_ERR_INVALID_ARG, "each slab needs >= fuse_k * radius rows/planes (plan with a smaller fuse_k)");
  const int64_t hl = c->rank > 0 ? H : R, hh = c->rank < c->nranks - 1 ? H : R;
  const int64_t row = p->ndim == 1 ? 1 : (p->ndim == 2 ? p->P[1] : p->P[1] * p->P[2]);
  const size_t elems = size_t(hl + n0 + hh) * size_t(row);
  if (c->dbuf_elems < elems) {
    for (double*& b : c->dbuf) { if (b) cudaFree(b); b = nullptr; }
    c->dbuf_elems = 0;
    for (double*& b : c->dbuf)
      if (cudaMalloc(&b, elems * sizeof(double)) != cudaSuccess) { cudaGetLastError(); return fail(LORA_ERR_OOM, "cudaMalloc(deep-halo slab buffers)"); }
    c->dbuf_elems = elems;
  }
  lora::Plan v = *p;   // the view: hl + n0 + hh rows with an R-deep halo
  v.N[0] = n0 + (hl - R) + (hh - R);
  v.P[0] = v.N[0] + 2 * R;
  v.elems = elems;
  v.graph_exec = nullptr;
  v.scratch = nullptr;
  v.dev_in = v.dev_out = nullptr;
  v.xbuf = nullptr;
  v.xbuf_elems = 0;
  const int64_t shift = (hl - R) * row;   // caller row 0 -> buffer row hl - R
  const size_t bytes = p->elems * sizeof(double);
  cudaError_t ce = cudaMemcpyAsync(c->dbuf[0] + shift, in_local, bytes, cudaMemcpyDeviceToDevice, s);
  if (ce != cudaSuccess) return cuda_fail(ce, "copy-in");
  int e = copy_halo_launch(*p, in_local, c->dbuf[1] + shift, s);   // the Dirichlet ring of the own rows
  if (e) return cuda_fail(e, "copy_halo launch");
  int rc = exchange(p, c, c->dbuf[0], s, H);                        // step-0 deep halos
  if (rc) return rc;
  int cur = 0;
  for (int64_t done = 0; done < T;) {
    const int kk = (int)std::min<int64_t>(k, T - done);
    if ((e = step_launch_k(v, c->dbuf[cur], c->dbuf[cur ^ 1], s, kk))) return cuda_fail(e, "fused stencil launch");
    cur ^= 1;
    if ((rc = exchange(p, c, c->dbuf[cur], s, H))) return rc;
    done += kk;
  }
  ce = cudaMemcpyAsync(out_local, c->dbuf[cur] + shift, bytes, cudaMemcpyDeviceToDevice, s);
  if (ce != cudaSuccess) return cuda_fail(ce, "copy-out");
  return LORA_OK;
}
}  // namespace

extern "C" {

int lora_stencil_run_dist(lora_plan* p, lora_comm* c, const double* in_local, double* out_local, int64_t timesteps,
                          void* stream) {
  using namespace lora;
  if (!p || !c || !in_local || !out_local) return fail(LORA_ERR_INVALID_ARG, "NULL plan, comm, in or out");
  if (timesteps < 0) return fail(LORA_ERR_INVALID_ARG, "timesteps must be >= 0");
  if (c->nranks > 1 && p->N[0] < p->R) return fail(LORA_ERR_INVALID_ARG, "each slab needs >= radius rows/planes");
  const size_t bytes = p->elems * sizeof(double);
  const char* a = reinterpret_cast<const char*>(in_local);
  const char* b = reinterpret_cast<const char*>(out_local);
  if (a < b + bytes && b < a + bytes) return fail(LORA_ERR_ALIAS, "in and out overlap");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  int dev = -1;
  if (cudaGetDevice(&dev) != cudaSuccess || dev != c->device)
    return fail(LORA_ERR_INVALID_ARG, "communicator is bound to another CUDA device");
  if (timesteps == 0) {
    cudaError_t e = cudaMemcpyAsync(out_local, in_local, bytes, cudaMemcpyDeviceToDevice, s);
    return e == cudaSuccess ? LORA_OK : cuda_fail(e, "cudaMemcpyAsync");
  }
  int rc = ensure_device(*p, timesteps >= 2);
  if (rc) return rc;
  const char* ff = std::getenv("LORA_DIST_FUSED");   // tests: the fused path on one rank
  if (p->engine == LORA_ENGINE_RDG_CUDA && p->fuse_k > 1 && (c->nranks > 1 || (ff && ff[0] == '1'))) {
    rc = run_fused(p, c, in_local, out_local, timesteps, s);
    if (rc == LORA_OK && sync_check()) {
      cudaError_t ce = cudaStreamSynchronize(s);
      if (ce != cudaSuccess) return cuda_fail(ce, "LORA_SYNC_CHECK stream sync");
    }
    return rc;
  }
  int e = copy_halo_launch(*p, in_local, out_local, s);
  if (e) return cuda_fail(e, "copy_halo launch");
  if (timesteps >= 2) {
    e = copy_halo_launch(*p, in_local, p->scratch, s);
    if (e) return cuda_fail(e, "copy_halo launch");
  }
  // in_local's slab-edge halos hold the neighbours' initial rows (a slice of the global padded
  // array); every later buffer gets them from the exchange after each step.
  const int64_t n0 = p->N[0];
  const int64_t row = p->ndim == 2 ? p->P[1] : p->P[1] * p->P[2];
  const int64_t B = std::max<int64_t>(p->R, std::min<int64_t>(64, n0 / 4));   // edge strip height
  const char* fs = std::getenv("LORA_DIST_SPLIT");  // tests: exercise the split path on one rank
  const bool force_split = fs && fs[0] == '1';
  const bool split = (c->nranks > 1 || force_split) && n0 >= 2 * B + 1;
  auto view = [&](int64_t r0, int64_t r1) {  // rows [r0, r1) of the local slab as a stand-alone plan
    lora::Plan v = *p;
    v.N[0] = r1 - r0;
    v.P[0] = v.N[0] + 2 * p->R;
    v.elems = size_t(v.P[0]) * size_t(row);
    v.graph_exec = nullptr;
    return v;
  };
  const lora::Plan top = split ? view(0, B) : *p, bot = split ? view(n0 - B, n0) : *p, mid = split ? view(B, n0 - B) : *p;
  const double* src = in_local;
  for (int64_t t = 1; t <= timesteps; ++t) {
    double* dst = ((timesteps - t) % 2 == 0) ? out_local : p->scratch;
    if (!split) {
      e = step_launch(*p, src, dst, s);
      if (e) return cuda_fail(e, "stencil kernel launch");
      rc = exchange(p, c, dst, s);
      if (rc) return rc;
    } else {
      if ((e = step_launch(top, src, dst, s))) return cuda_fail(e, "edge strip launch");
      if ((e = step_launch(bot, src + (n0 - B) * row, dst + (n0 - B) * row, s))) return cuda_fail(e, "edge strip launch");
      cudaEventRecord(c->ev_edge, s);
      cudaStreamWaitEvent(c->comm_stream, c->ev_edge, 0);
      rc = exchange(p, c, dst, c->comm_stream);
      if (rc) return rc;
      cudaEventRecord(c->ev_comm, c->comm_stream);
      if ((e = step_launch(mid, src + B * row, dst + B * row, s))) return cuda_fail(e, "interior strip launch");
      cudaStreamWaitEvent(s, c->ev_comm, 0);  // the next step reads dst's exchanged halo rows
    }
    src = dst;
  }
  if (sync_check()) {
    cudaError_t ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "LORA_SYNC_CHECK stream sync");
  }
  return LORA_OK;
}

void lora_stencil_comm_destroy(lora_comm* c) {
  if (!c) return;
  for (double* b : c->dbuf)
    if (b) cudaFree(b);
  if (c->comm && nccl().ok) nccl().CommDestroy(c->comm);
  if (c->ev_edge) cudaEventDestroy(c->ev_edge);
  if (c->ev_comm) cudaEventDestroy(c->ev_comm);
  if (c->comm_stream) cudaStreamDestroy(c->comm_stream);
  delete c;
}

}  // extern "C"
