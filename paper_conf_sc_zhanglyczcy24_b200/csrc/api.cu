// C-ABI layer (include/lora_stencil.h): validation, device state, the time loop.
// The time loop (P:21 Jacobi iteration; eq. 18 counts T steps) ping-pongs between `out` and one
// plan-owned scratch buffer so that the last step lands in `out`; `in` is never written.
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <algorithm>
#include <string>
#include <vector>

#include "kernels.hpp"
#include "plan.hpp"

namespace lora {
thread_local std::string g_err;
thread_local int g_status = LORA_OK;   // status of the last failure on this thread (plan creation returns NULL)
int fail(int code, const std::string& msg) { g_err = msg; g_status = code; return code; }
int cuda_fail(int e, const char* what) {
  g_err = std::string(what) + ": " + cudaGetErrorString(static_cast<cudaError_t>(e));
  g_status = LORA_ERR_CUDA;
  return LORA_ERR_CUDA;
}
bool sync_check() {
  static int v = [] { const char* e = std::getenv("LORA_SYNC_CHECK"); return e && e[0] == '1' ? 1 : 0; }();
  return v != 0;
}

// Binds the plan to the current device at first use and allocates `want_scratch` buffers.
int ensure_device(Plan& p, bool want_scratch) {
  int dev = -1;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
  if (p.device < 0) p.device = dev;
  if (p.device != dev) return fail(LORA_ERR_INVALID_ARG, "plan is bound to another CUDA device");
  if (want_scratch && !p.scratch) {
    e = cudaMalloc(&p.scratch, p.elems * sizeof(double));
    if (e != cudaSuccess) { cudaGetLastError(); p.scratch = nullptr; return fail(LORA_ERR_OOM, "cudaMalloc(scratch) failed"); }
  }
  return LORA_OK;
}

// One launch advancing `k` time steps (k > 1 only for engines that fuse, see plan.fuse_k).
cudaError_t step(const Plan& p, const double* src, double* dst, cudaStream_t s, int k = 1) {
  if (p.ndim == 1) return launch_1d(p, src, dst, s, p.engine == LORA_ENGINE_DIRECT ? 1 : k);
  switch (p.engine) {
    case LORA_ENGINE_TC: return launch_tc2d(p, src, dst, s, k);
    case LORA_ENGINE_RDG_CUDA: return launch_rdg2d(p, src, dst, s, k);
    default: return launch_direct(p, src, dst, s);
  }
}
int step_launch(const Plan& p, const double* src, double* dst, void* stream) {
  return (int)step(p, src, dst, static_cast<cudaStream_t>(stream));
}
int step_launch_k(const Plan& p, const double* src, double* dst, void* stream, int k) {
  return (int)step(p, src, dst, static_cast<cudaStream_t>(stream), k);
}
int copy_halo_launch(const Plan& p, const double* in, double* dst, void* stream) {
  return (int)launch_copy_halo(p, in, dst, static_cast<cudaStream_t>(stream));
}

// Steps advanced by each launch of the time loop: ceil(T/k) launches of k fused steps, the last one
// taking the remainder — except that the tensor-core engine's composed kernel exists only for k
// itself, so a remainder other than 1 runs as single steps.
std::vector<int> launch_plan(const Plan& p, int64_t T) {
  const int64_t k = p.fuse_k < 1 ? 1 : p.fuse_k;
  std::vector<int> v;
  for (int64_t done = 0; done < T;) {
    int64_t st = std::min<int64_t>(k, T - done);
    if (p.engine == LORA_ENGINE_TC && st != k) st = 1;
    v.push_back((int)st);
    done += st;
  }
  return v;
}

// Enqueues the whole time loop on stream s (no synchronisation).
cudaError_t enqueue(Plan& p, const double* in, double* out, int64_t T, bool two, cudaStream_t s) {
  cudaError_t e = launch_copy_halo(p, in, out, s);
  if (e != cudaSuccess) return e;
  if (two) {
    e = launch_copy_halo(p, in, p.scratch, s);
    if (e != cudaSuccess) return e;
  }
  // launch i writes `out` when (L - 1 - i) is even, else the scratch buffer, so the last lands in `out`
  const std::vector<int> steps = launch_plan(p, T);
  const int64_t L = (int64_t)steps.size();
  const double* src = in;
  for (int64_t i = 0; i < L; ++i) {
    double* dst = ((L - 1 - i) % 2 == 0) ? out : p.scratch;
    e = step(p, src, dst, s, steps[i]);
    if (e != cudaSuccess) return e;
    src = dst;
  }
  return cudaSuccess;
}

// Launch-bound problems (small grids, many launches) replay the time loop as a CUDA graph: the
// second identical call (same in, out, T, stream) captures it, later identical calls replay it.
bool use_graph(const Plan& p, int64_t launches, cudaStream_t s) {
  static int off = [] { const char* e = std::getenv("LORA_NO_GRAPH"); return e && e[0] == '1' ? 1 : 0; }();
  // the legacy / per-thread default streams cannot be captured
  if (s == nullptr || s == cudaStreamLegacy || s == cudaStreamPerThread) return false;
  // a stream the caller is already capturing (e.g. torch.cuda.graph around run): enqueue eagerly into
  // the caller's capture instead of starting a nested one, which would fail and invalidate it
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(s, &cs) != cudaSuccess) { cudaGetLastError(); return false; }
  if (cs != cudaStreamCaptureStatusNone) return false;
  return !off && launches >= 4 && p.elems <= (size_t(1) << 22);
}

int run_device(Plan& p, const double* in, double* out, int64_t T, cudaStream_t s) {
  const size_t bytes = p.elems * sizeof(double);
  if (T == 0) {
    cudaError_t e = cudaMemcpyAsync(out, in, bytes, cudaMemcpyDeviceToDevice, s);
    return e == cudaSuccess ? LORA_OK : cuda_fail(e, "cudaMemcpyAsync");
  }
  cudaError_t e;
  if (small2d_eligible(p)) {   // small 2D grid: every step in one cluster launch (kernels_small.cu)
    int rc = ensure_device(p, false);
    if (rc) return rc;
    e = launch_small2d(p, in, out, T, s);
    if (e == cudaSuccess) {
      if (sync_check() && (e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_fail(e, "LORA_SYNC_CHECK stream sync");
      return LORA_OK;
    }
    if (e != cudaErrorNotSupported) return cuda_fail(e, "small-grid cluster launch");
    cudaGetLastError();   // the device cannot schedule the cluster: the streaming path below
  }
  const int64_t L = (int64_t)launch_plan(p, T).size();
  const bool two = L >= 2;
  int rc = ensure_device(p, two);
  if (rc) return rc;
  if (use_graph(p, L, s)) {
    const bool same = p.g_in == in && p.g_out == out && p.g_T == T && p.g_stream == (void*)s;
    if (same && p.graph_exec) {
      e = cudaGraphLaunch(static_cast<cudaGraphExec_t>(p.graph_exec), s);
      if (e != cudaSuccess) return cuda_fail(e, "cudaGraphLaunch");
    } else if (same) {  // second identical call: capture, instantiate, launch
      cudaGraph_t g = nullptr;
      e = cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
      if (e != cudaSuccess) return cuda_fail(e, "cudaStreamBeginCapture");
      cudaError_t le = enqueue(p, in, out, T, two, s);
      e = cudaStreamEndCapture(s, &g);
      if (le != cudaSuccess) { if (g) cudaGraphDestroy(g); return cuda_fail(le, "stencil kernel launch (capture)"); }
      if (e != cudaSuccess) return cuda_fail(e, "cudaStreamEndCapture");
      cudaGraphExec_t ex = nullptr;
      e = cudaGraphInstantiate(&ex, g, 0);
      cudaGraphDestroy(g);
      if (e != cudaSuccess) return cuda_fail(e, "cudaGraphInstantiate");
      p.graph_exec = ex;
      e = cudaGraphLaunch(ex, s);
      if (e != cudaSuccess) return cuda_fail(e, "cudaGraphLaunch");
    } else {  // new key: run eagerly and remember it
      if (p.graph_exec) { cudaGraphExecDestroy(static_cast<cudaGraphExec_t>(p.graph_exec)); p.graph_exec = nullptr; }
      p.g_in = in; p.g_out = out; p.g_T = T; p.g_stream = (void*)s;
      e = enqueue(p, in, out, T, two, s);
      if (e != cudaSuccess) return cuda_fail(e, "stencil kernel launch");
    }
  } else {
    e = enqueue(p, in, out, T, two, s);
    if (e != cudaSuccess) return cuda_fail(e, "stencil kernel launch");
  }
  if (sync_check()) {
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "LORA_SYNC_CHECK stream sync");
  }
  return LORA_OK;
}
}  // namespace lora

using namespace lora;

extern "C" {

const char* lora_stencil_last_error(void) { return g_err.c_str(); }
int lora_stencil_last_status(void) { return g_status; }
const char* lora_stencil_version(void) { return "lora_stencil_b200 0.1 (sm_100a)"; }

lora_plan* lora_stencil_plan_ex(const double* weights, int ndim, int radius, const int64_t* grid_shape,
                                const lora_plan_opts* opts) {
  lora_plan* p = new (std::nothrow) lora_plan();
  if (!p) { g_err = "out of host memory"; g_status = LORA_ERR_OOM; return nullptr; }
  std::string err;
  int rc = plan_build(*p, weights, ndim, radius, grid_shape, opts, err);
  if (rc != LORA_OK) { g_err = err; g_status = rc; delete p; return nullptr; }
  g_err.clear();
  g_status = LORA_OK;
  return p;
}

lora_plan* lora_stencil_plan(const double* weights, int ndim, int radius, const int64_t* grid_shape) {
  return lora_stencil_plan_ex(weights, ndim, radius, grid_shape, nullptr);
}

void lora_stencil_plan_destroy(lora_plan* p) {
  if (!p) return;
  if (p->device >= 0) {
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != p->device) cudaSetDevice(p->device);
    if (p->graph_exec) cudaGraphExecDestroy(static_cast<cudaGraphExec_t>(p->graph_exec));
    if (p->scratch) cudaFree(p->scratch);
    if (p->dev_in) cudaFree(p->dev_in);
    if (p->dev_out) cudaFree(p->dev_out);
    if (p->xbuf) cudaFree(p->xbuf);
    if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
  }
  delete p;
}

int lora_stencil_plan_query(const lora_plan* p, lora_plan_info* info) {
  if (!p || !info) return fail(LORA_ERR_INVALID_ARG, "NULL plan or info");
  std::memset(info, 0, sizeof(*info));
  info->ndim = p->ndim; info->radius = p->R;
  for (int i = 0; i < 3; ++i) info->grid[i] = i < p->ndim ? p->N[i] : 1;
  info->engine = p->engine;
  info->n_terms = (int)p->terms.size();
  for (const Term& t : p->terms) {
    if (t.kind == kChain) info->n_tc_chain++;
    else if (t.kind == kArm) info->n_tc_single++;
    else info->n_cuda++;
  }
  info->n_planes_pointwise = p->n_planes_point;
  info->z_symmetric = p->z_symmetric;
  info->fuse_k = p->fuse_k;
  info->halo_depth = p->fuse_k * p->R;
  info->tile_m = p->tile_m; info->tile_n = p->tile_n;
  info->single_launch = small2d_eligible(*p) ? 1 : 0;
  info->recon_err = p->recon_err;
  info->growth = p->growth;
  info->fma_per_point_issued = p->fma_issued;
  info->fma_per_point_direct = p->fma_direct;
  info->fma_per_point_separable = p->fma_separable;
  {  // the paper's cost model at h = R (include/lora_stencil.h; eq. 12-14, eq. 16)
    const int h = p->R;
    auto cdiv = [](int a, int b) { return (a + b - 1) / b; };
    const int pts = 32 * cdiv(h, 2) * cdiv(h, 4);
    const int box = cdiv((2 * h + 1) * (2 * h + 1), 4);
    info->paper_points_per_update = pts;
    info->paper_rdg_frag_per_point = 1.0 / 8.0;
    info->paper_convstencil_frag_per_point = 2.0 * box / (8.0 * (2 * h + 2));
    info->paper_convstencil_over_rdg = double(box) / (h + 1);
    info->paper_mma_per_point = double(2 * h * cdiv(h, 2) * (2 * cdiv(h, 4) + 1)) / pts;
    info->paper_convstencil_mma_per_point = info->paper_convstencil_frag_per_point;   // no fragment reuse
    info->paper_fragment_waste = 256 - (8 + 2 * h) * (8 + 2 * h);
  }
  return LORA_OK;
}

int lora_stencil_plan_terms(const lora_plan* p, int max_terms, int* n_terms, int* term_plane, int* term_kind,
                            int* term_radius, double* u, double* v) {
  if (!p || !n_terms) return fail(LORA_ERR_INVALID_ARG, "NULL plan or n_terms");
  if (max_terms > 0 && (!term_plane || !term_kind || !term_radius || !u || !v))
    return fail(LORA_ERR_INVALID_ARG, "NULL output buffer");
  const int n = 2 * p->R + 1;
  *n_terms = (int)p->terms.size();
  for (int k = 0; k < max_terms && k < (int)p->terms.size(); ++k) {
    const Term& t = p->terms[k];
    term_plane[k] = t.plane; term_kind[k] = t.kind; term_radius[k] = t.r;
    for (int i = 0; i < n; ++i) { u[k * n + i] = t.u[i]; v[k * n + i] = t.v[i]; }
  }
  return LORA_OK;
}

int lora_stencil_run(lora_plan* p, const double* in, double* out, int64_t timesteps, void* stream) {
  if (!p || !in || !out) return fail(LORA_ERR_INVALID_ARG, "NULL plan, in or out");
  if (timesteps < 0) return fail(LORA_ERR_INVALID_ARG, "timesteps must be >= 0");
  if ((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(out)) & 7)
    return fail(LORA_ERR_INVALID_ARG, "in/out must be 8-byte aligned");
  const size_t bytes = p->elems * sizeof(double);
  const char* a = reinterpret_cast<const char*>(in);
  const char* b = reinterpret_cast<const char*>(out);
  if (a < b + bytes && b < a + bytes) return fail(LORA_ERR_ALIAS, "in and out overlap");
  int rc = run_device(*p, in, out, timesteps, static_cast<cudaStream_t>(stream));
  if (rc == LORA_OK) g_err.clear();
  return rc;
}

static int run_host_enqueue(lora_plan* p, const double* in_host, double* out_host, int64_t timesteps,
                            cudaStream_t s) {
  int rc = ensure_device(*p, false);
  if (rc) return rc;
  const size_t bytes = p->elems * sizeof(double);
  if (!p->dev_in) {
    if (cudaMalloc(&p->dev_in, bytes) != cudaSuccess) { cudaGetLastError(); p->dev_in = nullptr; return fail(LORA_ERR_OOM, "cudaMalloc(dev_in)"); }
  }
  if (!p->dev_out) {
    if (cudaMalloc(&p->dev_out, bytes) != cudaSuccess) { cudaGetLastError(); p->dev_out = nullptr; return fail(LORA_ERR_OOM, "cudaMalloc(dev_out)"); }
  }
  cudaError_t e = cudaMemcpyAsync(p->dev_in, in_host, bytes, cudaMemcpyHostToDevice, s);
  if (e != cudaSuccess) return cuda_fail(e, "H2D copy");
  rc = run_device(*p, p->dev_in, p->dev_out, timesteps, s);
  if (rc) return rc;
  e = cudaMemcpyAsync(out_host, p->dev_out, bytes, cudaMemcpyDeviceToHost, s);
  if (e != cudaSuccess) return cuda_fail(e, "D2H copy");
  return LORA_OK;
}

int lora_stencil_run_host_async(lora_plan* p, const double* in_host, double* out_host, int64_t timesteps,
                                void* stream) {
  if (!p || !in_host || !out_host) return fail(LORA_ERR_INVALID_ARG, "NULL plan, in or out");
  if (timesteps < 0) return fail(LORA_ERR_INVALID_ARG, "timesteps must be >= 0");
  if (stream == nullptr) return fail(LORA_ERR_INVALID_ARG, "run_host_async needs an explicit stream");
  int rc = run_host_enqueue(p, in_host, out_host, timesteps, static_cast<cudaStream_t>(stream));
  if (rc) return rc;
  g_err.clear();
  return LORA_OK;
}

int lora_stencil_run_host(lora_plan* p, const double* in_host, double* out_host, int64_t timesteps, void* stream) {
  if (!p || !in_host || !out_host) return fail(LORA_ERR_INVALID_ARG, "NULL plan, in or out");
  if (timesteps < 0) return fail(LORA_ERR_INVALID_ARG, "timesteps must be >= 0");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  int rc = run_host_enqueue(p, in_host, out_host, timesteps, s);
  if (rc) return rc;
  cudaError_t e;
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(e, "stream sync");
  g_err.clear();
  return LORA_OK;
}

}  // extern "C"
