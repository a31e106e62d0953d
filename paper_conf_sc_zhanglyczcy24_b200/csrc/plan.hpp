// Internal plan representation shared by the planner, the C-ABI layer and the launchers.
// Not part of the public ABI (include/lora_stencil.h is).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "lora_stencil.h"

namespace lora {

constexpr int kMaxRadius = 4;
constexpr int kMaxN = 2 * kMaxRadius + 1;  // 9

enum TermKind { kChain = 0, kArm = 1, kPoint = 2 };

// One rank-1 term u v^T of a 2D plane (eq. 3), stored centred in length 2R+1
// (R = plan radius).  `r` is the term's own support radius (PMA pyramid level: eq. 15).
// kPoint terms carry the single weight in v[jc] with u = e_ic (offset (ic-R, jc-R)).
struct Term {
  int plane = 0;       // 3D: z-offset index a0 in 0..2R (2D: 0)
  int kind = kChain;
  int r = 0;
  double u[kMaxN] = {0};
  double v[kMaxN] = {0};
};

struct Plan {
  int ndim = 2, R = 1;
  int64_t N[3] = {1, 1, 1};
  std::vector<double> W;  // (2R+1)^ndim, row-major copy
  std::vector<Term> terms;
  // Composed-kernel fusion for the tensor-core engine (§IV-A): k steps of W are
  // the single (2kR+1)^2 stencil W * ... * W, factored like any other plane (radius cR = kR <= 4).
  int cR = 0;
  std::vector<double> cW;
  std::vector<Term> cterms;
  int engine = LORA_ENGINE_AUTO;
  int fuse_k = 1;
  int tile_m = 0, tile_n = 0;
  int z_symmetric = 0;
  int force_no_tma = 0;   // LORA_NO_TMA=1: use the LDGSTS staging path (tests both loaders)
  int tc_no_bvs = 0;
  int no_small = 0;       // LORA_NO_SMALL=1: no single-launch path for small 2D grids (tests)
  int small_mode = 0;     // LORA_SMALL_MODE: 0 2D tiles for short runs, else the grid variant; 1 ("cluster")
                          // the DSMEM cluster variant; 2 ("grid") the cooperative-grid variant (tests)
  int small_rp = 2;       // LORA_SMALL_RP: rows per CTA of its cooperative-grid variant (experiments)      // LORA_TC_NO_BVS=1: the Fig. 9 ablation (shuffle-based stage 2) in the TC engine
  int n_planes_point = 0;
  // CUDA-core engine, 2D, radius >= 3, W reflection-symmetric in both axes with a nonzero centre
  // column: evaluate W as the row-pair rank-1 split u_a = c_a (e_{R+a} + e_{R-a}), v_a = W[R+a,:] / c_a
  // (c_a = W[R+a,R], a = 0..R; exact up to the rounding of v_a, growth 1), which issues
  // R + R(R+1) + 2R + 1 FP64 ops per point against PMA's (22 vs 25 at R = 3).
  // LORA_RDG_PMA=1 keeps the PMA factors on that engine (ablation).
  int rdg_rows = 0;
  double recon_err = 0, growth = 0;
  double fma_issued = 0, fma_direct = 0, fma_separable = 0;
  // device state (lazily created at first run)
  int device = -1;
  double* scratch = nullptr;      // one padded buffer for the ping-pong
  double* dev_in = nullptr;       // run_host staging (device copies of host in/out)
  double* dev_out = nullptr;
  double* xbuf = nullptr;         // small-grid kernel: exchange buffer of the cooperative-grid variant
  size_t xbuf_elems = 0;
  unsigned long long xflag_base = 0;   // its per-CTA step counters are monotonic across launches
  size_t elems = 0;               // padded element count
  void* graph_exec = nullptr;     // cudaGraphExec_t of the cached time loop (small grids)
  const double* g_in = nullptr;   // its key
  double* g_out = nullptr;
  int64_t g_T = -1;
  void* g_stream = nullptr;
  int64_t P[3] = {1, 1, 1};       // padded extents
};

// planner.cpp
int plan_build(Plan& p, const double* weights, int ndim, int radius, const int64_t* grid, const lora_plan_opts* o,
               std::string& err);
double tc_fma_per_point(const Plan& p);
double cuda_fma_per_point(const Plan& p);

// api.cu
int fail(int code, const std::string& msg);
int cuda_fail(int /*cudaError_t*/ e, const char* what);
int ensure_device(Plan& p, bool want_scratch);
int step_launch(const Plan& p, const double* src, double* dst, void* stream);       // cudaError_t
int step_launch_k(const Plan& p, const double* src, double* dst, void* stream, int k);   // k fused steps
int copy_halo_launch(const Plan& p, const double* in, double* dst, void* stream);   // cudaError_t
bool sync_check();

}  // namespace lora

struct lora_plan : lora::Plan {};
