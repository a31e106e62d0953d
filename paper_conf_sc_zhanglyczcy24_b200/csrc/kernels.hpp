// Launchers for the device kernels (internal).  Every launcher enqueues on `s` and returns
// cudaGetLastError() of the launch.
#pragma once
#include <cuda_runtime.h>

#include <cstdlib>

#include "plan.hpp"

namespace lora {

// Radius-1 PMA plane factors (palindromic 3-tap u, v) rescaled so that the centre tap of v is
// exactly 1: v' = v / v[1], u' = u * v[1] (u' v'^T = u v^T up to one rounding per factor).  The 3D
// CUDA-core kernels then form the horizontal gather as T = x_0 + v'[0] (x_-1 + x_+1), one DADD and
// one DFMA instead of a DADD, a DMUL and a DFMA.  Both 3D kernels (unfused and fused) use the same
// rescaled factors, so their per-point arithmetic stays identical.  Returns false if v[1] == 0.
inline bool pma1_unit_centre(const double* u, const double* v, double* uo, double* vo) {
  if (v[1] == 0.0) return false;
  const double c = v[1];
  for (int i = 0; i < 3; ++i) { uo[i] = u[i] * c; vo[i] = v[i] / c; }
  vo[1] = 1.0;
  return true;
}

// Radius-1 3D planes with the full symmetry of a radially symmetric stencil:
// plane a0 of W is [a b a; b c b; a b a].  When planes 0 and 1 both have it and plane 2 mirrors
// plane 0 (Box-3D27P), the 3D CUDA-core kernels evaluate the two plane operators JOINTLY on the
// symmetric class sums they share (mode PM_SYM3, reading Q18): with px = x_l + x_r per
// row, s1 = x_u + x_d, pc = px_u + px_d (corners), e = px + s1 (edges),
//   d_0 = a_0 pc + (b_0 e + c_0 x); plane 1 straight into its accumulator: acc = a_1 pc + (b_1 e + (c_1 x + acc))
// 12 FP64 ops per point for both operators (incl. accumulation) instead of 16 for the two PMA chains.  Both kernels
// (unfused and fused) use the same formula in the same order, so they stay bitwise equal.
// LORA_NO_SYM3=1 keeps the PMA form (A/B).  Returns false unless the plane has the symmetry.
inline bool sym3_plane(const double* W, int a0, double& c, double& b, double& a) {
  const double* q = W + 9 * a0;
  a = q[0]; b = q[1]; c = q[4];
  return q[2] == a && q[6] == a && q[8] == a && q[3] == b && q[5] == b && q[7] == b;
}

inline bool sym3_enabled() {
  const char* e = std::getenv("LORA_NO_SYM3");
  return !(e && e[0] == '1');
}

// Device-initiated halo exchange (csrc/dist_p2p.cu): the slab's boundary work items
// store their edge rows/planes straight into the neighbour's halo over peer memory (NVLink P2P /
// CUDA IPC) and publish a per-unit step counter there; the neighbour's boundary items wait on it
// before staging their halo.  Interior items neither wait nor signal, so the exchange overlaps the
// interior tile by tile.  A "unit" is a 64-column band (2D) or a 64 x BY column (3D); a boundary
// item of unit b waits for the neighbour's units b-1..b+1 (2D) / the 3 x 3 around b (3D), whose
// staged tiles overlap the columns it reads and writes.
struct P2PArgs {
  int active = 0;                  // 0: ordinary single-GPU launch
  int nunits = 0;                  // flag units per side
  int nux = 0;                     // 3D: units per y row (unit = bx + nux * by)
  int pad_ = 0;
  const unsigned long long* wait_lo = nullptr;   // my flags written by the lower neighbour (null: none)
  const unsigned long long* wait_hi = nullptr;   // my flags written by the upper neighbour
  unsigned long long* sig_lo = nullptr;          // the lower neighbour's flags for me
  unsigned long long* sig_hi = nullptr;          // the upper neighbour's flags for me
  double* dst_lo = nullptr;        // the lower neighbour's destination buffer of this step
  double* dst_hi = nullptr;
  long long off_lo = 0;            // my padded element index + off_lo = its index (n0_lo * row)
  long long off_hi = 0;            // -(n0 * row)
  unsigned long long wait_val = 0; // boundary items wait until flags >= wait_val
  unsigned long long sig_val = 0;  // and publish sig_val when their stores are done
  int* err = nullptr;              // device error word (spin timeout => 1)
  // Row bookkeeping in the launch's padded rows (2D; 3D uses planes with H = R).  A fused launch of k
  // steps runs on a slab whose internal edges carry H = k_max R deep halos, presented to the kernel
  // as a taller "view" (the deep halo rows beyond R count as interior rows of the view): only the
  // rows [store_lo, store_hi) are this rank's and stored; the first H of them ([store_lo, lo_end))
  // go to the lower neighbour, the last H ([hi_begin, store_hi)) to the upper one.
  int H = 0, lo_end = 0, hi_begin = 0, store_lo = 0, store_hi = 0;
  int prepare_only = 0;            // 1: only load the kernel (lazy module loading must not happen
                                   // while a spin-waiting kernel of this process runs) and return
  int wait_units = 0;              // > 0: wait on units [0, wait_units) (the neighbour's previous
                                   // launch had another band geometry: a remainder launch)
};

// Copies the Dirichlet halo ring of `in` into `dst` (both padded arrays of the plan's shape).
cudaError_t launch_copy_halo(const Plan& p, const double* in, double* dst, cudaStream_t s);

// K11: CUDA-core direct (2R+1)^d-point stencil, one time step src -> dst (interior only).  2D runs on
// the RDG warp-streaming machinery (launch_direct2d_stream, kernels_rdg.cu) so that the comparison
// with the rank-1 engines is like for like.
cudaError_t launch_direct2d_stream(const Plan& p, const double* src, double* dst, cudaStream_t s);
cudaError_t launch_direct3d_stream(const Plan& p, const double* src, double* dst, cudaStream_t s);  // R <= 2
cudaError_t launch_direct(const Plan& p, const double* src, double* dst, cudaStream_t s);

// K1 (2D): RDG chains U_k X V_k on FP64 tensor cores (DMMA m8n8k4) with BVS, one step; k > 1: the
// composed k-step kernel (§IV-A) on the points farther than (k-1)R from the halo plus an
// exact stepwise recomputation of the band next to it.
cudaError_t launch_tc2d(const Plan& p, const double* src, double* dst, cudaStream_t s, int k = 1);

// K6 (2D): RDG chains as banded passes on the FP64 CUDA-core pipe, k fused steps (exact temporal
// blocking, halo re-imposed every sub-step); 3D dispatches to launch_rdg3d (k = 1).
cudaError_t launch_rdg2d(const Plan& p, const double* src, double* dst, cudaStream_t s, int k);
// One unfused step of the 2D CUDA-core engine (any signature incl. the direct comparison kernel) or
// of the 3D one, with the device-initiated halo exchange of `d` (d.active = 1).
cudaError_t launch_step_p2p(const Plan& p, const double* src, double* dst, cudaStream_t s, const P2PArgs& d, int k);
int p2p_units(const Plan& p, int* nux);   // flag units per side (unfused), 0 if the plan's engine has no P2P path
int p2p_units_k(const Plan& p, int k);     // 2D: band count of the k-fused stream kernel
int rdg2d_max_fuse(const Plan& p);

// K2 on CUDA cores (3D, Alg. 2 with RDG per plane), one step.
cudaError_t launch_rdg3d(const Plan& p, const double* src, double* dst, cudaStream_t s);

// K2 on tensor cores (3D, Alg. 2 with DMMA chains per plane, point-wise planes on DFMA), R = 1.
cudaError_t launch_tc3d(const Plan& p, const double* src, double* dst, cudaStream_t s);
bool tc3d_supported(const Plan& p);

// 1D stencils (kernels_1d.cu): one banded pass, k fused steps per launch.
cudaError_t launch_1d(const Plan& p, const double* src, double* dst, cudaStream_t s, int k);

bool tc2d_supported(const Plan& p);

// Small 2D grids (kernels_small.cu): all T steps in ONE launch of a thread-block cluster holding the
// whole padded grid in its shared memory (DSMEM halo exchange between the CTAs); two-arm star
// plans of the CUDA-core engine whose grid fits.  Bitwise equal to the streaming engine.
// launch_small2d returns cudaErrorNotSupported when the device cannot schedule the cluster.
bool small2d_eligible(const Plan& p);
cudaError_t launch_small2d(Plan& p, const double* in, double* out, int64_t T, cudaStream_t s);   // may allocate p.xbuf
bool rdg3d_supported(const Plan& p);
int rdg3d_p2p_units(const Plan& p, int* nux);
cudaError_t launch_rdg3d_p2p(const Plan& p, const double* src, double* dst, cudaStream_t s, const P2PArgs& d);
// k = 2, 3 fused 3D steps (radius 1), kernels_rdg3df.cu.
cudaError_t launch_rdg3d_fused(const Plan& p, const double* src, double* dst, cudaStream_t s, int k,
                               const P2PArgs* d = nullptr);
int rdg3d_fused_units(const Plan& p, int k, int* nux);   // flag units (columns) of the k-fused 3D kernel
bool rdg3d_fused_supported(const Plan& p);
bool rdg2d_supported(const Plan& p);

}  // namespace lora
