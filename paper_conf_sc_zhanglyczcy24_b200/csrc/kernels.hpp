// Launchers for the device kernels (internal).  Every launcher enqueues on `s` and returns
// cudaGetLastError() of the launch.
#pragma once
#include <cuda_runtime.h>

#include "plan.hpp"

namespace lora {

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
int rdg2d_max_fuse(const Plan& p);

// K2 on CUDA cores (3D, Alg. 2 with RDG per plane), one step.
cudaError_t launch_rdg3d(const Plan& p, const double* src, double* dst, cudaStream_t s);

// K2 on tensor cores (3D, Alg. 2 with DMMA chains per plane, point-wise planes on DFMA), R = 1.
cudaError_t launch_tc3d(const Plan& p, const double* src, double* dst, cudaStream_t s);
bool tc3d_supported(const Plan& p);

// 1D stencils (kernels_1d.cu): one banded pass, k fused steps per launch.
cudaError_t launch_1d(const Plan& p, const double* src, double* dst, cudaStream_t s, int k);

bool tc2d_supported(const Plan& p);
bool rdg3d_supported(const Plan& p);
// k = 2, 3 fused 3D steps (radius 1), kernels_rdg3df.cu.
cudaError_t launch_rdg3d_fused(const Plan& p, const double* src, double* dst, cudaStream_t s, int k);
bool rdg3d_fused_supported(const Plan& p);
bool rdg2d_supported(const Plan& p);

}  // namespace lora
