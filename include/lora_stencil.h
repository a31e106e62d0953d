/*
 * lora_stencil.h — C-ABI of the B200-native LoRAStencil engine.
 *
 * What the library computes (PAPER.md = /root/reference/PAPER.md, "P:n" = its line n):
 *   A time-iterated d-dimensional FP64 stencil (d = 1, 2, 3): every interior point is replaced,
 *   T times, by the weighted sum of its (2r+1)^d neighbourhood (§I; eq. 2).
 *   The weights are factored on the host into rank-1 terms u_k v_k^T (eq. 8 P:149-153;
 *   Pyramidal Matrix Adaptation, eq. 15) and each term is evaluated as the banded
 *   Toeplitz chain U_k X V_k (eq. 5-7, eq. 9): Residual Dimension
 *   Gathering (§III-B), on FP64 tensor cores with Butterfly Vector Swapping (§III-D, eq. 17)
 *   or on the FP64 CUDA-core pipe, chosen per plan (see lora_engine).  3D stencils are
 *   evaluated plane by plane (Alg. 2).
 *
 * Conventions:
 *   * Arrays are PADDED: extent N_i + 2r along axis i, C order, slowest axis first.
 *     The r-wide halo holds fixed Dirichlet boundary values and is never updated.
 *   * weights[a0][a1]([a2]) multiplies in[x0+a0-r][x1+a1-r]([x2+a2-r])  (correlation).
 *   * Jacobi: each step reads only the previous step.
 *
 * Errors: functions return LORA_OK (0) or a negative lora_status; lora_stencil_plan returns
 * NULL on failure.  lora_stencil_last_error() returns a thread-local message for the last
 * failure on the calling thread.  Kernel launch errors are reported synchronously;
 * asynchronous device faults surface at the caller's next synchronisation (set the
 * environment variable LORA_SYNC_CHECK=1 to synchronise and check inside every run call).
 *
 * Threading: a plan is not re-entrant (its device scratch is shared); distinct plans may be
 * used concurrently from different threads.
 */
#ifndef LORA_STENCIL_H_
#define LORA_STENCIL_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct lora_plan lora_plan; /* opaque; owns host factors, device scratch/pinned buffers */
typedef struct lora_comm lora_comm; /* opaque; owns an ncclComm_t and two CUDA streams        */

typedef enum {
  LORA_OK = 0,
  LORA_ERR_INVALID_ARG = -1, /* bad pointer, size, radius, ndim, timesteps < 0           */
  LORA_ERR_UNSUPPORTED = -2, /* radius > 4, engine not available for this shape          */
  LORA_ERR_ALIAS = -3,       /* in and out overlap                                        */
  LORA_ERR_CUDA = -4,        /* a CUDA runtime call or kernel launch failed               */
  LORA_ERR_NCCL = -5,        /* NCCL missing or a NCCL call failed                        */
  LORA_ERR_OOM = -6,         /* device or pinned host allocation failed                   */
  LORA_ERR_FACTOR = -7       /* the factorisation does not reconstruct W to 1e-14          */
} lora_status;

/* Engine used for the rank-1 terms (the scalar C_{h+1} term and single-weight 3D planes are
 * always point-wise DFMA, P:275 and Alg. 2 lines 3-5). */
typedef enum {
  LORA_ENGINE_AUTO = 0,     /* planner picks the engine with the lowest issued FP64 work    */
  LORA_ENGINE_TC = 1,       /* RDG chains U X V on FP64 tensor cores (mma.m8n8k4.f64), BVS  */
  LORA_ENGINE_RDG_CUDA = 2, /* RDG chains as two banded passes on the FP64 CUDA-core pipe   */
  LORA_ENGINE_DIRECT = 3    /* no factorisation: the (2r+1)^d-point sum on CUDA cores (K11) */
} lora_engine;

typedef struct {
  int engine;  /* lora_engine; 0 = AUTO                                                     */
  int fuse_k;  /* time steps per HBM round trip; 0 = planner's choice, 1 = no fusion          */
  int reserved[6];
} lora_plan_opts;

typedef struct {               /* filled by lora_stencil_plan_query                          */
  int ndim, radius;
  int64_t grid[3];             /* interior extents (slowest first); grid[2] = 1 in 2D         */
  int engine;                  /* lora_engine actually used                                   */
  int n_terms;                 /* rank-1 terms over all planes, incl. scalar / point-wise     */
  int n_tc_chain;              /* terms evaluated as a two-stage chain U X V                  */
  int n_tc_single;             /* star arms: one banded stage (a unit-vector factor)          */
  int n_cuda;                  /* scalar / point-wise terms on the DFMA pipe                  */
  int n_planes_pointwise;      /* 3D planes with exactly one nonzero weight (Alg. 2 line 3)   */
  int z_symmetric;             /* 3D: W[r-k] == W[r+k] for all k (planes pre-added)          */
  int fuse_k;                  /* time steps per HBM round trip                               */
  int halo_depth;              /* fuse_k * radius                                             */
  int tile_m, tile_n;          /* CTA output tile (rows, columns of the fastest axis)         */
  int single_launch;           /* 1: small 2D grid, all T steps in ONE thread-block-cluster launch
                                  holding the grid in shared memory (DSMEM halo exchange)       */
  double recon_err;            /* max|sum u v^T - W| / max|W|                                 */
  double growth;               /* sum_k ||u_k||_1 ||v_k||_1 / ||W||_1                         */
  double fma_per_point_issued; /* FP64 work per point per step of the chosen engine's rank-1
                                  form: DFMA/DADD/DMUL lane-ops (CUDA-core engines) or DMMA FMA
                                  slots incl. band padding (tensor-core engine); halo recompute
                                  of fused launches not counted                                  */
  double fma_per_point_direct; /* (2r+1)^d, nonzero weights only                              */
  double fma_per_point_separable; /* sum over terms of (len u + len v) + point-wise terms      */
  /* The paper's analytic cost model for its A100 tiling at the plan's radius h (host arithmetic on
   * h only; reported so that the counts printed in the paper can be checked against the library):
   *   P:225  grid points updated at once            32 ceil(h/2) ceil(h/4)
   *   eq. 12 RDG fragment loads from shared memory  ab/8            -> per point 1/8
   *   eq. 13 ConvStencil fragment loads             2 ceil((2h+1)^2/4) per 8(2h+2) points
   *   eq. 14 ConvStencil / RDG                      ceil((2h+1)^2/4) / (h+1)   (3.25 at h=3, 4.2 at h=4)
   *   eq. 16 LoRAStencil MMAs                       2h ceil(h/2) (2 ceil(h/4)+1) per 32 ceil(h/2) ceil(h/4) points
   *                                                 (36 per 64 points at h=3; ConvStencil: eq. 13, 26)
   *   P:340  FP64 fragment elements wasted by one 8x8 update (eight 4x8 fragments = 256 loaded,
   *          (8+2h)^2 used): 256 - (8+2h)^2 (156 at h=1, 60 at h=3: fusing 3 Box-2D9P steps saves 96) */
  int    paper_points_per_update;
  double paper_rdg_frag_per_point;
  double paper_convstencil_frag_per_point;
  double paper_convstencil_over_rdg;
  double paper_mma_per_point;
  double paper_convstencil_mma_per_point;
  int    paper_fragment_waste;
} lora_plan_info;

/* Plans a stencil.  Host-only work (no CUDA call): validates, factors every 2D plane
 * (star arms / PMA / complete-pivot elimination, Q6), checks the reconstruction
 * (<= 1e-14 relative, else NULL with LORA_ERR_FACTOR), and picks engine, tile and fusion.
 *   weights    host, (2*radius+1)^ndim doubles, row-major, copied (caller keeps ownership)
 *   ndim       1, 2 or 3 (1D: a single banded gather; tensor-core engine 2D/3D only)
 *   radius     1..4
 *   grid_shape host, ndim interior extents (slowest first), each >= 1
 * The plan binds to the CUDA device that is current at its first run call. */
lora_plan* lora_stencil_plan(const double* weights, int ndim, int radius, const int64_t* grid_shape);
/* As lora_stencil_plan with options (opts may be NULL = defaults). */
lora_plan* lora_stencil_plan_ex(const double* weights, int ndim, int radius, const int64_t* grid_shape,
                                const lora_plan_opts* opts);

/* Runs `timesteps` Jacobi steps.  `in` and `out` are DEVICE pointers to padded arrays of
 * prod(N_i + 2r) doubles, 8-byte aligned (16-byte alignment and an even padded last extent
 * enable TMA staging).  `in` is never written; on return (stream-ordered) `out` holds step T
 * in its interior and a copy of `in`'s halo.  timesteps = 0 copies.  in/out must not overlap
 * (LORA_ERR_ALIAS).  `stream` is a cudaStream_t (NULL = legacy default stream).  The first
 * call allocates the plan's device scratch (one padded buffer) on the current device.
 * Launch-bound problems (<= 4 Mi padded points, >= 4 launches, a non-default stream): the second
 * identical call (same in, out, T, stream) captures the time loop as a CUDA graph and later identical
 * calls replay it; a stream the caller is already capturing gets the launches enqueued eagerly. */
int lora_stencil_run(lora_plan* p, const double* in, double* out, int64_t timesteps, void* stream);

/* The same computation from HOST buffers: copies `in_host` to plan-owned device memory,
 * runs, and copies the result to `out_host`, all ordered on `stream`, and synchronises the
 * stream before returning.  Pinned (cudaHostAlloc / cudaHostRegister) buffers give full
 * PCIe/C2C bandwidth; pageable buffers work but are staged by the driver. */
int lora_stencil_run_host(lora_plan* p, const double* in_host, double* out_host, int64_t timesteps, void* stream);

/* As lora_stencil_run_host but returns once the H2D copy, the run and the D2H copy are
 * ENQUEUED on `stream` (which must not be the legacy NULL stream: LORA_ERR_INVALID_ARG).
 * The caller synchronises `stream` before reading out_host or writing in_host, and must not
 * enqueue another call on the same plan from a different stream before then (the plan's
 * device buffers are reused).  Host buffers should be pinned, else the copies are
 * synchronous.  Independent problems on two plans and two streams overlap one problem's
 * copies with the other's stencil steps (bench.py e2e). */
int lora_stencil_run_host_async(lora_plan* p, const double* in_host, double* out_host, int64_t timesteps,
                                void* stream);

/* Fills *info from the plan (host-only). */
int lora_stencil_plan_query(const lora_plan* p, lora_plan_info* info);

/* Host-only access to the factorisation, for tests and tools.  For plane q (0 in 2D,
 * 0..2r in 3D) the plan holds terms k = 0..n-1, each a pair of vectors of length 2r+1
 * (centred, zero-padded) with  W_plane = sum_k u_k v_k^T.  Writes at most max_terms terms:
 * term_plane[k], term_kind[k] (0 chain, 1 single-stage arm, 2 scalar/point-wise),
 * term_radius[k] (support radius of the term), u[k*(2r+1) + i], v[k*(2r+1) + j].
 * *n_terms receives the total count.  Buffers may be NULL when max_terms = 0. */
int lora_stencil_plan_terms(const lora_plan* p, int max_terms, int* n_terms, int* term_plane, int* term_kind,
                            int* term_radius, double* u, double* v);

void lora_stencil_plan_destroy(lora_plan* p);

/* ---- multi-GPU: slab decomposition along the slowest axis, halo exchange over NCCL ---- */

/* Size of the opaque NCCL unique id (ncclUniqueId, 128 bytes). */
size_t lora_stencil_comm_id_size(void);
/* Rank 0 creates an id (host bytes, lora_stencil_comm_id_size() long) and broadcasts it,
 * e.g. with torch.distributed.broadcast_object_list.  NCCL is loaded at run time from the
 * libnccl.so.2 the process already has (torch's) or the system one. */
int lora_stencil_comm_get_id(void* id_out);
/* Collective over `nranks` processes, one GPU each (current device). */
int lora_stencil_comm_init(lora_comm** c, int nranks, int rank, const void* nccl_unique_id);
/* Collective: every rank calls with the same timesteps.  `p` is planned with this rank's
 * LOCAL interior shape (n0_local, N1[, N2]) — uneven splits are allowed.  CUDA-core plans with
 * fuse_k > 1 keep their fusion depth: the communicator then owns two deep-halo slab buffers
 * (fuse_k * radius rows/planes at internal edges; every slab needs at least that many) and the
 * exchange runs once per fused launch (after it, not overlapped); other plans step unfused with the
 * edge strips computed first and the exchange overlapped with the interior strip.  in_local/out_local
 * are device padded arrays of that local shape.  Rank 0's low halo and rank n-1's high halo
 * are the physical Dirichlet boundary; the other slab-edge halos are overwritten each step
 * by the neighbours' edge rows/planes.  Ordered on `stream`. */
int lora_stencil_run_dist(lora_plan* p, lora_comm* c, const double* in_local, double* out_local, int64_t timesteps,
                          void* stream);
void lora_stencil_comm_destroy(lora_comm* c);

/* Host-only: the halo exchange `rank` of `nranks` performs after every step of
 * lora_stencil_run_dist on a buffer of plan p's local padded shape (used by the run itself and by
 * the CPU tests).  Writes up to 4 entries, in issue order inside one NCCL group: kind[i]
 * (0 = send, 1 = recv), peer[i], offset[i] (elements from the buffer start) and count[i]
 * (elements, contiguous).  Returns the number of entries (0..4) or a negative lora_status. */
int lora_stencil_dist_exchange_plan(const lora_plan* p, int rank, int nranks, int64_t* kind, int64_t* peer,
                                    int64_t* offset, int64_t* count);
/* The same for a slab buffer whose internal edges carry halo_depth (>= radius) rows/planes: rows
 * [0, hl) low halo, [hl, hl + n0) own, then hh high-halo rows, with hl = halo_depth below a neighbour
 * and radius at the physical boundary (likewise hh).  lora_stencil_run_dist uses halo_depth =
 * fuse_k * radius for CUDA-core plans with fuse_k > 1 (comm-owned deep-halo buffers, one exchange
 * per fused launch); halo_depth = radius is lora_stencil_dist_exchange_plan. */
int lora_stencil_dist_exchange_plan_ex(const lora_plan* p, int rank, int nranks, int64_t halo_depth, int64_t* kind,
                                       int64_t* peer, int64_t* offset, int64_t* count);

/* ---- multi-GPU: the same slab decomposition with a DEVICE-INITIATED halo exchange ----
 * (north star (d) "halo exchange over NVLink ... overlapped with interior
 * compute").  Instead of host-issued ncclSend/ncclRecv after every step, the stencil kernel's
 * boundary work items store the slab's first/last r interior rows (2D) or planes (3D) straight
 * into the neighbour's halo through peer memory (NVLink P2P via CUDA IPC, or plain device
 * pointers within one process) and then publish a per-tile step counter in the neighbour's
 * memory; the neighbour's boundary items wait for that counter before staging their halo.
 * Interior tiles never wait, so the exchange overlaps the interior tile by tile and there is no
 * collective call per step at all.  Results are bitwise equal to lora_stencil_run_dist and to a
 * single-GPU run of the global grid (same kernels, same per-point arithmetic).
 *
 * Engines: the CUDA-core engine (2D, 3D radius <= 2) and the direct comparison kernel; other
 * plans return LORA_ERR_UNSUPPORTED.  CUDA-core plans keep their fusion depth k (plan fuse_k; 2D,
 * and 3D radius 1): each launch advances k steps and internal slab edges carry k*r-deep halos
 * (every slab needs >= k*r rows/planes, else LORA_ERR_INVALID_ARG); direct plans and 3D radius-2
 * plans step unfused.  Every rank's plan has the same trailing extents, radius and fuse_k (the
 * local n0 may differ).
 *
 * Exchange buffers: the communicator owns two padded slabs (the ping-pong pair the neighbours
 * write into; rows = lower halo depth + n0 + upper halo depth) plus the flag words, allocated with
 * cudaMalloc on the current device (IPC-exportable).  lora_stencil_p2p_buffer exposes them, and
 * lora_stencil_p2p_view the caller-layout array inside each (the padded local slab with R-deep halos,
 * same row pitch, starting at buffer row hl - R; the buffer itself for an unfused endpoint): a caller
 * that fills view 0 directly and passes it as `in_local` (and view L%2 as `out_local`, L = the
 * number of launches, ceil(T / k)) avoids the copy-in / copy-out, fused or not.
 *
 * A spin-wait that sees no progress for 20 s (a neighbour that never runs) gives up instead of
 * hanging the GPU and sets a device error word: lora_stencil_p2p_status reports it. */
typedef struct lora_p2p lora_p2p;

/* Creates this rank's endpoint for plan p (LOCAL shape) on the current device. */
int lora_stencil_p2p_create(lora_p2p** c, const lora_plan* p, int nranks, int rank);
/* Size of the opaque exchange handle (128 bytes: a cudaIpcMemHandle_t plus the slab layout). */
size_t lora_stencil_p2p_handle_size(void);
/* Writes this endpoint's handle (host bytes) for the neighbours, e.g. via
 * torch.distributed.all_gather_object. */
int lora_stencil_p2p_get_handle(const lora_p2p* c, void* handle_out);
/* Opens the neighbours' handles (rank-1's as lo_handle, rank+1's as hi_handle; NULL where there
 * is no neighbour) with cudaIpcOpenMemHandle.  Neighbours must live in OTHER processes. */
int lora_stencil_p2p_connect(lora_p2p* c, const void* lo_handle, const void* hi_handle);
/* Same-process wiring (one process driving several slabs, on one or several devices; peer
 * access is enabled where the devices differ).  lo / hi may be NULL. */
int lora_stencil_p2p_connect_local(lora_p2p* c, const lora_p2p* lo, const lora_p2p* hi);
/* Device pointer of exchange buffer i (0 or 1), or NULL. */
double* lora_stencil_p2p_buffer(const lora_p2p* c, int i);
/* Device pointer of the caller-layout view of exchange buffer i (0 or 1; see above), or NULL.
 * Owned by the endpoint; valid until lora_stencil_p2p_destroy. */
double* lora_stencil_p2p_view(const lora_p2p* c, int i);
/* Collective over the connected ranks (every rank calls with the same timesteps), ordered on
 * `stream`: copy-in (skipped if in_local is buffer 0), T steps with the in-kernel exchange, a
 * final wait for the neighbours' last rows, copy-out (skipped if out_local is buffer T%2). */
int lora_stencil_run_dist_p2p(lora_plan* p, lora_p2p* c, const double* in_local, double* out_local,
                              int64_t timesteps, void* stream);
/* Synchronises the device and reports a spin-wait timeout (LORA_ERR_CUDA) if one occurred.  A
 * timeout leaves the endpoint's monotonic step counters out of step with its neighbours for good:
 * once reported, the endpoint is POISONED and every later lora_stencil_run_dist_p2p on it returns
 * LORA_ERR_INVALID_ARG — destroy it and create (and connect) a new one. */
int lora_stencil_p2p_status(lora_p2p* c);
void lora_stencil_p2p_destroy(lora_p2p* c);

/* Thread-local message for the last failure on this thread ("" if none). */
const char* lora_stencil_last_error(void);
/* Thread-local lora_status of the last failure on this thread (LORA_OK after a successful
 * lora_stencil_plan / _plan_ex): the reason a plan call returned NULL. */
int lora_stencil_last_status(void);
/* Library version string. */
const char* lora_stencil_version(void);

#ifdef __cplusplus
}
#endif
#endif /* LORA_STENCIL_H_ */
