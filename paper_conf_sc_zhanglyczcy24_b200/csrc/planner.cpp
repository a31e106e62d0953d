// Host planner: factor the stencil weights into rank-1 terms and choose the engine.
//
// Paper: eq. 8 "W can be decomposed into r matrices each with rank = 1";
// PMA (§III-C, eq. 15): peel the radially symmetric W ring by ring with the
// corner pivot, C_i = (R[:,0]/R[0,0]) (x) R[0,:], leaving a (2h-1)^2 radially symmetric
// remainder, down to the 1x1 scalar C_{h+1} ("no additional MM is required").
// Where the paper is silent (zero/tiny pivots, star stencils, non-symmetric W) this follows
// DESIGN.md reading Q6: star arms, rank-revealing stop, complete-pivot elimination.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "kernels.hpp"
#include "plan.hpp"

namespace lora {
namespace {

struct Mat {  // n x n, row-major
  int n;
  std::vector<double> a;
  explicit Mat(int n_) : n(n_), a(size_t(n_) * n_, 0.0) {}
  double& operator()(int i, int j) { return a[size_t(i) * n + j]; }
  double operator()(int i, int j) const { return a[size_t(i) * n + j]; }
};

double maxabs(const Mat& m) {
  double s = 0;
  for (double x : m.a) s = std::max(s, std::fabs(x));
  return s;
}

int support_radius(const double* x, int n) {  // max |i - c| over nonzeros, c = (n-1)/2
  int c = (n - 1) / 2, r = 0;
  for (int i = 0; i < n; ++i)
    if (x[i] != 0.0) r = std::max(r, std::abs(i - c));
  return r;
}

// Factor one (2R+1)^2 plane into terms appended to `out`.
void factor_plane(const Mat& P, int R, int plane, double tol, std::vector<Term>& out) {
  const int n = 2 * R + 1;
  int nnz = 0, zi = 0, zj = 0;
  bool star = true;
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < n; ++j)
      if (P(i, j) != 0.0) {
        ++nnz; zi = i; zj = j;
        if (i != R && j != R) star = false;
      }
  if (nnz == 0) return;                       // (0) W == 0: no terms
  if (nnz == 1) {                             // single weight: point-wise (Alg. 2 lines 3-5)
    Term t; t.plane = plane; t.kind = kPoint;
    t.u[zi] = 1.0; t.v[zj] = P(zi, zj);
    t.r = std::max(std::abs(zi - R), std::abs(zj - R));
    out.push_back(t);
    return;
  }
  if (star) {                                 // (i) arms: one unit-vector factor each
    bool has_h = false, has_v = false;
    for (int j = 0; j < n; ++j) if (j != R && P(R, j) != 0.0) has_h = true;
    for (int i = 0; i < n; ++i) if (i != R && P(i, R) != 0.0) has_v = true;
    if (has_h) {  // horizontal arm incl. the centre: u = e_R, v = P[R,:]
      Term t; t.plane = plane; t.kind = kArm; t.u[R] = 1.0;
      for (int j = 0; j < n; ++j) t.v[j] = P(R, j);
      t.r = support_radius(t.v, n);
      out.push_back(t);
    }
    if (has_v) {  // vertical arm: u = P[:,R] (centre only if no horizontal arm), v = e_R
      Term t; t.plane = plane; t.kind = kArm; t.v[R] = 1.0;
      for (int i = 0; i < n; ++i) t.u[i] = (i == R && has_h) ? 0.0 : P(i, R);
      t.r = support_radius(t.u, n);
      out.push_back(t);
    }
    return;
  }
  // (ii) PMA ring by ring while the remainder is radially (reflection) symmetric.
  Mat Rm = P;
  const double normW1 = [&] { double s = 0; for (double x : P.a) s += std::fabs(x); return s; }();
  double growth = 0;
  int k = 0;
  for (; k <= R; ++k) {
    if (maxabs(Rm) <= tol) break;             // rank revealed: stop (no 0/0 on separable W)
    const int m = n - 2 * k;                  // current ring size 2(R-k)+1
    if (m == 1) {                             // the scalar C_{h+1}
      Term t; t.plane = plane; t.kind = kPoint; t.r = 0;
      t.u[R] = 1.0; t.v[R] = Rm(R, R);
      out.push_back(t);
      Rm(R, R) = 0.0;
      break;
    }
    bool border_zero = true, sym = true;
    for (int i = k; i < n - k; ++i)
      for (int j = k; j < n - k; ++j) {
        bool on_border = (i == k || i == n - 1 - k || j == k || j == n - 1 - k);
        if (on_border && std::fabs(Rm(i, j)) > tol) border_zero = false;
        if (Rm(i, j) != Rm(n - 1 - i, j) || Rm(i, j) != Rm(i, n - 1 - j)) sym = false;  // exact: PMA factors stay exactly palindromic
      }
    if (border_zero) continue;               // ring already empty: skip it
    const double piv = Rm(k, k);
    if (!sym || std::fabs(piv) <= tol) break; // hand the remainder to elimination
    Term t; t.plane = plane; t.kind = kChain; t.r = R - k;
    for (int i = k; i < n - k; ++i) t.u[i] = Rm(i, k) / piv;   // u = R[:,0] / R[0,0]
    for (int j = k; j < n - k; ++j) t.v[j] = Rm(k, j);         // v = R[0,:]
    double g = 0, nu = 0, nv = 0;
    for (int i = 0; i < n; ++i) { nu += std::fabs(t.u[i]); nv += std::fabs(t.v[i]); }
    g = nu * nv / normW1;
    if (growth + g > 1e3) break;               // unbounded growth: use elimination instead
    growth += g;
    for (int i = k; i < n - k; ++i)
      for (int j = k; j < n - k; ++j) Rm(i, j) -= t.u[i] * t.v[j];
    for (int i = k; i < n - k; ++i) { Rm(i, k) = 0.0; Rm(i, n - 1 - k) = 0.0; Rm(k, i) = 0.0; Rm(n - 1 - k, i) = 0.0; }
    out.push_back(t);
  }
  // (iii) complete-pivot elimination on whatever remains (PMA is its corner-pivot case).
  for (int it = 0; it < n && maxabs(Rm) > tol; ++it) {
    int pi = 0, pj = 0;
    double best = -1;
    for (int i = 0; i < n; ++i)
      for (int j = 0; j < n; ++j)
        if (std::fabs(Rm(i, j)) > best) { best = std::fabs(Rm(i, j)); pi = i; pj = j; }
    const double piv = Rm(pi, pj);
    Term t; t.plane = plane;
    for (int i = 0; i < n; ++i) t.u[i] = Rm(i, pj) / piv;
    for (int j = 0; j < n; ++j) t.v[j] = Rm(pi, j);
    t.u[pi] = 1.0;
    int nzu = 0, nzv = 0;
    for (int i = 0; i < n; ++i) { nzu += t.u[i] != 0.0; nzv += t.v[i] != 0.0; }
    for (int i = 0; i < n; ++i)
      for (int j = 0; j < n; ++j) Rm(i, j) -= t.u[i] * t.v[j];
    for (int i = 0; i < n; ++i) { Rm(i, pj) = 0.0; Rm(pi, i) = 0.0; }
    if (nzu == 1 && nzv == 1) { t.kind = kPoint; t.r = std::max(std::abs(pi - R), std::abs(pj - R)); }
    else if (nzu == 1 && pi == R) { t.kind = kArm; t.r = support_radius(t.v, n); }
    else if (nzv == 1 && pj == R) { t.kind = kArm; t.r = support_radius(t.u, n); }
    else { t.kind = kChain; t.r = std::max(support_radius(t.u, n), support_radius(t.v, n)); }
    out.push_back(t);
  }
}

}  // namespace

// Issued FP64 FMAs per output point per step for the tensor-core engine:
// stage 1 computes 8 x ceil8(BN + 2r) T values with K1 = ceil4(8 + 2r) per element, stage 2
// 8 x BN outputs with K2 = 16 (BVS fragments of two T blocks); arms are one stage with
// K = ceil4(8 + 2r) (horizontal arms: per output; vertical arms: per output too);
// point-wise terms are 1 DFMA.
double tc_fma_per_point(const Plan& p) {
  const double BN = 64.0;
  const int n = 2 * p.R + 1;
  auto term_cost = [&](const Term& t) {
    const int r = t.r;
    const double K = 4.0 * std::ceil((8.0 + 2 * r) / 4.0);
    if (t.kind == kPoint) return 1.0;
    if (t.kind == kArm) return K;
    return K * (8.0 * std::ceil((BN + 2 * r) / 8.0)) / BN + (r <= 2 ? 12.0 : 16.0);  // grouped BVS for r <= 2
  };
  double f = 0;
  const int nplanes = p.ndim == 2 ? 1 : n;
  for (int q = 0; q < nplanes; ++q) {
    bool mirrored = false;
    if (p.ndim == 3 && q > p.R) {  // kernels_tc3d.cu computes a z-symmetric plane pair once
      mirrored = true;
      for (int e = 0; e < n * n; ++e)
        if (p.W[size_t(q) * n * n + e] != p.W[size_t(2 * p.R - q) * n * n + e]) { mirrored = false; break; }
    }
    if (mirrored) { f += 1; continue; }
    double fp = 0;
    for (const Term& t : p.terms)
      if (t.plane == q) fp += term_cost(t);
    f += fp + (p.ndim == 3 && fp > 0 ? 1 : 0);  // + the add of the plane result into its output plane
  }
  return f;
}

// Issued FMAs per point for the CUDA-core RDG engine (kernels_rdg.cu / kernels_rdg3d.cu): the
// PMA and star signatures issue each term at its own radius; the general signature issues every
// term at the full radius R.  3D: per plane (Alg. 2), a mirrored plane pair (W_a == W_{2R-a})
// is computed once and added twice.
double cuda_fma_per_point(const Plan& p) {
  const int n = 2 * p.R + 1;
  auto plane_cost = [&](int q) {
    double f = 0;
    int cnt = 0;
    bool all_arms = true, pma_like = true;
    for (const Term& t : p.terms) {
      if (t.plane != q) continue;
      ++cnt;
      if (t.kind != kArm) all_arms = false;
      if (t.kind == kPoint) f += 1;
      else if (t.kind == kArm) f += 2 * t.r + 1;
      else f += 2.0 * (2 * t.r + 1);
    }
    (void)pma_like;
    if (p.ndim == 3 && cnt > 0 && !(cnt == 1) && !(cnt == 2 && all_arms)) {
      bool pma1 = p.R == 1 && cnt == 2;
      f = pma1 ? 2.0 * 1.5 + 3.0 + 1.0 : cnt * 2.0 * n;  // PM_PMA1 (unit centre tap: T = 1 DADD + 1 DFMA; BY = 4: 6 T rows per 4 outputs) / general
    }
    return f;
  };
  if (p.ndim == 2) {
    const int R = p.R;
    // SIG_ROWS (kernels_rdg.cu): R shared pair sums, R DFMA per row term (unit centre tap), 2R DFMA
    // for the vertical gather and one DMUL for the fresh ring slot
    if (p.rdg_rows) return R + (R + 1) * R + 2 * R + 1;
    // PMA pyramid (SIG_PMA): R shared tap-pair sums, then per chain of radius H a palindromic
    // horizontal gather (H: the chain is rescaled to a unit centre tap of v, kernels_rdg.cu
    // signature()) and a vertical scatter (2H+1), plus the scalar C_{h+1}
    bool pma = (int)p.terms.size() == R + 1;
    for (int k = 0; pma && k < R; ++k) pma = p.terms[k].kind == kChain && p.terms[k].r == R - k;
    if (pma) pma = p.terms[R].kind == kPoint && p.terms[R].r == 0;
    if (pma) {
      double f = R + 1;
      for (int k = 0; k < R; ++k) f += (R - k) + (2 * (R - k) + 1);
      return f;
    }
    return plane_cost(0);
  }
  if (p.ndim == 3 && p.R == 1 && sym3_enabled()) {
    // PM_SYM3 (kernels.hpp sym3_plane; chosen by the 3D kernels when planes 0 and 1 are PMA planes
    // with the full [a b a; b c b; a b a] symmetry and plane 2 mirrors plane 0): px 1.5 (6 rows per 4
    // outputs), 3 shared class sums, 3 per plane operator, 2 accumulating adds (plane 1's operator
    // accumulates through its FMAs)
    auto pma1 = [&](int q) {
      int cnt = 0, chain = 0, point = 0;
      for (const Term& t : p.terms)
        if (t.plane == q) { ++cnt; chain += t.kind == kChain && t.r == 1; point += t.kind == kPoint; }
      return cnt == 2 && chain == 1 && point == 1;
    };
    bool mir = true;
    for (int e = 0; e < 9; ++e) mir = mir && p.W[size_t(18) + e] == p.W[size_t(e)];
    double c, b, a;
    if (mir && pma1(0) && pma1(1) && sym3_plane(p.W.data(), 0, c, b, a) && sym3_plane(p.W.data(), 1, c, b, a))
      return 1.5 + 3.0 + 2 * 3.0 + 2.0;
  }
  double f = 0;
  for (int q = 0; q < n; ++q) {
    bool mirrored = false;
    if (q > p.R) {
      const int m = 2 * p.R - q;
      mirrored = true;
      for (int e = 0; e < n * n; ++e)
        if (p.W[size_t(q) * n * n + e] != p.W[size_t(m) * n * n + e]) { mirrored = false; break; }
    }
    if (!mirrored) f += plane_cost(q);
    else f += 1;  // the extra add into the mirrored output plane
  }
  return f;
}

int plan_build(Plan& p, const double* weights, int ndim, int radius, const int64_t* grid, const lora_plan_opts* o,
               std::string& err) {
  if (!weights || !grid) { err = "weights and grid_shape must be non-NULL"; return LORA_ERR_INVALID_ARG; }
  if (ndim < 1 || ndim > 3) { err = "ndim must be 1, 2 or 3"; return LORA_ERR_INVALID_ARG; }
  if (radius < 1) { err = "radius must be >= 1"; return LORA_ERR_INVALID_ARG; }
  if (radius > kMaxRadius) { err = "radius > 4 is not supported (DESIGN.md Q14)"; return LORA_ERR_UNSUPPORTED; }
  for (int i = 0; i < ndim; ++i)
    if (grid[i] < 1) { err = "grid extents must be >= 1"; return LORA_ERR_INVALID_ARG; }
  const int n = 2 * radius + 1;
  const size_t nw = ndim == 1 ? size_t(n) : (ndim == 2 ? size_t(n) * n : size_t(n) * n * n);
  for (size_t i = 0; i < nw; ++i)
    if (!std::isfinite(weights[i])) { err = "weights must be finite"; return LORA_ERR_INVALID_ARG; }
  p.ndim = ndim; p.R = radius;
  p.N[0] = p.N[1] = p.N[2] = 1;
  for (int i = 0; i < ndim; ++i) p.N[i] = grid[i];
  p.W.assign(weights, weights + nw);
  p.elems = 1;
  for (int i = 0; i < 3; ++i) p.P[i] = 1;
  for (int i = 0; i < ndim; ++i) { p.P[i] = p.N[i] + 2 * radius; p.elems *= size_t(p.P[i]); }

  double wmax = 0, w1 = 0;
  int nnz = 0;
  for (size_t i = 0; i < nw; ++i) { wmax = std::max(wmax, std::fabs(weights[i])); w1 += std::fabs(weights[i]); nnz += weights[i] != 0.0; }
  const double tol = 1e-15 * wmax;
  p.terms.clear();
  const int nplanes = ndim == 3 ? n : 1;
  p.z_symmetric = 0; p.n_planes_point = 0;
  for (int q = 0; q < nplanes; ++q) {
    if (ndim == 1) {  // one banded gather: a horizontal arm u = e_R, v = w; or a point
      int nz = 0, zj = 0;
      for (int j = 0; j < n; ++j) if (weights[j] != 0.0) { ++nz; zj = j; }
      if (nz == 0) break;
      Term t; t.plane = 0; t.u[radius] = 1.0;
      for (int j = 0; j < n; ++j) t.v[j] = weights[j];
      t.kind = nz == 1 ? kPoint : kArm;
      t.r = nz == 1 ? std::abs(zj - radius) : support_radius(t.v, n);
      p.terms.push_back(t);
      break;
    }
    Mat P(n);
    for (int i = 0; i < n; ++i)
      for (int j = 0; j < n; ++j) P(i, j) = weights[size_t(q) * n * n + size_t(i) * n + j];
    int plane_nnz = 0;
    for (double x : P.a) plane_nnz += x != 0.0;
    if (ndim == 3 && plane_nnz == 1) ++p.n_planes_point;
    factor_plane(P, radius, ndim == 2 ? 0 : q, tol, p.terms);
  }
  if (ndim == 3) {
    bool zs = true;
    for (int q = 0; q < radius && zs; ++q)
      for (int e = 0; e < n * n; ++e)
        if (weights[size_t(q) * n * n + e] != weights[size_t(n - 1 - q) * n * n + e]) { zs = false; break; }
    p.z_symmetric = zs ? 1 : 0;
  }
  // reconstruction check and growth (Q6: reject if > 1e-14)
  std::vector<double> Wr(nw, 0.0);
  double g = 0;
  for (const Term& t : p.terms) {
    double nu = 0, nv = 0;
    for (int i = 0; i < n; ++i) { nu += std::fabs(t.u[i]); nv += std::fabs(t.v[i]); }
    g += nu * nv;
    if (ndim == 1) {
      for (int j = 0; j < n; ++j) Wr[j] += t.u[radius] * t.v[j];
      continue;
    }
    for (int i = 0; i < n; ++i)
      for (int j = 0; j < n; ++j) Wr[size_t(t.plane) * n * n + size_t(i) * n + j] += t.u[i] * t.v[j];
  }
  double e = 0;
  for (size_t i = 0; i < nw; ++i) e = std::max(e, std::fabs(Wr[i] - weights[i]));
  p.recon_err = wmax > 0 ? e / wmax : 0.0;
  p.growth = w1 > 0 ? g / w1 : 0.0;
  if (p.recon_err > 1e-14) { err = "factorisation does not reconstruct W to 1e-14"; return LORA_ERR_FACTOR; }

  {  // row-pair split for the CUDA-core engine (Plan::rdg_rows)
    bool rows = ndim == 2 && radius >= 3;
    for (int a = 0; rows && a <= radius; ++a) rows = weights[size_t(radius + a) * n + radius] != 0.0;   // unit centre taps
    // integer-valued W (the integer-exact mode, pin P9): the unit-centre rescale W[R+a,:] / c_a is
    // not exact in general (c_a = 31 for the integer pyramid), so keep the planner's exact factors
    bool integral = true;
    for (size_t i = 0; integral && i < nw; ++i) integral = weights[i] == std::nearbyint(weights[i]);
    if (integral) rows = false;
    for (int i = 0; rows && i < n; ++i)
      for (int j = 0; j < n; ++j)
        if (weights[size_t(i) * n + j] != weights[size_t(n - 1 - i) * n + j] ||
            weights[size_t(i) * n + j] != weights[size_t(i) * n + (n - 1 - j)]) { rows = false; break; }
    const char* e = std::getenv("LORA_RDG_PMA");
    if (e && e[0] == '1') rows = false;
    p.rdg_rows = 0;
    if (rows) {  // only where it issues less than the planner's own factors (not for star arms)
      const double f_terms = cuda_fma_per_point(p);
      p.rdg_rows = 1;
      // Box-2D49P: 22 (row pairs, unit centre taps) vs 25 (PMA pyramid, unit centre taps)
      if (cuda_fma_per_point(p) > f_terms) p.rdg_rows = 0;
    }
  }
  p.fma_direct = nnz;
  p.fma_separable = 0;
  for (const Term& t : p.terms) {
    int lu = 0, lv = 0;
    for (int i = 0; i < n; ++i) { lu += t.u[i] != 0.0; lv += t.v[i] != 0.0; }
    p.fma_separable += (t.kind == kPoint) ? 1 : (t.kind == kArm ? std::max(lu, lv) : lu + lv);
  }
  // engine choice: lowest issued FP64 work at the measured pipe rates (DESIGN.md §Step 0:
  // DMMA 37 TF, DFMA 34 TF, one shared FP64 budget).
  int eng = o ? o->engine : LORA_ENGINE_AUTO;
  if (eng < 0 || eng > LORA_ENGINE_DIRECT) { err = "unknown engine"; return LORA_ERR_INVALID_ARG; }
  const double dense = p.ndim == 1 ? double(n) : (p.ndim == 2 ? double(n) * n : double(n) * n * n);  // every tap
  const double c_tc = tc_fma_per_point(p) / 37.0, c_rdg = cuda_fma_per_point(p) / 34.0, c_dir = dense / 34.0;
  const bool ok_tc = p.ndim >= 2 && tc2d_supported(p), ok_rdg = p.ndim == 1 || rdg2d_supported(p);
  if (eng == LORA_ENGINE_AUTO && p.ndim == 1) {
    eng = LORA_ENGINE_RDG_CUDA;  // 1D: the banded pass with temporal fusion (HBM-bound)
  } else if (eng == LORA_ENGINE_AUTO) {
    eng = LORA_ENGINE_DIRECT;
    double best = c_dir;
    if (ok_tc && c_tc < best) { best = c_tc; eng = LORA_ENGINE_TC; }
    if (ok_rdg && c_rdg < best) { best = c_rdg; eng = LORA_ENGINE_RDG_CUDA; }
  } else if ((eng == LORA_ENGINE_TC && !ok_tc) || (eng == LORA_ENGINE_RDG_CUDA && !ok_rdg)) {
    err = "requested engine does not support this stencil (ndim / term count)";
    return LORA_ERR_UNSUPPORTED;
  }
  p.engine = eng;
  p.fma_issued = eng == LORA_ENGINE_TC ? tc_fma_per_point(p) : eng == LORA_ENGINE_RDG_CUDA ? cuda_fma_per_point(p) : dense;
  int fk = o ? o->fuse_k : 0;
  if (fk < 0) { err = "fuse_k must be >= 0"; return LORA_ERR_INVALID_ARG; }
  const int max_k = eng == LORA_ENGINE_RDG_CUDA ? (p.ndim == 1 ? 8 : rdg2d_max_fuse(p))
                   : (eng == LORA_ENGINE_TC && p.ndim == 2 ? kMaxRadius / radius : 1);
  if (fk > max_k) { err = "fuse_k exceeds what the chosen engine supports for this stencil"; return LORA_ERR_UNSUPPORTED; }
  if (fk == 0) {
    // default fusion depth (exact temporal blocking), from B200 measurements
    // (profiles/r01_quickbench_*.jsonl): fusing pays while the CUDA-core engine is HBM-bound, i.e.
    // for light stencils (2D <= 20, 3D <= 12 issued FMA per point: Box-2D9P, Star-2D13P, Heat-3D,
    // 1D).  Box-2D49P (row-pair form, 25 FP64 ops/pt) fuses k = 2: unfused it is HBM-bound and hits
    // the 1 kW power cap under sustained load (~1.7 GHz), fused it is FP64-bound at full clock
    // (bench.py, 8 x 100 steps: 303 -> 320 GS/s); the same holds for Box-3D27P (307 -> 320).
    const double work = cuda_fma_per_point(p);
    if (eng != LORA_ENGINE_RDG_CUDA) fk = 1;   // composed fusion on tensor cores is opt-in (fuse_k > 1)
    else if (p.ndim == 1) fk = 8;
    else if (p.ndim == 3) fk = 2;   // Heat-3D; Box-3D27P too: sustained 307 (power-capped) -> 320 GS/s
    else if (p.rdg_rows && radius == 3) fk = 2;   // Box-2D49P: sustained (power-capped) 303 -> 320 GS/s
    else if (work > 20.0) fk = 1;
    else fk = radius == 1 ? 3 : 2;
    fk = std::min(max_k, fk);
  }
  p.fuse_k = fk;
  if (eng == LORA_ENGINE_TC && p.fuse_k > 1) {
    // composed kernel: W_k = W (*) W_{k-1} (full 2D convolution of the offset weights: applying the
    // correlation twice adds the offsets), radius kR; factored by the same planner (PMA / arms /
    // elimination).  Exact on points farther than (k-1)R from the Dirichlet halo; the band next
    // to it is recomputed stepwise by the launcher (reading Q5).
    const int k = p.fuse_k, cR = k * radius, cn = 2 * cR + 1;
    std::vector<double> Wk(p.W.begin(), p.W.end());
    int rk = radius;
    for (int step = 2; step <= k; ++step) {
      const int m = 2 * rk + 1, r2 = rk + radius, m2 = 2 * r2 + 1;
      std::vector<double> Wn(size_t(m2) * m2, 0.0);
      for (int a0 = 0; a0 < n; ++a0)
        for (int a1 = 0; a1 < n; ++a1)
          for (int b0 = 0; b0 < m; ++b0)
            for (int b1 = 0; b1 < m; ++b1) Wn[size_t(a0 + b0) * m2 + (a1 + b1)] += p.W[size_t(a0) * n + a1] * Wk[size_t(b0) * m + b1];
      Wk.swap(Wn);
      rk = r2;
    }
    p.cR = cR;
    p.cW = Wk;
    p.cterms.clear();
    Mat C(cn);
    double cmax = 0;
    for (int i = 0; i < cn * cn; ++i) { C.a[i] = Wk[i]; cmax = std::max(cmax, std::fabs(Wk[i])); }
    factor_plane(C, cR, 0, 1e-15 * cmax, p.cterms);
    double ce = 0;
    for (int i = 0; i < cn; ++i)
      for (int j = 0; j < cn; ++j) {
        double acc = 0;
        for (const Term& t : p.cterms) acc += t.u[i] * t.v[j];
        ce = std::max(ce, std::fabs(acc - C(i, j)));
      }
    if (cmax > 0 && ce / cmax > 1e-13) { err = "composed kernel does not factor to 1e-13"; return LORA_ERR_FACTOR; }
    if ((int)p.cterms.size() > 16) { err = "composed kernel has too many rank-1 terms for the TC engine"; return LORA_ERR_UNSUPPORTED; }
    lora::Plan cv = p;
    cv.R = cR; cv.W = Wk; cv.terms = p.cterms;
    p.fma_issued = tc_fma_per_point(cv) / k;
  }
  {
    const char* e = std::getenv("LORA_NO_TMA");
    p.force_no_tma = (e && e[0] == '1') ? 1 : 0;
    const char* b = std::getenv("LORA_TC_NO_BVS");
    p.tc_no_bvs = (b && b[0] == '1') ? 1 : 0;
    const char* sm = std::getenv("LORA_NO_SMALL");
    p.no_small = (sm && sm[0] == '1') ? 1 : 0;
    const char* smode = std::getenv("LORA_SMALL_MODE");   // tests: "cluster" / "grid" variants
    p.small_mode = !smode ? 0 : (std::strcmp(smode, "cluster") == 0 ? 1 : (std::strcmp(smode, "grid") == 0 ? 2 : 0));
    const char* srp = std::getenv("LORA_SMALL_RP");       // experiments: rows per CTA of the grid variant
    p.small_rp = srp ? std::max(1, std::atoi(srp)) : 2;   // Heat-2D 256^2 x 10: 2 -> 14.8 us, 4 -> 15.8, 8 -> 18.1
  }
  p.tile_m = eng == LORA_ENGINE_TC ? 64 : (p.ndim == 2 ? 64 : 8);
  p.tile_n = eng == LORA_ENGINE_TC ? 64 : 32;
  return LORA_OK;
}

}  // namespace lora
