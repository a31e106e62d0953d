/*
 * TEST INFRASTRUCTURE ONLY — the CPU oracle for the LoRAStencil hot path.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  The product (paper_conf_sc_zhanglyczcy24_b200/) never
 * links, imports or calls it, and shares no code with it.
 *
 * What it computes: the plain definition of a time-iterated stencil.
 *   * PAPER.md P:21 (§I): "iteratively updates each point within a d-dimensional spatial
 *     grid along the temporal dimension by the weighted sum of itself and neighboring points".
 *   * PAPER.md P:98-105 (§II-D, eq. 2): the update of one point is the Frobenius inner
 *     product <C, X>_F = sum_i sum_j c_ij x_ij of the weight matrix with the neighbourhood.
 *   * Readings: Dirichlet halo of width h held
 *     fixed; correlation orientation (W[a] multiplies in[x + a - h]); Jacobi double buffer.
 *
 * Loop order: weights lexicographic, last axis fastest; s starts at +0.0 and each product
 * is rounded before the add (built with -ffp-contract=off, no FMA contraction).  The result
 * is therefore bitwise independent of the OpenMP thread count (each point is computed by
 * one thread in a fixed order).
 *
 * d = 1, 2, 3.  Layout: `in`/`out` are padded arrays of extent (N_i + 2h) per axis, C order, slowest first.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static void step1d(const double* W, int h, int64_t N0, const double* A, double* B) {
  const int n = 2 * h + 1;
#pragma omp parallel for schedule(static)
  for (int64_t x0 = h; x0 < h + N0; ++x0) {
    double s = 0.0;
    for (int a0 = 0; a0 < n; ++a0) {
      double p = W[a0] * A[x0 + a0 - h];
      s = s + p;
    }
    B[x0] = s;
  }
}

static void step2d(const double* W, int h, int64_t N0, int64_t N1, const double* A, double* B) {
  const int64_t P1 = N1 + 2 * h;
  const int n = 2 * h + 1;
#pragma omp parallel for schedule(static)
  for (int64_t x0 = h; x0 < h + N0; ++x0) {
    for (int64_t x1 = h; x1 < h + N1; ++x1) {
      double s = 0.0;
      for (int a0 = 0; a0 < n; ++a0)
        for (int a1 = 0; a1 < n; ++a1) {
          double p = W[a0 * n + a1] * A[(x0 + a0 - h) * P1 + (x1 + a1 - h)];
          s = s + p;
        }
      B[x0 * P1 + x1] = s;
    }
  }
}

static void step3d(const double* W, int h, int64_t N0, int64_t N1, int64_t N2, const double* A, double* B) {
  const int64_t P1 = N1 + 2 * h, P2 = N2 + 2 * h;
  const int n = 2 * h + 1;
#pragma omp parallel for schedule(static)
  for (int64_t x0 = h; x0 < h + N0; ++x0) {
    for (int64_t x1 = h; x1 < h + N1; ++x1) {
      for (int64_t x2 = h; x2 < h + N2; ++x2) {
        double s = 0.0;
        for (int a0 = 0; a0 < n; ++a0)
          for (int a1 = 0; a1 < n; ++a1)
            for (int a2 = 0; a2 < n; ++a2) {
              double p = W[(a0 * n + a1) * n + a2] *
                         A[((x0 + a0 - h) * P1 + (x1 + a1 - h)) * P2 + (x2 + a2 - h)];
              s = s + p;
            }
        B[(x0 * P1 + x1) * P2 + x2] = s;
      }
    }
  }
}

/* Runs T Jacobi steps.  `out` receives the padded result (halo = input halo).
 * nthreads <= 0 keeps the OpenMP default.  Returns 0, or -1 on bad arguments / OOM. */
int oracle_stencil_run(const double* W, int ndim, int h, const int64_t* N, const double* in, double* out,
                       int64_t T, int nthreads) {
  if (ndim < 1 || ndim > 3 || h < 1 || T < 0 || !W || !N || !in || !out) return -1;
  int64_t total = 1;
  for (int i = 0; i < ndim; ++i) {
    if (N[i] < 1) return -1;
    total *= N[i] + 2 * h;
  }
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
  double* A = out;
  double* B = (double*)malloc((size_t)total * sizeof(double));
  if (!B) return -1;
  memcpy(A, in, (size_t)total * sizeof(double));
  memcpy(B, in, (size_t)total * sizeof(double)); /* halo of both buffers = the fixed boundary */
  for (int64_t t = 0; t < T; ++t) {
    if (ndim == 1) step1d(W, h, N[0], A, B);
    else if (ndim == 2) step2d(W, h, N[0], N[1], A, B);
    else step3d(W, h, N[0], N[1], N[2], A, B);
    double* tmp = A; A = B; B = tmp;
  }
  if (A != out) { /* odd T: the result landed in the scratch buffer */
    memcpy(out, A, (size_t)total * sizeof(double));
    free(A);
  } else {
    free(B);
  }
  return 0;
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
