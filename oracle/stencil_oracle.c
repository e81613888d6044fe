/*
 * oracle/stencil_oracle.c -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.
 *
 * The CPU oracle for the FlashFFTStencil hot path: the plain definition of an
 * iterated stencil, applied directly, one time step at a time, in FP64.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this file's shared object.  It shares no code,
 * header, table or helper with the CUDA path (paper_conf_ppopp_hanlcbzyczcy25_b200/).
 *
 * What it follows (PAPER.md line numbers, /root/reference/PAPER.md):
 *   L93  (§2.2)  "The value of a point at time t is a weighted sum of the values of
 *                its neighboring points from the previous time steps."
 *   Eq. 2 L162   Y[n] = sum_m K[m] X[n-m]   (one time step is a weighted sum)
 *   Fig. 2 left L111-L128  the time-step loop  for t = 1..T: a_t <- stencil(a_{t-1})
 *   Eq. 10 L290  a_T is the result after T time iterations (the FFT path must equal it).
 * Readings:
 *   Q1  correlation form: u'[c] = sum_{o in [-r,r]^d} w[o] * u[c+o]; weights in
 *       offset-cube row-major order, axis 0 outermost (Eq. 2 with K[m] = w[r-m]).
 *   Q2  fixed boundary: ring cells (some c_a < r or c_a >= n_a - r) keep their input
 *       value for every step; periodic wrap-around exists for oracle self-tests only.
 *   Q17 summation order: lexicographic over o (o_0 outermost), starting from 0.0,
 *       plain IEEE FP64 (compiled without -ffast-math, with -ffp-contract=off).
 *
 * Two entry points evaluate the SAME definition:
 *   oracle_stencil_run    the whole grid, step by step;
 *   oracle_stencil_point  one cell, by stepping only the sub-box of radius r*steps
 *                         around it (its dependency cone).  Every cell that can
 *                         influence the result is updated by the identical
 *                         expression in the identical order, so the value is
 *                         bitwise equal to oracle_stencil_run's at that cell
 *                         (pinned in tests/test_oracle.py).
 *
 * Parity pins (tests/test_oracle.py): hand-expanded sums, binomial closed form,
 * constant-field invariance, plane-wave eigenvalue (periodic), Toeplitz sine-mode
 * eigenvalues (fixed ring), impulse response vs numpy/scipy convolution,
 * linearity, semigroup, maximum principle.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Embed the grid in 3 axes: a d-dim grid becomes (1,..,1,n_0..n_{d-1}). */
static void embed3(int ndim, const int64_t* ext, int64_t n[3], int active[3]) {
  for (int a = 0; a < 3; ++a) { n[a] = 1; active[a] = 0; }
  for (int a = 0; a < ndim; ++a) { n[3 - ndim + a] = ext[a]; active[3 - ndim + a] = 1; }
}

/*
 * One time step on a box of the grid: dst <- stencil(src).
 * The box is [blo, blo+bn) in global coordinates of a grid of extents n; src/dst
 * hold the box in C order.  Definition of L93 / Eq. 2 with readings Q1, Q2:
 *   ring cell                -> keeps its value (fixed boundary)
 *   neighbourhood in the box -> sum_o w[o] * src[c+o], lexicographic o, from 0.0
 *   otherwise (box edge)     -> keeps its value; such cells are outside the
 *                               dependency cone of every cell the caller reads.
 * periodic=1 only with the box equal to the whole grid: every cell is updated and
 * c+o wraps modulo n.
 */
static void one_step(const int64_t n[3], const int active[3], const int64_t blo[3],
                     const int64_t bn[3], int r, int periodic, const double* w,
                     const double* src, double* dst) {
  const int64_t lo[3] = {active[0] ? -r : 0, active[1] ? -r : 0, active[2] ? -r : 0};
  const int64_t hi[3] = {active[0] ? r : 0, active[1] ? r : 0, active[2] ? r : 0};
  const int64_t wd = 2 * (int64_t)r + 1;
#pragma omp parallel for schedule(static)
  for (int64_t b0 = 0; b0 < bn[0]; ++b0) {
    for (int64_t b1 = 0; b1 < bn[1]; ++b1) {
      for (int64_t b2 = 0; b2 < bn[2]; ++b2) {
        const int64_t b[3] = {b0, b1, b2};
        const int64_t c[3] = {blo[0] + b0, blo[1] + b1, blo[2] + b2}; /* global cell */
        const int64_t idx = (b0 * bn[1] + b1) * bn[2] + b2;
        int keep = 0;
        for (int a = 0; a < 3 && !periodic; ++a) {
          if (!active[a]) continue;
          if (c[a] < r || c[a] >= n[a] - r) keep = 1;               /* ring cell */
          if (b[a] + lo[a] < 0 || b[a] + hi[a] >= bn[a]) keep = 1;  /* box edge */
        }
        if (keep) { dst[idx] = src[idx]; continue; }
        double acc = 0.0;
        for (int64_t o0 = lo[0]; o0 <= hi[0]; ++o0)
          for (int64_t o1 = lo[1]; o1 <= hi[1]; ++o1)
            for (int64_t o2 = lo[2]; o2 <= hi[2]; ++o2) {
              const int64_t o[3] = {o0, o1, o2};
              int64_t p[3];
              for (int a = 0; a < 3; ++a) {
                p[a] = b[a] + o[a];
                if (periodic) p[a] = ((p[a] % bn[a]) + bn[a]) % bn[a];
              }
              /* weight index: offset-cube row-major over the active axes */
              int64_t k = 0;
              for (int a = 0; a < 3; ++a)
                if (active[a]) k = k * wd + (o[a] + r);
              acc += w[k] * src[(p[0] * bn[1] + p[1]) * bn[2] + p[2]];
            }
        dst[idx] = acc;
      }
    }
  }
}

static int set_threads(int nthreads) {
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
  return 0;
}

/*
 * oracle_stencil_run: out <- `steps` time steps of the stencil applied to u0.
 *   ndim in {1,2,3}; extents[ndim] (axis 0 outermost, C order, includes the ring);
 *   weights[(2r+1)^ndim]; periodic = 0 (fixed ring, the product's semantics) or 1.
 *   nthreads <= 0 uses the OpenMP default.  Returns 0, or -1 on invalid arguments.
 *   u0 and out may alias.
 */
int oracle_stencil_run(int ndim, const int64_t* extents, const double* weights, int radius,
                       int64_t steps, int periodic, const double* u0, double* out,
                       int nthreads) {
  if (ndim < 1 || ndim > 3 || radius < 1 || steps < 0 || !extents || !weights || !u0 || !out)
    return -1;
  int64_t n[3]; int active[3];
  embed3(ndim, extents, n, active);
  for (int a = 0; a < 3; ++a) if (n[a] < 1) return -1;
  const int64_t total = n[0] * n[1] * n[2];
  const int64_t zero[3] = {0, 0, 0};
  set_threads(nthreads);
  double* a = (double*)malloc(sizeof(double) * (size_t)total);
  double* b = (double*)malloc(sizeof(double) * (size_t)total);
  if (!a || !b) { free(a); free(b); return -1; }
  memcpy(a, u0, sizeof(double) * (size_t)total);
  for (int64_t s = 0; s < steps; ++s) {            /* Fig. 2 left: for t = 1..T */
    one_step(n, active, zero, n, radius, periodic, weights, a, b);
    double* t = a; a = b; b = t;
  }
  memcpy(out, a, sizeof(double) * (size_t)total);
  free(a); free(b);
  return 0;
}

/*
 * oracle_stencil_point: the fixed-boundary value of ONE cell after `steps` steps.
 *   cells[npts*ndim] global coordinates; writes values[npts].  Same definition as
 *   oracle_stencil_run (fixed ring only).  Returns 0 or -1.
 */
int oracle_stencil_point(int ndim, const int64_t* extents, const double* weights, int radius,
                         int64_t steps, const double* u0, int64_t npts, const int64_t* cells,
                         double* values, int nthreads) {
  if (ndim < 1 || ndim > 3 || radius < 1 || steps < 0 || !extents || !weights || !u0 ||
      !cells || !values || npts < 0)
    return -1;
  int64_t n[3]; int active[3];
  embed3(ndim, extents, n, active);
  set_threads(nthreads);
  for (int64_t q = 0; q < npts; ++q) {
    int64_t c[3] = {0, 0, 0}, blo[3], bn[3];
    for (int a = 0; a < ndim; ++a) c[3 - ndim + a] = cells[q * ndim + a];
    for (int a = 0; a < 3; ++a) {
      if (c[a] < 0 || c[a] >= n[a]) return -1;
      int64_t reach = active[a] ? (int64_t)radius * steps : 0;
      int64_t l = c[a] - reach, h = c[a] + reach;
      if (l < 0) l = 0;
      if (h > n[a] - 1) h = n[a] - 1;
      blo[a] = l; bn[a] = h - l + 1;
    }
    const int64_t tot = bn[0] * bn[1] * bn[2];
    double* a = (double*)malloc(sizeof(double) * (size_t)tot);
    double* b = (double*)malloc(sizeof(double) * (size_t)tot);
    if (!a || !b) { free(a); free(b); return -1; }
    for (int64_t i0 = 0; i0 < bn[0]; ++i0)
      for (int64_t i1 = 0; i1 < bn[1]; ++i1)
        memcpy(a + (i0 * bn[1] + i1) * bn[2],
               u0 + ((blo[0] + i0) * n[1] + (blo[1] + i1)) * n[2] + blo[2],
               sizeof(double) * (size_t)bn[2]);
    for (int64_t s = 0; s < steps; ++s) {
      one_step(n, active, blo, bn, radius, 0, weights, a, b);
      double* t = a; a = b; b = t;
    }
    values[q] = a[((c[0] - blo[0]) * bn[1] + (c[1] - blo[1])) * bn[2] + (c[2] - blo[2])];
    free(a); free(b);
  }
  return 0;
}

/* The number of OpenMP threads a parallel region would use (for reporting). */
int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
