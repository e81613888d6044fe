// Register-chained length-64 line transforms shared by the factored (Cooley-Tukey 8 x 8)
// kernels, sm_100a.  One 64-element complex line is one 8x8 matrix held by one warp in
// DMMA.8x8x4 fragments (device_common.cuh); F8 and the 8x8 twiddles w64^(ka lb) stay in
// registers.  Both routes contract the columns of the current C fragment (§3.3
// "Swizzling Fragments", L266-L272):
//   B-route  C' = F8 . C^T     (C's fragment is the B fragment of C^T)
//   A-route  C' = C . F8^T     (C's fragment is the A fragment of C)
// A line read at positions cl[j] = 16q + 8j + g (natural index l = 8 la + lb) maps through
// B-route, twiddle, A-route to its DFT-64 at the same positions (k = ka + 8 kb = cl[j]);
// the inverse (conjugated) chain maps frequencies at cl[j] back to positions cl[j].
#pragma once

#include "device_common.cuh"

namespace fstencil {
namespace ct {

using dev::dmma;

constexpr int L = 64;

// XOR-swizzled dense layout: both fragment patterns (row r fixed, c = 16q + 8j + g; and
// column c fixed, r = 16q + 8j + g) are conflict-free per half-warp (8-byte accesses are
// served 16 lanes at a time: lanes 4g + q, g in one half), the optimal 2 wavefronts per 32
// doubles; a permutation within each row; 64 KB for the two planes (3 CTAs / SM).
__device__ __forceinline__ int sw(int r, int c) {
  return r * L + (c ^ (((((c >> 4) & 3) ^ ((r >> 4) & 3))) << 2) ^ (r & 3));
}

// B-route: C = F8 . B (F8 fragments f*, data fragments b*), CONJ -> conj(F8).
template <bool CONJ>
__device__ __forceinline__ void broute(double (&cr)[2], double (&ci)[2], const double (&fr)[2], const double (&fi)[2],
                                       const double (&br)[2], const double (&bi)[2]) {
  cr[0] = cr[1] = ci[0] = ci[1] = 0.0;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    if (CONJ) {
      dmma(cr, fr[j], br[j]);
      dmma(ci, fr[j], bi[j]);
      dmma(cr, fi[j], bi[j]);
      dmma(ci, -fi[j], br[j]);
    } else {
      dmma(cr, fr[j], br[j]);
      dmma(ci, fr[j], bi[j]);
      dmma(cr, -fi[j], bi[j]);
      dmma(ci, fi[j], br[j]);
    }
  }
}

// A-route: C = D . F8^T (data fragments d* as A, F8^T fragments = F8 fragments as B).
template <bool CONJ>
__device__ __forceinline__ void aroute(double (&cr)[2], double (&ci)[2], const double (&dr)[2], const double (&di)[2],
                                       const double (&fr)[2], const double (&fi)[2]) {
  cr[0] = cr[1] = ci[0] = ci[1] = 0.0;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    if (CONJ) {
      dmma(cr, dr[j], fr[j]);
      dmma(ci, di[j], fr[j]);
      dmma(cr, di[j], fi[j]);
      dmma(ci, -dr[j], fi[j]);
    } else {
      dmma(cr, dr[j], fr[j]);
      dmma(ci, di[j], fr[j]);
      dmma(cr, -di[j], fi[j]);
      dmma(ci, dr[j], fi[j]);
    }
  }
}

template <bool CONJ>
__device__ __forceinline__ void twiddle(double (&cr)[2], double (&ci)[2], const double (&tr)[2], const double (&ti)[2]) {
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const double t_i = CONJ ? -ti[j] : ti[j];
    const double r = cr[j] * tr[j] - ci[j] * t_i;
    const double i = cr[j] * t_i + ci[j] * tr[j];
    cr[j] = r;
    ci[j] = i;
  }
}

// NL independent lines per warp, their DMMA chains interleaved for latency hiding.
// Complex 8x8x8 products as real DMMAs.  FFTSTENCIL_CMUL3 = 1 (default): the 3-multiply
// form (Gauss / "3M"), P1 = Ar Br, P2 = Ai Bi, P3 = (Ar + Ai)(Br + Bi),
// Re = P1 - P2, Im = P3 - P1 - P2 -- 6 DMMA.8x8x4 per product instead of 8, for 8 FP64
// adds per thread; 0: the 4-multiply form.  The 1D and 2D factored kernels use it; the 3D one
// (less tensor-bound, measured profiles/r01_cmul3.jsonl) keeps 4M (FFTSTENCIL_CMUL3_3D).
#ifndef FFTSTENCIL_CMUL3
#define FFTSTENCIL_CMUL3 1
#endif
#ifndef FFTSTENCIL_CMUL3_3D
#define FFTSTENCIL_CMUL3_3D 0
#endif

template <int NL>
__device__ __forceinline__ void finish3(double (&cr)[NL][2], double (&ci)[NL][2], const double (&p1)[NL][2],
                                        const double (&p2)[NL][2], const double (&p3)[NL][2]) {
#pragma unroll
  for (int u = 0; u < NL; ++u)
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      cr[u][e] = p1[u][e] - p2[u][e];
      ci[u][e] = p3[u][e] - p1[u][e] - p2[u][e];
    }
}

// B-route: C = F8' . B with F8' = F8 (CONJ = false) or conj(F8).
template <bool CONJ, int NL, bool M3 = FFTSTENCIL_CMUL3 != 0>
__device__ __forceinline__ void broute_n(double (&cr)[NL][2], double (&ci)[NL][2], const double (&fr)[2],
                                         const double (&fi)[2], const double (&br)[NL][2], const double (&bi)[NL][2]) {
  if constexpr (M3) {
  double p1[NL][2], p2[NL][2], p3[NL][2];
#pragma unroll
  for (int u = 0; u < NL; ++u) p1[u][0] = p1[u][1] = p2[u][0] = p2[u][1] = p3[u][0] = p3[u][1] = 0.0;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const double f_i = CONJ ? -fi[j] : fi[j];
    const double fs = fr[j] + f_i;
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(p1[u], fr[j], br[u][j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(p2[u], f_i, bi[u][j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(p3[u], fs, br[u][j] + bi[u][j]);
  }
  finish3<NL>(cr, ci, p1, p2, p3);
  } else {
#pragma unroll
  for (int u = 0; u < NL; ++u) cr[u][0] = cr[u][1] = ci[u][0] = ci[u][1] = 0.0;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const double nfi = CONJ ? fi[j] : -fi[j];   // coefficient of bi in cr
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(cr[u], fr[j], br[u][j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(ci[u], fr[j], bi[u][j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(cr[u], nfi, bi[u][j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(ci[u], -nfi, br[u][j]);
  }
  }
}

// A-route: C = D . F8'^T.
template <bool CONJ, int NL, bool M3 = FFTSTENCIL_CMUL3 != 0>
__device__ __forceinline__ void aroute_n(double (&cr)[NL][2], double (&ci)[NL][2], const double (&dr)[NL][2],
                                         const double (&di)[NL][2], const double (&fr)[2], const double (&fi)[2]) {
  if constexpr (M3) {
  double p1[NL][2], p2[NL][2], p3[NL][2];
#pragma unroll
  for (int u = 0; u < NL; ++u) p1[u][0] = p1[u][1] = p2[u][0] = p2[u][1] = p3[u][0] = p3[u][1] = 0.0;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const double f_i = CONJ ? -fi[j] : fi[j];
    const double fs = fr[j] + f_i;
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(p1[u], dr[u][j], fr[j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(p2[u], di[u][j], f_i);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(p3[u], dr[u][j] + di[u][j], fs);
  }
  finish3<NL>(cr, ci, p1, p2, p3);
  } else {
#pragma unroll
  for (int u = 0; u < NL; ++u) cr[u][0] = cr[u][1] = ci[u][0] = ci[u][1] = 0.0;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const double nfi = CONJ ? fi[j] : -fi[j];
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(cr[u], dr[u][j], fr[j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(ci[u], di[u][j], fr[j]);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(cr[u], di[u][j], nfi);
#pragma unroll
    for (int u = 0; u < NL; ++u) dmma(ci[u], dr[u][j], -nfi);
  }
  }
}

template <bool CONJ, int NL>
__device__ __forceinline__ void twiddle_n(double (&cr)[NL][2], double (&ci)[NL][2], const double (&tr)[2],
                                          const double (&ti)[2]) {
#pragma unroll
  for (int u = 0; u < NL; ++u) twiddle<CONJ>(cr[u], ci[u], tr, ti);
}

}  // namespace ct
}  // namespace fstencil
