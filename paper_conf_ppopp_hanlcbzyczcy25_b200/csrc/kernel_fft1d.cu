// Fused 1D FFT-stencil kernel: prime-factor tiles, one warp per tile pair (sm_100a).
//
// A 1D tile of L = N1*N2 = 8*7 = 56 cells (halo h = rT, valid S = L - 2h) is reshaped to an
// N1 x N2 matrix by the CRT ("diagonal") map l -> (l mod N1, l mod N2) (§3.2.1
// PFA L212, Diagonal Data Indexing §3.2.2; reading Q8), so its length-L DFT becomes
// the dense 2D DFT F_N1 . X . F_N2^T whose output is in the Ruritanian order of Eq. 8
// (the plan stores the powered spectrum in that order).  This turns the paper's sparse
// mat-vec (87.5% idle, L208-L210) into 8x8 matrix products: with N2 padded to 8 a whole
// complex tile pair is ONE 8x8 C tile per warp, and the four transforms
//   M1 = F_N2 . X^T,  M2 = F_N1 . M1^T (* S_T),  M3 = conj(F_N2) . M2^T,  M4 = conj(F_N1) . M3^T
// chain C fragment -> B fragment in registers (Swizzling Fragments, L266-L272) with no
// shared memory at all.  The DFT fragments and the spectrum stay in registers for the
// whole launch (Squeezing Registers / recomputation of iF from F, L274-L278).
#include "device_common.cuh"
#include "kernels.cuh"

namespace fstencil {
namespace {

using dev::dmma;

using dev::cgemm8;

template <bool WRAP>   // periodic boundary: a separate instantiation (no wrap arithmetic otherwise)
__global__ void __launch_bounds__(kFft1dWarpsPerBlock * 32) fft1d_kernel(const Fft1dArgs a) {
  const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
  const int64_t warp = a.win.p_begin + (int64_t)blockIdx.x * kFft1dWarpsPerBlock + (threadIdx.x >> 5);
  const int64_t nwarps = (int64_t)gridDim.x * kFft1dWarpsPerBlock;

  // A fragments: chunk j of row g is logical column 2q+j (device_common.cuh)
  double f1r[2], f1i[2], f2r[2], f2i[2], sr[2], si[2];
  int pos[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const int c = 2 * q + j;
    f1r[j] = a.Fre[g * 8 + c];
    f1i[j] = a.Fim[g * 8 + c];
    f2r[j] = a.Fre[(8 + g) * 8 + c];
    f2i[j] = a.Fim[(8 + g) * 8 + c];
    sr[j] = a.Sre[g * 8 + c];
    si[j] = a.Sim[g * 8 + c];
    pos[j] = a.crt[g * 8 + c];      // tile position of matrix cell (g, 2q+j); -1 = pad
  }
  const int L = a.L, S = a.S, h = a.h;

  const int64_t g0 = a.win.g0, g1 = a.win.g0 + a.win.gn;
  for (int64_t p = warp; p < a.win.p_end; p += nwarps) {
    const int64_t oa = 2 * p * S + a.bd.shift, ob = oa + S;   // global cell of tile position 0
    const bool has_b = 2 * p + 1 < a.ntiles;
    // B fragment of X^T:  X[l1 = g][l2 = 2q+j] = x[crt(g, 2q+j)]  (CRT gather, L1-resident)
    double xr[2], xi[2];
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      xr[j] = 0.0;
      xi[j] = 0.0;
      if (pos[j] >= 0) {
        int64_t xa = oa + pos[j], xb = ob + pos[j];
        if (WRAP) { xa = wrap_index(xa, a.n); xb = wrap_index(xb, a.n); }
        if (xa >= 0 && xa < a.n && xa >= g0 && xa < g1) xr[j] = __ldg(a.src + (xa - g0));
        if (has_b && xb >= 0 && xb < a.n && xb >= g0 && xb < g1) xi[j] = __ldg(a.src + (xb - g0));
      }
    }
    double m1r[2], m1i[2], m2r[2], m2i[2];
    cgemm8<false>(f2r, f2i, xr, xi, m1r, m1i);     // M1[k2][l1]
    cgemm8<false>(f1r, f1i, m1r, m1i, m2r, m2i);   // M2[k1][k2]  (Ruritanian spectrum)
#pragma unroll
    for (int j = 0; j < 2; ++j) {                  // * S_T (Eq. 10), 1/L folded in
      const double r = m2r[j] * sr[j] - m2i[j] * si[j];
      const double i = m2r[j] * si[j] + m2i[j] * sr[j];
      m2r[j] = r;
      m2i[j] = i;
    }
    cgemm8<true>(f2r, f2i, m2r, m2i, m1r, m1i);    // M3[l2][k1]
    cgemm8<true>(f1r, f1i, m1r, m1i, m2r, m2i);    // Y[l1][l2]
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      const int l = pos[j];
      if (l >= h && l < L - h) {                   // valid window (Eq. 7, reading Q4)
        const int64_t xa = oa + l, xb = ob + l;
        if (xa < a.bd.lim0 && xa >= a.win.w_lo && xa < a.win.w_hi) a.dst[xa - g0] = m2r[j];
        if (has_b && xb < a.bd.lim0 && xb >= a.win.w_lo && xb < a.win.w_hi) a.dst[xb - g0] = m2i[j];
      }
    }
  }
  (void)S;
}

}  // namespace

cudaError_t fused1d_configure(int* max_blocks) {
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft1d_kernel<false>, kFft1dWarpsPerBlock * 32, 0);
}

cudaError_t launch_fused1d(const Fft1dArgs& a, int grid, cudaStream_t s) {
  if (a.bd.wrap)
    fft1d_kernel<true><<<grid, kFft1dWarpsPerBlock * 32, 0, s>>>(a);
  else
    fft1d_kernel<false><<<grid, kFft1dWarpsPerBlock * 32, 0, s>>>(a);
  return cudaGetLastError();
}

}  // namespace fstencil
