// Register-resident radix-4 line transforms on the FP64 ALU (sm_100a).
//
// Why not the tensor pipe here: on B200 the FP64 tensor path (DMMA.8x8x4, 37 TF/s) and the
// FP64 FMA pipe (34 TF/s) have the same throughput and share it (profiles/r01_fp64_shared.txt),
// so a DFT-8 as a complex 8x8 GEMM costs 24-32 FP64 pipe operations per output while a
// butterfly FFT needs ~10 per output for a whole 16-point line.  The paper's choice of tensor
// cores (A100: DMMA = 2x DFMA) is prior art; on B200 the operation count decides.
//
// Conventions (reading Q7): forward X[k] = sum_n x[n] w^(nk) with
// w = exp(-2 pi i / N); the inverse uses conj(w) and is unnormalised (1/prod(L) is folded into
// the powered spectrum S_T).  Inputs and outputs are in natural order; the digit permutation
// of Cooley-Tukey is a compile-time register renaming.
#pragma once

namespace fstencil {
namespace radix {

// Multiply (re, im) by w16^m (forward) or its conjugate (INV), m in 0..15 a compile-time constant.
template <int M, bool INV>
__device__ __forceinline__ void tw16(double& re, double& im) {
  constexpr int m = M & 15;
  constexpr double C1 = 0.92387953251128673848, S1 = 0.38268343236508978178;   // cos, sin(pi/8)
  constexpr double K = 0.70710678118654752440;                                 // sqrt(2)/2
  constexpr double kCos[16] = {1, C1, K, S1, 0, -S1, -K, -C1, -1, -C1, -K, -S1, 0, S1, K, C1};
  constexpr double kSin[16] = {0, S1, K, C1, 1, C1, K, S1, 0, -S1, -K, -C1, -1, -C1, -K, -S1};
  // w16^m = c - i s with c = cos(pi m/8), s = sin(pi m/8); INV conjugates (s -> -s).
  // (re + i im)(c - i s) = (re c + im s) + i (im c - re s)
  constexpr double c = kCos[m];
  constexpr double s = INV ? -kSin[m] : kSin[m];
  if constexpr (m == 0) {
    return;
  } else if constexpr (c == 0.0) {        // +-i: a swap and a sign
    const double r = re;
    if constexpr (s > 0) { re = im; im = -r; } else { re = -im; im = r; }
  } else if constexpr (s == 0.0) {        // -1
    re = -re; im = -im;
  } else if constexpr (c == s) {          // K-forms: two adds, two multiplies
    const double a = re + im, b = im - re;
    re = a * c; im = b * c;
  } else if constexpr (c == -s) {
    const double a = re - im, b = im + re;
    re = a * c; im = b * c;
  } else {                                // general: two multiplies, two FMAs
    const double t = im * s;
    const double u = re * s;
    re = fma(re, c, t);
    im = fma(im, c, -u);
  }
}

// DFT-4 of (a0, a1, a2, a3) in place (natural order out); forward w4 = -i, INV +i.
template <bool INV>
__device__ __forceinline__ void dft4(double& r0, double& i0, double& r1, double& i1, double& r2, double& i2, double& r3,
                                     double& i3) {
  const double sr0 = r0 + r2, si0 = i0 + i2, dr0 = r0 - r2, di0 = i0 - i2;
  const double sr1 = r1 + r3, si1 = i1 + i3, dr1 = r1 - r3, di1 = i1 - i3;
  r0 = sr0 + sr1; i0 = si0 + si1;
  r2 = sr0 - sr1; i2 = si0 - si1;
  if (!INV) {   // X1 = d0 - i d1, X3 = d0 + i d1
    r1 = dr0 + di1; i1 = di0 - dr1;
    r3 = dr0 - di1; i3 = di0 + dr1;
  } else {      // X1 = d0 + i d1, X3 = d0 - i d1
    r1 = dr0 - di1; i1 = di0 + dr1;
    r3 = dr0 + di1; i3 = di0 - dr1;
  }
}

// FP64 pipe instructions (adds, multiplies, FMAs) of one fft16: 8 DFT-4 (128 adds) + the
// nine twiddles w16^(n2 k1) (m = 1,2,3,2,4,6,3,6,9: four general (2 mul + 2 fma), four
// K(1 -+ i) (2 add + 2 mul), one -i (free)) = 160 instructions, 168 flops (an FMA is 2).
constexpr int kFft16Instr = 160;
constexpr int kFft16Flops = 168;

// 16-point DFT in registers, 16 = 4 x 4 (n = 4 n1 + n2, k = k1 + 4 k2):
//   X[k1 + 4 k2] = sum_n2 w4^(n2 k2) w16^(n2 k1) sum_n1 w4^(n1 k1) x[4 n1 + n2]
template <bool INV>
__device__ __forceinline__ void fft16(double (&xr)[16], double (&xi)[16]) {
#pragma unroll
  for (int n2 = 0; n2 < 4; ++n2)   // DFT-4 over n1: Y[n2][k1] lands in slot 4 k1 + n2
    dft4<INV>(xr[n2], xi[n2], xr[4 + n2], xi[4 + n2], xr[8 + n2], xi[8 + n2], xr[12 + n2], xi[12 + n2]);
  tw16<1, INV>(xr[5], xi[5]);     // slot 4 k1 + n2 gets w16^(n2 k1)
  tw16<2, INV>(xr[6], xi[6]);
  tw16<3, INV>(xr[7], xi[7]);
  tw16<2, INV>(xr[9], xi[9]);
  tw16<4, INV>(xr[10], xi[10]);
  tw16<6, INV>(xr[11], xi[11]);
  tw16<3, INV>(xr[13], xi[13]);
  tw16<6, INV>(xr[14], xi[14]);
  tw16<9, INV>(xr[15], xi[15]);
#pragma unroll
  for (int k1 = 0; k1 < 4; ++k1)   // DFT-4 over n2: X[k1 + 4 k2] lands in slot 4 k1 + k2
    dft4<INV>(xr[4 * k1], xi[4 * k1], xr[4 * k1 + 1], xi[4 * k1 + 1], xr[4 * k1 + 2], xi[4 * k1 + 2],
              xr[4 * k1 + 3], xi[4 * k1 + 3]);
  // slot 4 k1 + k2 holds X[k1 + 4 k2]: transpose the 4 x 4 register block (renaming only)
  double yr[16], yi[16];
#pragma unroll
  for (int k1 = 0; k1 < 4; ++k1)
#pragma unroll
    for (int k2 = 0; k2 < 4; ++k2) {
      yr[k1 + 4 * k2] = xr[4 * k1 + k2];
      yi[k1 + 4 * k2] = xi[4 * k1 + k2];
    }
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    xr[k] = yr[k];
    xi[k] = yi[k];
  }
}

// 8-point DFT in registers (radix-2 DIT over two DFT-4s), natural order in and out:
//   X[k] = E[k] + w8^k O[k], X[k + 4] = E[k] - w8^k O[k], E/O = DFT-4 of the even/odd inputs.
// 56 FP64 instructions (2 x 16 + two K-form twiddles of 4 + 16 butterfly adds), 56 flops.
constexpr int kFft8Instr = 56;
template <bool INV>
__device__ __forceinline__ void fft8(double (&xr)[8], double (&xi)[8]) {
  dft4<INV>(xr[0], xi[0], xr[2], xi[2], xr[4], xi[4], xr[6], xi[6]);   // E0..E3 in slots 0, 2, 4, 6
  dft4<INV>(xr[1], xi[1], xr[3], xi[3], xr[5], xi[5], xr[7], xi[7]);   // O0..O3 in slots 1, 3, 5, 7
  tw16<2, INV>(xr[3], xi[3]);   // w8^1 O1
  tw16<4, INV>(xr[5], xi[5]);   // w8^2 O2
  tw16<6, INV>(xr[7], xi[7]);   // w8^3 O3
  double yr[8], yi[8];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    yr[k] = xr[2 * k] + xr[2 * k + 1];
    yi[k] = xi[2 * k] + xi[2 * k + 1];
    yr[k + 4] = xr[2 * k] - xr[2 * k + 1];
    yi[k + 4] = xi[2 * k] - xi[2 * k + 1];
  }
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    xr[k] = yr[k];
    xi[k] = yi[k];
  }
}

// (re + i im) *= (wr + i wi): 2 multiplies + 2 FMAs (6 flops).
__device__ __forceinline__ void cmul(double& re, double& im, double wr, double wi) {
  const double t = im * wi, u = re * wi;
  re = fma(re, wr, -t);
  im = fma(im, wr, u);
}

}  // namespace radix
}  // namespace fstencil
