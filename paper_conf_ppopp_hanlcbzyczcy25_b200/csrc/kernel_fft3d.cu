// Fused 3D FFT-stencil tile kernel: 16^3 tiles, FP64 tensor cores (DMMA.8x8x4), sm_100a.
//
// PAPER.md §3.2.1 "Multidimensional Data Handling" (L220, Fig. 4a): higher-dimensional
// data is processed as 2D slices.  One CTA takes a pair of 16^3 overlap-save tiles (halo
// h = rT; Double-layer Filling Eq. 9 makes them the Re/Im planes of one complex tile) and
// runs Algorithm 1 (L252-L258) in three phases separated by the two shared-memory
// transpositions of ownership a 3D transform needs:
//   phase 1  warps own l0 slices:   Q[l0] = F . X[l0] . F^T     (axes 2 and 1, registers chain)
//   phase 2  warps own (k1,k2) rows: Z = Q^(0) . F (axis 0, data as the A operand from SMEM),
//            Z *= S_T (Eq. 10), W = conj(F)[h:h+S] . Z^T (inverse axis 0, crop-aware)
//   phase 3  warps own output l0 slices: Y[l0] = conj(F)[h:h+S] . (conj(F)[h:h+S] . W[l0]^T)^T
//            (inverse axes 2 and 1, crop-aware), then the S^3 window is stored (Eq. 7).
// Every product flips orientation so its C fragments are the next product's B fragments
// (Swizzling Fragments, L266-L272); phase 2 writes W over the columns it alone read.
#include "device_common.cuh"
#include "kernels.cuh"

namespace fstencil {
namespace {

using dev::dmma;
using dev::perm8;

constexpr int L = 16;
constexpr int LD = 20;             // row stride (doubles) of a 16-wide row: 8-bank shift
constexpr int SL = 16 * LD + 4;    // slice stride: 8-bank shift between consecutive slices
constexpr int NW3 = 8;             // warps per CTA

template <bool CONJ>
__device__ __forceinline__ void cmma(double (&cr)[2], double (&ci)[2], double ar, double ai, double br, double bi) {
  if (CONJ) {
    dmma(cr, ar, br);
    dmma(cr, ai, bi);
    dmma(ci, ar, bi);
    dmma(ci, -ai, br);
  } else {
    dmma(cr, ar, br);
    dmma(cr, -ai, bi);
    dmma(ci, ar, bi);
    dmma(ci, ai, br);
  }
}

template <bool WRAP>   // periodic boundary: a separate instantiation
__global__ void __launch_bounds__(NW3 * 32) fft3d_kernel(const Fft3dArgs a) {
  extern __shared__ __align__(16) double smem[];
  double* sFr = smem;
  double* sFi = sFr + L * LD;
  double* sXa = sFi + L * LD;      // 16 slices x 16 rows x LD (+4 per slice)
  double* sXb = sXa + L * SL;

  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31, g = lane >> 2, q = lane & 3;
  for (int e = tid; e < L * L; e += NW3 * 32) {
    const int r = e >> 4, c = e & 15;
    sFr[r * LD + perm8(c)] = a.Fre[e];
    sFi[r * LD + perm8(c)] = a.Fim[e];
  }
  const int S = a.S, h = a.h;
  const int MT = (S + 7) >> 3;     // output 8-tiles per axis (1 or 2)
  // pair p = tiles (t0, t1, 2j) and (t0, t1, 2j+1): line = p / npr = t0 * nt1 + t1 (kernels.cuh)
  for (int64_t p = a.win.p_begin + blockIdx.x; p < a.win.p_end; p += gridDim.x) {
    __syncthreads();
    const int64_t line = p / a.npr, pj = p - line * a.npr;
    const int64_t t0 = line / a.nt1, t1 = line - t0 * a.nt1;
    const int64_t o0 = t0 * S + a.bd.shift, o1 = t1 * S + a.bd.shift;
    // ---- load the halo'd pair: rows of 16 doubles (128 B), OOB = 0 ----
#pragma unroll
    for (int t = 0; t < 2; ++t) {
      const int64_t t2 = 2 * pj + t;
      double* sX = t ? sXb : sXa;
      const bool have = t2 < a.nt2;
      const int64_t o2 = t2 * S + a.bd.shift;
      for (int e = tid; e < L * L * L; e += NW3 * 32) {
        const int l0 = e >> 8, l1 = (e >> 4) & 15, l2 = e & 15;
        double v = 0.0;
        if (have) {
          int64_t g0 = o0 + l0, g1 = o1 + l1, g2 = o2 + l2;
          if (WRAP) { g0 = wrap_index(g0, a.n0); g1 = wrap_index(g1, a.n1); g2 = wrap_index(g2, a.n2); }
          const int64_t lg0 = g0 - a.win.g0;
          if (g0 < a.n0 && lg0 >= 0 && lg0 < a.win.gn && g1 >= 0 && g1 < a.n1 && g2 >= 0 && g2 < a.n2)
            v = __ldg(a.src + (lg0 * a.n1 + g1) * a.n2 + g2);
        }
        sX[l0 * SL + l1 * LD + perm8(l2)] = v;
      }
    }
    __syncthreads();

    // ---- phase 1: per l0 slice, Q = F . X . F^T (forward along axes 2 then 1) ----
    for (int l0 = warp; l0 < L; l0 += NW3) {
      const double* xa = sXa + l0 * SL;
      const double* xb = sXb + l0 * SL;
      double M1r[2][2][2], M1i[2][2][2];   // [k2 tile][l1 tile][j]
#pragma unroll
      for (int m = 0; m < 2; ++m)
#pragma unroll
        for (int n = 0; n < 2; ++n) M1r[m][n][0] = M1r[m][n][1] = M1i[m][n][0] = M1i[m][n][1] = 0.0;
#pragma unroll
      for (int kc = 0; kc < 4; ++kc) {     // l2 chunk (physical columns 4kc..4kc+3)
        const int pc = 4 * kc + q;
        double br[2], bi[2];
#pragma unroll
        for (int n = 0; n < 2; ++n) { br[n] = xa[(8 * n + g) * LD + pc]; bi[n] = xb[(8 * n + g) * LD + pc]; }
#pragma unroll
        for (int m = 0; m < 2; ++m) {
          const double ar = sFr[(8 * m + g) * LD + pc], ai = sFi[(8 * m + g) * LD + pc];
#pragma unroll
          for (int n = 0; n < 2; ++n) cmma<false>(M1r[m][n], M1i[m][n], ar, ai, br[n], bi[n]);
        }
      }
      double M2r[2][2][2], M2i[2][2][2];   // [k1 tile][k2 tile][j]
#pragma unroll
      for (int m = 0; m < 2; ++m)
#pragma unroll
        for (int n = 0; n < 2; ++n) M2r[m][n][0] = M2r[m][n][1] = M2i[m][n][0] = M2i[m][n][1] = 0.0;
#pragma unroll
      for (int kg = 0; kg < 2; ++kg)       // l1 tile of M1 = contraction chunk group
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const int pc = 8 * kg + 4 * j + q;
#pragma unroll
          for (int m = 0; m < 2; ++m) {
            const double ar = sFr[(8 * m + g) * LD + pc], ai = sFi[(8 * m + g) * LD + pc];
#pragma unroll
            for (int n = 0; n < 2; ++n)      // n = k2 tile = M1's m index
              cmma<false>(M2r[m][n], M2i[m][n], ar, ai, M1r[n][kg][j], M1i[n][kg][j]);
          }
        }
      __syncwarp();
#pragma unroll
      for (int m = 0; m < 2; ++m)
#pragma unroll
        for (int n = 0; n < 2; ++n)
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            const int idx = l0 * SL + (8 * m + g) * LD + 8 * n + 4 * j + q;   // [l0][k1][perm k2]
            sXa[idx] = M2r[m][n][j];
            sXb[idx] = M2i[m][n][j];
          }
    }
    __syncthreads();

    // ---- phase 2: per (k1, k2-half) row block: axis 0 forward, * S_T, axis 0 inverse ----
    for (int mb = warp; mb < 32; mb += NW3) {
      const int k1 = mb >> 1, k2b = 8 * (mb & 1);
      const int colA = k1 * LD + k2b + perm8(g);   // A[m = g][k = l0] = Q[l0][k1][k2b + g]
      double Zr[2][2], Zi[2][2];                     // [k0 tile][j]
#pragma unroll
      for (int n = 0; n < 2; ++n) Zr[n][0] = Zr[n][1] = Zi[n][0] = Zi[n][1] = 0.0;
#pragma unroll
      for (int kg = 0; kg < 2; ++kg)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const int l0 = 8 * kg + 2 * q + j;          // chunk order shared with B = F[l0][k0]
          const double ar = sXa[l0 * SL + colA], ai = sXb[l0 * SL + colA];
          const int pc = 8 * kg + 4 * j + q;
#pragma unroll
          for (int n = 0; n < 2; ++n) {
            const double br = sFr[(8 * n + g) * LD + pc], bi = sFi[(8 * n + g) * LD + pc];  // F symmetric
            cmma<false>(Zr[n], Zi[n], ar, ai, br, bi);
          }
        }
      // Z[m = (k1, k2b+g)][k0 = 8n + 2q + j] *= S_T[k1][k2][k0]
#pragma unroll
      for (int n = 0; n < 2; ++n) {
        const int64_t si = ((int64_t)(k1 * L + k2b + g)) * L + 8 * n + 2 * q;
        const double2 sr = __ldg(reinterpret_cast<const double2*>(a.Sre + si));
        const double2 sm = __ldg(reinterpret_cast<const double2*>(a.Sim + si));
        const double r0 = Zr[n][0] * sr.x - Zi[n][0] * sm.x, i0 = Zr[n][0] * sm.x + Zi[n][0] * sr.x;
        const double r1 = Zr[n][1] * sr.y - Zi[n][1] * sm.y, i1 = Zr[n][1] * sm.y + Zi[n][1] * sr.y;
        Zr[n][0] = r0; Zi[n][0] = i0; Zr[n][1] = r1; Zi[n][1] = i1;
      }
      // W[l0][m] = sum_k0 conj(F)[h + l0][k0] Z[m][k0]   (B = Z's C fragments)
      double Wr[2][2], Wi[2][2];                     // [l0 tile][j]
#pragma unroll
      for (int t = 0; t < 2; ++t) Wr[t][0] = Wr[t][1] = Wi[t][0] = Wi[t][1] = 0.0;
#pragma unroll
      for (int kg = 0; kg < 2; ++kg)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const int pc = 8 * kg + 4 * j + q;
#pragma unroll
          for (int t = 0; t < 2; ++t) {
            if (t < MT) {
              const int row = min(h + 8 * t + g, L - 1);
              cmma<true>(Wr[t], Wi[t], sFr[row * LD + pc], sFi[row * LD + pc], Zr[kg][j], Zi[kg][j]);
            }
          }
        }
      __syncwarp();   // every lane has read its Q column block before it is overwritten
#pragma unroll
      for (int t = 0; t < 2; ++t) {
        if (t < MT) {
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            const int idx = (8 * t + g) * SL + k1 * LD + k2b + 4 * j + q;   // [l0][k1][perm k2]
            sXa[idx] = Wr[t][j];
            sXb[idx] = Wi[t][j];
          }
        }
      }
    }
    __syncthreads();

    // ---- phase 3: per output slice l0 < S: inverse along axes 2 then 1, crop, store ----
    const bool has_b = 2 * pj + 1 < a.nt2;
    const int64_t oa2 = 2 * pj * S + a.bd.shift, ob2 = oa2 + S;
    for (int l0 = warp; l0 < S; l0 += NW3) {
      const int64_t c0 = o0 + h + l0;
      if (c0 >= a.bd.lim0 || c0 < a.win.w_lo || c0 >= a.win.w_hi) continue;
      double* dplane = a.dst + (c0 - a.win.g0) * a.n1 * a.n2;
      const double* wa = sXa + l0 * SL;
      const double* wb = sXb + l0 * SL;
      // M5[l2][k1] = sum_k2 conj(F)[h + l2][k2] W[l0][k1][k2]
      double M5r[2][2][2], M5i[2][2][2];   // [l2 tile][k1 tile][j]
#pragma unroll
      for (int m = 0; m < 2; ++m)
#pragma unroll
        for (int n = 0; n < 2; ++n) M5r[m][n][0] = M5r[m][n][1] = M5i[m][n][0] = M5i[m][n][1] = 0.0;
#pragma unroll
      for (int kc = 0; kc < 4; ++kc) {
        const int pc = 4 * kc + q;
        double br[2], bi[2];
#pragma unroll
        for (int n = 0; n < 2; ++n) { br[n] = wa[(8 * n + g) * LD + pc]; bi[n] = wb[(8 * n + g) * LD + pc]; }
#pragma unroll
        for (int m = 0; m < 2; ++m) {
          if (m < MT) {
            const int row = min(h + 8 * m + g, L - 1);
            const double ar = sFr[row * LD + pc], ai = sFi[row * LD + pc];
#pragma unroll
            for (int n = 0; n < 2; ++n) cmma<true>(M5r[m][n], M5i[m][n], ar, ai, br[n], bi[n]);
          }
        }
      }
      // Y[l1][l2] = sum_k1 conj(F)[h + l1][k1] M5[l2][k1]
      double Yr[2][2][2], Yi[2][2][2];     // [l1 tile][l2 tile][j]
#pragma unroll
      for (int m = 0; m < 2; ++m)
#pragma unroll
        for (int n = 0; n < 2; ++n) Yr[m][n][0] = Yr[m][n][1] = Yi[m][n][0] = Yi[m][n][1] = 0.0;
#pragma unroll
      for (int kg = 0; kg < 2; ++kg)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const int pc = 8 * kg + 4 * j + q;
#pragma unroll
          for (int m = 0; m < 2; ++m) {
            if (m < MT) {
              const int row = min(h + 8 * m + g, L - 1);
              const double ar = sFr[row * LD + pc], ai = sFi[row * LD + pc];
#pragma unroll
              for (int n = 0; n < 2; ++n)
                if (n < MT) cmma<true>(Yr[m][n], Yi[m][n], ar, ai, M5r[n][kg][j], M5i[n][kg][j]);
            }
          }
        }
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        if (m >= MT) continue;
        const int l1 = 8 * m + g;
#pragma unroll
        for (int n = 0; n < 2; ++n) {
          if (n >= MT) continue;
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            const int l2 = 8 * n + 2 * q + j;
            const int64_t c1 = o1 + h + l1;
            if (l1 < S && l2 < S && c1 < a.bd.lim1) {
              int64_t c2 = oa2 + h + l2;
              if (c2 < a.bd.lim2) dplane[c1 * a.n2 + c2] = Yr[m][n][j];
              c2 = ob2 + h + l2;
              if (has_b && c2 < a.bd.lim2) dplane[c1 * a.n2 + c2] = Yi[m][n][j];
            }
          }
        }
      }
    }
  }
}

}  // namespace

size_t fused3d_smem() { return (size_t)(2 * L * LD + 2 * L * SL) * sizeof(double); }

cudaError_t fused3d_configure(int* max_blocks) {
  const size_t smem = fused3d_smem();
  cudaError_t e = cudaFuncSetAttribute(fft3d_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(fft3d_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft3d_kernel<false>, NW3 * 32, smem);
}

cudaError_t launch_fused3d(const Fft3dArgs& a, int grid, cudaStream_t s) {
  if (a.bd.wrap)
    fft3d_kernel<true><<<grid, NW3 * 32, fused3d_smem(), s>>>(a);
  else
    fft3d_kernel<false><<<grid, NW3 * 32, fused3d_smem(), s>>>(a);
  return cudaGetLastError();
}

}  // namespace fstencil
