// Fused 2D FFT-stencil tile kernel (sm_100a, FP64 tensor cores via DMMA.8x8x4).
//
// One CTA owns a pair of overlap-save tiles at a time (persistent grid-stride loop) and
// runs the whole of PAPER.md Algorithm 1 (L252-L258) on it in shared memory/registers:
//   load    tiles 2p and 2p+1 (L x L, halo h = rT, zero outside the grid) become the
//           real and imaginary planes of one complex tile  (Double-layer Filling, §3.2.3,
//           Eq. 9; Splitting Eq. 3)
//   M1      P^T = F . X^T        forward DFT along axis 1  (Alg. 1 line 1, right factor)
//   M2      Q   = F . P          forward DFT along axis 0  (Alg. 1 line 1, left factor)
//   mult    Q  *= S_T            powered spectrum, 1/L^2 folded in (Alg. 1 line 2; Eq. 10)
//   M3      R   = G . Q^T        inverse DFT along axis 1, crop-aware: G = conj(F)[h:h+S]
//   M4      Y   = G . R^T        inverse DFT along axis 0, crop-aware (Alg. 1 lines 3-4;
//                                 iF recomputed from F by conjugation, L258/L278)
//   store   Re(Y) -> tile 2p, Im(Y) -> tile 2p+1, valid S x S window only (Stitching,
//           Eq. 7; reading Q4)
// Warp w owns the 8-wide stripe w of the transform: in M1/M2 a frequency stripe of axis 1,
// in M3/M4 an output stripe of axis 1.  M1->M2 and M3->M4 chain C fragments straight into
// B fragments (Swizzling Fragments, L266-L272); the only shared-memory round trip is the
// transposition of ownership between the forward and inverse halves.
//
// Variants (template V, selected by the plan; FFTSTENCIL_VARIANT overrides for ablations):
//   V = 0  single pair buffer, synchronous loads, F in shared memory (first version)
//   V = 1  double-buffered pair: the next pair is fetched with cp.async (zero-fill OOB)
//          while the inverse half (M3/M4) of the current pair runs; F in shared memory
//   V = 2  as V = 1 but F is read through L1 (column-permuted copy in HBM), so a CTA's
//          shared memory is just the two pair buffers (more CTAs per SM)
// Stages (template ST, the UNFUSED ablation of NEXT-3 / PAPER.md Fig. 2 left and Fig. 7):
//   ST = 0  the fused pass above
//   ST = 1  load + forward DFT only; the spectrum goes to HBM (a.spec, [pair][re|im][k0][k1])
//   ST = 2  reads the spectrum back from HBM, inverse DFT + crop + store only
// with spec_mul_kernel in between: three kernels and two spectrum round trips per pass,
// the "standard FFT stencil" structure Kernel Tailoring removes.
#include <algorithm>

#include "device_common.cuh"

#pragma nv_diag_suppress 128   // ST = 1 leaves the inverse half unreachable by design
#include "kernels.cuh"

namespace fstencil {
namespace {

using dev::dmma;
using dev::perm8;

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// Pair p = tiles (t0, 2j) and (t0, 2j+1) with t0 = p / npr, j = p % npr (kernels.cuh).
template <int L, bool ASYNC, bool WRAP>
__device__ __forceinline__ void load_pair(double* sXa, double* sXb, const Fft2dArgs& a, int64_t p, int tid) {
  constexpr int LD = L + 4, NTHR = L * 4;
  const int64_t t0 = p / a.npr, j = p - t0 * a.npr;
  const int64_t o0 = t0 * a.S + a.bd.shift;   // global row of tile row 0
#pragma unroll
  for (int t = 0; t < 2; ++t) {
    const int64_t t1 = 2 * j + t;
    double* sX = t ? sXb : sXa;
    const bool have = t1 < a.nt1;
    const int64_t o1 = t1 * a.S + a.bd.shift;
    for (int e = tid; e < L * L; e += NTHR) {
      const int r = e / L, c = e - r * L;
      int64_t gr = o0 + r, gc = o1 + c;
      if (WRAP) { gr = wrap_index(gr, a.n0); gc = wrap_index(gc, a.n1); }
      const int64_t lr = gr - a.win.g0;
      const bool valid = have && gr < a.n0 && lr >= 0 && lr < a.win.gn && gc < a.n1;   // gc >= 0 always
      double* dst = sX + r * LD + perm8(c);
      if (ASYNC) {
        cp_async8(dst, valid ? a.src + lr * a.n1 + gc : a.src, valid);
      } else {
        *dst = valid ? __ldg(a.src + lr * a.n1 + gc) : 0.0;
      }
    }
  }
}

template <bool GLOBAL>
__device__ __forceinline__ double ldF(const double* p) {
  if (GLOBAL) return __ldg(p);
  return *p;
}

// WRAP: periodic boundary (NEXT-2), a separate instantiation so the fixed-ring kernel carries
// no wrap-around arithmetic in its load loop.
template <int L, int V, int ST = 0, bool WRAP = false>
__global__ void __launch_bounds__(L * 4) fft2d_kernel(const Fft2dArgs a) {
  constexpr int NT = L / 8;      // 8x8 tiles per side == warps
  constexpr int LD = L + 4;      // padded row stride (doubles): 8-bank shift per row
  constexpr int NTHR = L * 4;
  constexpr bool FSM = V != 2;   // F in shared memory
  constexpr bool DB = V != 0;    // double-buffered pair with cp.async prefetch
  constexpr int FLD = FSM ? LD : L;
  extern __shared__ __align__(16) double smem[];
  double* sbuf = smem + (FSM ? 2 * L * LD : 0);
  const double* Fr;
  const double* Fi;
  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31, g = lane >> 2, q = lane & 3;
  if (FSM) {
    double* sFr = smem;
    double* sFi = sFr + L * LD;
    for (int e = tid; e < L * L; e += NTHR) {
      const int r = e / L, c = e - r * L;     // a.Fre is already column-permuted
      sFr[r * LD + c] = a.Fre[e];
      sFi[r * LD + c] = a.Fim[e];
    }
    Fr = sFr;
    Fi = sFi;
  } else {
    Fr = a.Fre;
    Fi = a.Fim;
  }
  const int S = a.S, h = a.h;
  const int MT = (S + 7) >> 3;   // output 8-tiles per axis (S padded to 8)
  int cur = 0;

  if (DB && a.win.p_begin + blockIdx.x < a.win.p_end) {
    load_pair<L, true, WRAP>(sbuf, sbuf + L * LD, a, a.win.p_begin + blockIdx.x, tid);
    cp_async_commit();
    cp_async_wait_all();
  }
  for (int64_t p = a.win.p_begin + blockIdx.x; p < a.win.p_end; p += gridDim.x) {
    double* sXa = sbuf + cur * 2 * L * LD;   // tile 2p (real part) ... later Q' real part
    double* sXb = sXa + L * LD;              // tile 2p+1 (imag part) ... later Q' imag part
    if (ST == 2) {
      // ---- unfused inverse stage: the multiplied spectrum comes back from HBM ----
      __syncthreads();
      const double* sp = a.spec + (size_t)p * 2 * L * L;
      for (int e = tid; e < L * L; e += NTHR) {
        const int k0 = e / L, k1 = e - k0 * L;
        sXa[k0 * LD + perm8(k1)] = sp[e];
        sXb[k0 * LD + perm8(k1)] = sp[L * L + e];
      }
      __syncthreads();
    } else {
    if (!DB) {
      __syncthreads();
      load_pair<L, false, WRAP>(sXa, sXb, a, p, tid);
    }
    __syncthreads();

    // ---- M1: P^T[k1 stripe][l0] = sum_l1 F[k1][l1] X[l0][l1]  (B from shared) ----
    double Pr[NT][2], Pi[NT][2];
#pragma unroll
    for (int i = 0; i < NT; ++i) Pr[i][0] = Pr[i][1] = Pi[i][0] = Pi[i][1] = 0.0;
    {
      const double* fr = Fr + (8 * warp + g) * FLD + q;
      const double* fi = Fi + (8 * warp + g) * FLD + q;
#pragma unroll
      for (int kc = 0; kc < L / 4; ++kc) {
        const int pc = 4 * kc;
        const double ar = ldF<!FSM>(fr + pc), ai = ldF<!FSM>(fi + pc), nai = -ai;
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
          const double br = sXa[(8 * nt + g) * LD + q + pc];
          const double bi = sXb[(8 * nt + g) * LD + q + pc];
          dmma(Pr[nt], ar, br);
          dmma(Pr[nt], nai, bi);
          dmma(Pi[nt], ar, bi);
          dmma(Pi[nt], ai, br);
        }
      }
    }
    // ---- M2: Q[k0][k1 stripe] = sum_l0 F[k0][l0] P[l0][k1]  (B = M1's C fragments) ----
    double Qr[NT][2], Qi[NT][2];
#pragma unroll
    for (int i = 0; i < NT; ++i) Qr[i][0] = Qr[i][1] = Qi[i][0] = Qi[i][1] = 0.0;
#pragma unroll
    for (int kg = 0; kg < NT; ++kg) {
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const double br = Pr[kg][j], bi = Pi[kg][j];
        const int pc = 8 * kg + 4 * j + q;
#pragma unroll
        for (int mt = 0; mt < NT; ++mt) {
          const double ar = ldF<!FSM>(Fr + (8 * mt + g) * FLD + pc);
          const double ai = ldF<!FSM>(Fi + (8 * mt + g) * FLD + pc);
          dmma(Qr[mt], ar, br);
          dmma(Qr[mt], -ai, bi);
          dmma(Qi[mt], ar, bi);
          dmma(Qi[mt], ai, br);
        }
      }
    }
    if (ST == 1) {
      // ---- unfused forward stage: the spectrum goes to HBM ----
      double* sp = a.spec + (size_t)p * 2 * L * L;
#pragma unroll
      for (int mt = 0; mt < NT; ++mt) {
        const int k0 = 8 * mt + g, k1 = 8 * warp + 2 * q;
        *reinterpret_cast<double2*>(sp + k0 * L + k1) = make_double2(Qr[mt][0], Qr[mt][1]);
        *reinterpret_cast<double2*>(sp + L * L + k0 * L + k1) = make_double2(Qi[mt][0], Qi[mt][1]);
      }
      continue;
    }
    // ---- pointwise multiply by the powered spectrum (Eq. 10) in the C fragments ----
#pragma unroll
    for (int mt = 0; mt < NT; ++mt) {
      const int k0 = 8 * mt + g, k1 = 8 * warp + 2 * q;
      const double2 sr = __ldg(reinterpret_cast<const double2*>(a.Sre + k0 * L + k1));
      const double2 si = __ldg(reinterpret_cast<const double2*>(a.Sim + k0 * L + k1));
      const double r0 = Qr[mt][0] * sr.x - Qi[mt][0] * si.x;
      const double i0 = Qr[mt][0] * si.x + Qi[mt][0] * sr.x;
      const double r1 = Qr[mt][1] * sr.y - Qi[mt][1] * si.y;
      const double i1 = Qr[mt][1] * si.y + Qi[mt][1] * sr.y;
      Qr[mt][0] = r0; Qi[mt][0] = i0; Qr[mt][1] = r1; Qi[mt][1] = i1;
    }
    __syncthreads();   // every warp is past M1: the tile planes may be overwritten
#pragma unroll
    for (int mt = 0; mt < NT; ++mt)
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int idx = (8 * mt + g) * LD + 8 * warp + 4 * j + q;   // perm8 of k1
        sXa[idx] = Qr[mt][j];
        sXb[idx] = Qi[mt][j];
      }
    __syncthreads();
    }   // ST != 2
    // ---- prefetch the next pair into the other buffer while the inverse half runs ----
    if (DB) {
      const int64_t pn = p + gridDim.x;
      if (pn < a.win.p_end) {
        double* nb = sbuf + (cur ^ 1) * 2 * L * LD;
        load_pair<L, true, WRAP>(nb, nb + L * LD, a, pn, tid);
      }
      cp_async_commit();
    }

    if (warp < MT) {
      // ---- M3: R[l1 stripe][k0] = sum_k1 conj(F)[h+l1][k1] Q'[k0][k1] (B from shared) ----
      double Rr[NT][2], Ri[NT][2];
#pragma unroll
      for (int i = 0; i < NT; ++i) Rr[i][0] = Rr[i][1] = Ri[i][0] = Ri[i][1] = 0.0;
      {
        const int arow = min(h + 8 * warp + g, L - 1);   // rows past S are padding
        const double* fr = Fr + arow * FLD + q;
        const double* fi = Fi + arow * FLD + q;
#pragma unroll
        for (int kc = 0; kc < L / 4; ++kc) {
          const int pc = 4 * kc;
          const double ar = ldF<!FSM>(fr + pc), ai = ldF<!FSM>(fi + pc), nai = -ai;
#pragma unroll
          for (int nt = 0; nt < NT; ++nt) {
            const double br = sXa[(8 * nt + g) * LD + q + pc];
            const double bi = sXb[(8 * nt + g) * LD + q + pc];
            dmma(Rr[nt], ar, br);     // conj(F) . Q'^T
            dmma(Rr[nt], ai, bi);
            dmma(Ri[nt], ar, bi);
            dmma(Ri[nt], nai, br);
          }
        }
      }
      // ---- M4: Y[l0][l1 stripe] = sum_k0 conj(F)[h+l0][k0] R[l1][k0] (B = M3's C) ----
      double Yr[NT][2], Yi[NT][2];
#pragma unroll
      for (int i = 0; i < NT; ++i) Yr[i][0] = Yr[i][1] = Yi[i][0] = Yi[i][1] = 0.0;
#pragma unroll
      for (int kg = 0; kg < NT; ++kg) {
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const double br = Rr[kg][j], bi = Ri[kg][j];
          const int pc = 8 * kg + 4 * j + q;
#pragma unroll
          for (int mt = 0; mt < NT; ++mt) {
            if (mt < MT) {
              const int arow = min(h + 8 * mt + g, L - 1);
              const double ar = ldF<!FSM>(Fr + arow * FLD + pc);
              const double ai = ldF<!FSM>(Fi + arow * FLD + pc);
              dmma(Yr[mt], ar, br);
              dmma(Yr[mt], ai, bi);
              dmma(Yi[mt], ar, bi);
              dmma(Yi[mt], -ai, br);
            }
          }
        }
      }
      // ---- stitch: the S x S valid window of each tile, exact region and window only ----
      const int64_t t0 = p / a.npr, pj = p - t0 * a.npr;
      const int64_t a1 = 2 * pj, b1 = a1 + 1;
      const bool has_b = b1 < a.nt1;
#pragma unroll
      for (int mt = 0; mt < NT; ++mt) {
        if (mt < MT) {
          const int l0 = 8 * mt + g;
          const int64_t c0 = t0 * S + a.bd.shift + h + l0;
          const bool row_ok = l0 < S && c0 < a.bd.lim0 && c0 >= a.win.w_lo && c0 < a.win.w_hi;
          double* drow = a.dst + (c0 - a.win.g0) * a.n1;
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            const int l1 = 8 * warp + 2 * q + j;
            if (row_ok && l1 < S) {
              int64_t c1 = a1 * S + a.bd.shift + h + l1;
              if (c1 < a.bd.lim1) drow[c1] = Yr[mt][j];
              c1 = b1 * S + a.bd.shift + h + l1;
              if (has_b && c1 < a.bd.lim1) drow[c1] = Yi[mt][j];
            }
          }
        }
      }
    }
    if (DB) {
      cp_async_wait_all();
      __syncthreads();   // next pair landed; this pair's Q' reads are done
      cur ^= 1;
    }
  }
}

__global__ void spec_mul_kernel(double* spec, int64_t npairs, int vol, const double* __restrict__ Sre,
                                const double* __restrict__ Sim) {
  const int64_t total = npairs * vol;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t pr = i / vol;
    const int k = (int)(i - pr * vol);
    double* re = spec + pr * 2 * vol + k;
    double* im = re + vol;
    const double a = *re, b = *im, sr = __ldg(Sre + k), si = __ldg(Sim + k);
    *re = a * sr - b * si;
    *im = a * si + b * sr;
  }
}

template <int L, int V>
cudaError_t configure_LV(int* max_blocks) {
  const size_t smem = fused2d_smem(L, V);
  cudaError_t e = cudaFuncSetAttribute(fft2d_kernel<L, V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft2d_kernel<L, V>, L * 4, smem);
}

template <int L>
cudaError_t configure_L(int V, int* max_blocks) {
  {   // the unfused stages and the periodic instantiation share the V = 0 footprint
    const size_t smem = fused2d_smem(L, 0);
    cudaError_t e = cudaFuncSetAttribute(fft2d_kernel<L, 0, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(fft2d_kernel<L, 0, 0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(fft2d_kernel<L, 0, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
  }
  switch (V) {
    case 0: return configure_LV<L, 0>(max_blocks);
    case 1: return configure_LV<L, 1>(max_blocks);
    case 2: return configure_LV<L, 2>(max_blocks);
    default: return cudaErrorInvalidValue;
  }
}

template <int L>
void launch_L(int V, const Fft2dArgs& a, int grid, cudaStream_t s) {
  const size_t smem = fused2d_smem(L, V);
  if (a.bd.wrap) {   // periodic plans run the V = 0 structure
    fft2d_kernel<L, 0, 0, true><<<grid, L * 4, fused2d_smem(L, 0), s>>>(a);
    return;
  }
  switch (V) {
    case 0: fft2d_kernel<L, 0><<<grid, L * 4, smem, s>>>(a); break;
    case 1: fft2d_kernel<L, 1><<<grid, L * 4, smem, s>>>(a); break;
    default: fft2d_kernel<L, 2><<<grid, L * 4, smem, s>>>(a); break;
  }
}

}  // namespace

int fused2d_threads(int L) { return L * 4; }

size_t fused2d_smem(int L, int V) {
  const size_t plane = (size_t)L * (L + 4) * sizeof(double);
  const size_t f = V == 2 ? 0 : 2 * plane;
  const size_t bufs = V == 0 ? 2 * plane : 4 * plane;
  return f + bufs;
}

cudaError_t fused2d_configure(int L, int V, int* max_blocks) {
  switch (L) {
    case 16: return configure_L<16>(V, max_blocks);
    case 24: return configure_L<24>(V, max_blocks);
    case 32: return configure_L<32>(V, max_blocks);
    case 40: return configure_L<40>(V, max_blocks);
    case 48: return configure_L<48>(V, max_blocks);
    case 56: return configure_L<56>(V, max_blocks);
    case 64: return configure_L<64>(V, max_blocks);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_unfused2d(int L, int stage, const Fft2dArgs& a, int grid, cudaStream_t s) {
  const size_t smem = fused2d_smem(L, 0);
  switch (L * 10 + stage) {
#define FS_CASE(LL)                                                                  \
  case LL * 10 + 1: fft2d_kernel<LL, 0, 1><<<grid, LL * 4, smem, s>>>(a); break; \
  case LL * 10 + 2: fft2d_kernel<LL, 0, 2><<<grid, LL * 4, smem, s>>>(a); break;
    FS_CASE(16) FS_CASE(24) FS_CASE(32) FS_CASE(40) FS_CASE(48) FS_CASE(56) FS_CASE(64)
#undef FS_CASE
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_spec_mul(double* spec, int64_t npairs, int L, const double* Sre, const double* Sim,
                            cudaStream_t s) {
  const int64_t total = npairs * L * L;
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 16);
  spec_mul_kernel<<<grid, 256, 0, s>>>(spec, npairs, L * L, Sre, Sim);
  return cudaGetLastError();
}

cudaError_t launch_fused2d(int L, int V, const Fft2dArgs& a, int grid, cudaStream_t s) {
  if (V < 0 || V > 2) return cudaErrorInvalidValue;
  switch (L) {
    case 16: launch_L<16>(V, a, grid, s); break;
    case 24: launch_L<24>(V, a, grid, s); break;
    case 32: launch_L<32>(V, a, grid, s); break;
    case 40: launch_L<40>(V, a, grid, s); break;
    case 48: launch_L<48>(V, a, grid, s); break;
    case 56: launch_L<56>(V, a, grid, s); break;
    case 64: launch_L<64>(V, a, grid, s); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace fstencil
