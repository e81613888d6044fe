// Fused 2D FFT-stencil tile kernel with FACTORED DFT GEMMs: 64 = 8 x 8 per axis (sm_100a).
//
// The same fused pass as kernel_fft2d.cu (Algorithm 1, Double-layer
// Filling Eq. 9, temporal fusion Eq. 10, Stitching Eq. 7), but each length-64 axis DFT is
// factored the way §3.2.1 factors the 1D transform (L208-L218: reshape a length-N DFT into
// a 2D one so the tensor cores see dense 8x8 matrices), here by Cooley-Tukey:
//     x[8 la + lb] --(DFT8 over la)--> * w64^(ka lb) --(DFT8 over lb)--> X[ka + 8 kb]
// so every GEMM is a dense DFT-8 (8x8, K = 8 = two DMMA.8x8x4 k-steps) and the work per
// element and axis drops from 8L = 512 to 2 x 64 (+ 6 for the twiddle) flops.  F8 and the
// per-thread twiddles live in registers for the whole launch (Squeezing Registers, L274).
//
// Each 64-element line (row or column of the tile) is one 8x8 complex matrix held by one
// warp in m8n8k4 fragments.  Chaining without shared memory (Swizzling Fragments L266-L272)
// uses two register routes, both contracting the columns of the current C fragment:
//   B-route  C' = F8 . C^T     (C's fragment is the B fragment of C^T)  -> rows from F8
//   A-route  C' = C . F8^T     (C's fragment is the A fragment of C)    -> rows stay C's
// Per tile pair (Re = tile 2j, Im = tile 2j+1 of one outer tile row):
//   phase 1  rows l0 (64):     DFT8 over la1, twiddle, A-route DFT8 over lb1   -> row of Q
//   phase 2  columns k1 (64):  DFT8 over la0, twiddle, A-route DFT8 over lb0,
//                              * S_T (Eq. 10), B-route iDFT8 over kb0, twiddle*,
//                              A-route iDFT8 over ka0                          -> column of W
//   phase 3  output rows (S):  iDFT8 over kb1, twiddle*, B-route iDFT8 over ka1 -> store
// Phases 1 and 2 overwrite exactly the shared-memory words each thread read (in place);
// the two CTA barriers are the transpositions of ownership a 2D transform needs.
// Shared layout: plane[r][c] at r*64 + (c ^ 4(((c>>4) ^ (r>>4)) & 3) ^ (r & 3)) (XOR swizzle):
// both the row pattern (c = 16q + 8j + g) and the column pattern (r = 16q + 8j + g) are
// bank-conflict free per half-warp.
#include "ct_line.cuh"
#include "kernels.cuh"
#include "tma.cuh"

namespace fstencil {
namespace {

using namespace ct;

constexpr int PLANE = L * L;

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

// TMA = true: each tile arrives by one 64 x 64 TMA box (OOB -> 0) in a dense row-major
// layout; phase 1 reads its rows there (4-way bank conflicts on that pass only) and, the
// XOR swizzle being a permutation within a row, rewrites each row in place swizzled.
template <int NW, int NL, bool TMA, bool WRAP = false>   // WRAP: periodic (cp.async path only)
// FFTSTENCIL_CT2D_REGS (80): three CTAs per SM (72 would admit a band CTA beside them, but
// costs 1.5% in spills: profiles/r01_cmul3.jsonl)
#ifndef FFTSTENCIL_CT2D_REGS
#define FFTSTENCIL_CT2D_REGS 80
#endif
__global__ void __maxnreg__(NL > 2 ? 128 : (NW == 16 ? 40 : FFTSTENCIL_CT2D_REGS))
    fft2d_ct_kernel(const Fft2dArgs a, const __grid_constant__ CUtensorMap tm) {
  extern __shared__ __align__(128) double smem[];
  double* sR = smem;            // plane 0: tile 2j (Re), then Q/W real parts
  double* sI = smem + PLANE;    // plane 1: tile 2j+1 (Im), then Q/W imaginary parts
  __shared__ __align__(8) uint64_t bar;
  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31, g = lane >> 2, q = lane & 3;
  if (TMA && tid == 0) tma::mbar_init(&bar, 1);
  uint32_t parity = 0;

  // register-resident F8 fragments (row g, logical column 2q+j) and twiddles w64^(g (2q+j))
  double fr[2], fi[2], tr[2], ti[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const int c = 2 * q + j;
    fr[j] = a.Fre[g * 8 + c];
    fi[j] = a.Fim[g * 8 + c];
    tr[j] = a.Fre[64 + g * 8 + c];
    ti[j] = a.Fim[64 + g * 8 + c];
  }
  const int S = a.S, h = a.h;
  int cl[2];                     // the thread's line positions 16q + 8j + g
#pragma unroll
  for (int j = 0; j < 2; ++j) cl[j] = 16 * q + 8 * j + g;

  for (int64_t p = a.win.p_begin + blockIdx.x; p < a.win.p_end; p += gridDim.x) {
    const int64_t t0 = p / a.npr, pj = p - t0 * a.npr;
    const int64_t o0 = t0 * S + a.bd.shift, oa1 = 2 * pj * S + a.bd.shift, ob1 = oa1 + S;
    const bool has_b = 2 * pj + 1 < a.nt1;
    if (TMA) tma::fence_proxy_async();
    __syncthreads();   // previous pair's phase 3 reads are done
    if (TMA) {
      // ---- load the halo'd pair: two 64 x 64 TMA boxes (OOB rows/columns -> 0) ----
      if (tid == 0) {
        tma::mbar_expect_tx(&bar, (has_b ? 2u : 1u) * L * L * 8u);
        const int y = (int)(o0 - a.win.g0);
        tma::load_2d(sR, &tm, (int)oa1, y, &bar);
        if (has_b) tma::load_2d(sI, &tm, (int)ob1, y, &bar);
      }
      if (!has_b)
        for (int e = tid; e < L * L; e += NW * 32) sI[e] = 0.0;
      tma::mbar_wait(&bar, parity);
      parity ^= 1;
      __syncthreads();
      // ---- phase 1 from the dense staging rows; the swizzled layout permutes words within a
      // row only, so each warp rewrites its own rows in place ----
      for (int l0b = warp * NL; l0b < L; l0b += NW * NL) {
        double br[NL][2], bi[NL][2], c1r[NL][2], c1i[NL][2], c2r[NL][2], c2i[NL][2];
#pragma unroll
        for (int u = 0; u < NL; ++u)
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            br[u][j] = sR[(l0b + u) * L + cl[j]];
            bi[u][j] = sI[(l0b + u) * L + cl[j]];
          }
        broute_n<false, NL>(c1r, c1i, fr, fi, br, bi);
        twiddle_n<false, NL>(c1r, c1i, tr, ti);
        aroute_n<false, NL>(c2r, c2i, c1r, c1i, fr, fi);
        __syncwarp();
#pragma unroll
        for (int u = 0; u < NL; ++u)
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            sR[sw(l0b + u, cl[j])] = c2r[u][j];
            sI[sw(l0b + u, cl[j])] = c2i[u][j];
          }
      }
    } else {
    // ---- load the halo'd pair (cp.async, OOB = 0) ----
    for (int e = tid; e < 2 * L * L; e += NW * 32) {
      const int t = e >> 12, r = (e >> 6) & 63, c = e & 63;
      int64_t gr = o0 + r, gc = (t ? ob1 : oa1) + c;
      if (WRAP) { gr = wrap_index(gr, a.n0); gc = wrap_index(gc, a.n1); }
      const int64_t lr = gr - a.win.g0;
      const bool valid = (t == 0 || has_b) && gr < a.n0 && lr >= 0 && lr < a.win.gn && gc >= 0 && gc < a.n1;
      cp_async8((t ? sI : sR) + sw(r, c), valid ? a.src + lr * a.n1 + gc : a.src, valid);
    }
    asm volatile("cp.async.commit_group;\n" ::);
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    __syncthreads();

    // ---- phase 1: forward DFT along axis 1, every row (NL rows per warp step) ----
    for (int l0b = warp * NL; l0b < L; l0b += NW * NL) {
      double br[NL][2], bi[NL][2], c1r[NL][2], c1i[NL][2], c2r[NL][2], c2i[NL][2];
#pragma unroll
      for (int u = 0; u < NL; ++u)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          br[u][j] = sR[sw(l0b + u, cl[j])];
          bi[u][j] = sI[sw(l0b + u, cl[j])];
        }
      broute_n<false, NL>(c1r, c1i, fr, fi, br, bi);     // [ka1][lb1]
      twiddle_n<false, NL>(c1r, c1i, tr, ti);
      aroute_n<false, NL>(c2r, c2i, c1r, c1i, fr, fi);   // [ka1][kb1]: k1 = g + 8(2q+j) = cl[j]
#pragma unroll
      for (int u = 0; u < NL; ++u)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          sR[sw(l0b + u, cl[j])] = c2r[u][j];
          sI[sw(l0b + u, cl[j])] = c2i[u][j];
        }
    }
    }   // !TMA
    __syncthreads();

    // ---- phase 2: axis 0 forward, * S_T, axis 0 inverse, every column ----
    for (int k1b = warp * NL; k1b < L; k1b += NW * NL) {
      double br[NL][2], bi[NL][2], c1r[NL][2], c1i[NL][2], c2r[NL][2], c2i[NL][2];
      double s_r[NL][2], s_i[NL][2];
#pragma unroll
      for (int u = 0; u < NL; ++u) {
        const double2 sr = __ldg(reinterpret_cast<const double2*>(a.Sre + (k1b + u) * 64 + g * 8 + 2 * q));
        const double2 si = __ldg(reinterpret_cast<const double2*>(a.Sim + (k1b + u) * 64 + g * 8 + 2 * q));
        s_r[u][0] = sr.x; s_r[u][1] = sr.y; s_i[u][0] = si.x; s_i[u][1] = si.y;
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          br[u][j] = sR[sw(cl[j], k1b + u)];
          bi[u][j] = sI[sw(cl[j], k1b + u)];
        }
      }
      broute_n<false, NL>(c1r, c1i, fr, fi, br, bi);     // [ka0][lb0]
      twiddle_n<false, NL>(c1r, c1i, tr, ti);
      aroute_n<false, NL>(c2r, c2i, c1r, c1i, fr, fi);   // [ka0][kb0]: k0 = cl[j]
#pragma unroll
      for (int u = 0; u < NL; ++u)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const double r = c2r[u][j] * s_r[u][j] - c2i[u][j] * s_i[u][j];
          const double i = c2r[u][j] * s_i[u][j] + c2i[u][j] * s_r[u][j];
          c2r[u][j] = r;
          c2i[u][j] = i;
        }
      broute_n<true, NL>(c1r, c1i, fr, fi, c2r, c2i);    // [lb0][ka0]
      twiddle_n<true, NL>(c1r, c1i, tr, ti);
      aroute_n<true, NL>(c2r, c2i, c1r, c1i, fr, fi);    // [lb0][la0]: l0 = cl[j]
#pragma unroll
      for (int u = 0; u < NL; ++u)
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          sR[sw(cl[j], k1b + u)] = c2r[u][j];
          sI[sw(cl[j], k1b + u)] = c2i[u][j];
        }
    }
    __syncthreads();

    // ---- phase 3: inverse DFT along axis 1 on the S output rows, store the window ----
    for (int ib = warp * NL; ib < S; ib += NW * NL) {
      double br[NL][2], bi[NL][2], c1r[NL][2], c1i[NL][2], c2r[NL][2], c2i[NL][2];
#pragma unroll
      for (int u = 0; u < NL; ++u) {
        const int l0 = h + min(ib + u, S - 1);       // a clamped duplicate is computed, not stored
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          br[u][j] = sR[sw(l0, cl[j])];
          bi[u][j] = sI[sw(l0, cl[j])];
        }
      }
      broute_n<true, NL>(c1r, c1i, fr, fi, br, bi);      // [lb1][ka1]
      twiddle_n<true, NL>(c1r, c1i, tr, ti);
      broute_n<true, NL>(c2r, c2i, fr, fi, c1r, c1i);    // [la1][lb1]: l1 = 8g + 2q + j
#pragma unroll
      for (int u = 0; u < NL; ++u) {
        const int i = ib + u;
        const int64_t c0 = o0 + h + i;
        if (i >= S || c0 >= a.bd.lim0 || c0 < a.win.w_lo || c0 >= a.win.w_hi) continue;
        double* drow = a.dst + (c0 - a.win.g0) * a.n1;
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const int l1 = 8 * g + 2 * q + j;
          if (l1 >= h && l1 < h + S) {
            int64_t c1 = oa1 + l1;
            if (c1 < a.bd.lim1) drow[c1] = c2r[u][j];
            c1 = ob1 + l1;
            if (has_b && c1 < a.bd.lim1) drow[c1] = c2i[u][j];
          }
        }
      }
    }
  }
}

template <int NW, int NL, bool TMA>
cudaError_t configure_nw(int* max_blocks) {
  const size_t smem = fused2d_ct_smem();
  cudaError_t e =
      cudaFuncSetAttribute(fft2d_ct_kernel<NW, NL, TMA>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft2d_ct_kernel<NW, NL, TMA>, NW * 32, smem);
}

}  // namespace

size_t fused2d_ct_smem() { return (size_t)2 * PLANE * sizeof(double); }

// cfg = 10 * NW + NL: 81, 82, 84, 161, 162 (TMA instantiations for 81, 82 and 84)
cudaError_t fused2d_ct_configure(int cfg, int* max_blocks) {
  switch (cfg) {
    case 81: {
      cudaError_t e = cudaFuncSetAttribute(fft2d_ct_kernel<8, 1, false, true>,
                                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fused2d_ct_smem());
      if (e == cudaSuccess) e = configure_nw<8, 1, true>(max_blocks);
      return e != cudaSuccess ? e : configure_nw<8, 1, false>(max_blocks);
    }
    case 82: {
      cudaError_t e = configure_nw<8, 2, true>(max_blocks);
      return e != cudaSuccess ? e : configure_nw<8, 2, false>(max_blocks);
    }
    case 84: {
      cudaError_t e = configure_nw<8, 4, true>(max_blocks);
      return e != cudaSuccess ? e : configure_nw<8, 4, false>(max_blocks);
    }
    case 161: return configure_nw<16, 1, false>(max_blocks);
    case 162: return configure_nw<16, 2, false>(max_blocks);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_fused2d_ct(int cfg, const Fft2dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s) {
  const size_t smem = fused2d_ct_smem();
  static const CUtensorMap none = {};
  const CUtensorMap& m = tm ? *tm : none;
  if (a.bd.wrap) {   // periodic: cp.async loads with wrap-around (single instantiation)
    fft2d_ct_kernel<8, 1, false, true><<<grid, 256, smem, s>>>(a, m);
  } else if (tm && cfg == 81) {
    fft2d_ct_kernel<8, 1, true><<<grid, 256, smem, s>>>(a, m);
  } else if (tm && cfg == 82) {
    fft2d_ct_kernel<8, 2, true><<<grid, 256, smem, s>>>(a, m);
  } else if (tm && cfg == 84) {
    fft2d_ct_kernel<8, 4, true><<<grid, 256, smem, s>>>(a, m);
  } else {
    switch (cfg) {
      case 81: fft2d_ct_kernel<8, 1, false><<<grid, 256, smem, s>>>(a, m); break;
      case 82: fft2d_ct_kernel<8, 2, false><<<grid, 256, smem, s>>>(a, m); break;
      case 84: fft2d_ct_kernel<8, 4, false><<<grid, 256, smem, s>>>(a, m); break;
      case 161: fft2d_ct_kernel<16, 1, false><<<grid, 512, smem, s>>>(a, m); break;
      case 162: fft2d_ct_kernel<16, 2, false><<<grid, 512, smem, s>>>(a, m); break;
      default: return cudaErrorInvalidValue;
    }
  }
  return cudaGetLastError();
}

}  // namespace fstencil
