// Fused 2D FFT-stencil tile kernel with register-resident radix-8 FFTs on the FP64 ALU
// (sm_100a): the default 2D engine.
//
// Same fused pass and tile geometry as kernel_fft2d_ct.cu (Algorithm 1 L252-L258 on
// 64 x 64 overlap-save tiles, Double-layer Filling Eq. 9, temporal fusion Eq. 10, Stitching
// Eq. 7), with every length-64 axis DFT evaluated as the Cooley-Tukey 64 = 8 x 8 factorisation
// (§3.2.1's reshaping, L208-L218):
//   X[k1 + 8 k2] = sum_n2 w8^(n2 k2) w64^(n2 k1) sum_n1 w8^(n1 k1) x[8 n1 + n2]
// where each DFT-8 is a 56-instruction butterfly (fft_radix.cuh) held by one thread ("chunk" =
// 8 complex values), instead of 8x8 complex GEMMs on DMMA (3-6x more FP64 pipe slots on B200,
// whose DMMA and DFMA peaks are equal and shared, profiles/r01_fp64_shared.txt).
//
// Stages per tile pair (each a shared-memory read -> registers -> write of 512 chunks, in place):
//   R1 rows, stage a  (chunk (r, n2), n2 pairs as 16-byte words): DFT-8 over n1, * w64^(n2 k1)
//   R2 rows, stage b  (chunk (r, k1), 4 x 16-byte words):          DFT-8 over n2 -> X[k1 + 8 k2]
//                                                                     at column 8 k1 + k2
//   C1 cols, stage a  (chunk (c, n2)):                               DFT-8 over n1, * w64^(n2 k1)
//   C2 cols, stage b, * S_T, inverse stage b (chunk (c, k1)):       DFT-8 over n2, * S, IDFT-8
//                                                                     over k2, * conj w64^(n2 k1)
//   C3 cols, inverse stage a (chunk (c, n2)):                        IDFT-8 over k1 -> rows
//                                                                     8 n1 + n2, S output rows kept
//   R3 S output rows, inverse stage b (chunk (r, k1)):               IDFT-8 over k2, * conj twiddle
//   R4 S output rows, inverse stage a (chunk (r, n2 pair)):          IDFT-8 over k1 -> store window
// Shared layout: four 16-column blocks, each the TMA SWIZZLE_128B image of a 64 x 16 box:
//   word(r, c) = 1024 (c >> 4) + 16 r + ((c & 15) ^ 2 (r & 7)).
// Bank check (8-byte words: a half-warp per wavefront; 16-byte: a quarter-warp): column stages
// (lanes = 16 consecutive c, rows 8 m + n2) hit banks (c & 15) ^ 2 n2 -- distinct; row stages
// use 16-byte words at 16-byte chunk ((c & 15) >> 1) ^ (r & 7) with lanes = 8 consecutive r --
// distinct.  Twiddle indices (n2 or k1 of a chunk) are warp-uniform, so w64^m comes from a
// 1 KB shared table by broadcast.  S_T sits in shared memory in position order (dense [64][64],
// position 8a + b <-> frequency a + 8b on each axis; plan.cpp).
//
// TMA path: one persistent CTA (8 warps) per SM holding two pair buffers (the next pair's
// eight 64 x 16 boxes land while the current pair is transformed) and S_T, 194 KB; the
// cp.async path (periodic wrap-around, or a pitch TMA cannot describe) uses one buffer.
#include "fft_radix.cuh"
#include "kernels.cuh"
#include "tma.cuh"

namespace fstencil {
namespace {

constexpr int L = 64;
constexpr int PLANE = L * L;
constexpr int NW = 8;
constexpr int NT = NW * 32;
constexpr int kAlign = 1024;

__device__ __forceinline__ int wd(int r, int c) { return ((c >> 4) << 10) | (r << 4) | ((c & 15) ^ ((r & 7) << 1)); }

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

using radix::cmul;
using radix::fft8;

// Tuning switches (ablation builds via FFTSTENCIL_NVCC_DEFS): BF_TW_POW = 0 twiddles from the
// shared table, 1 the lane-varying R1 twiddles as powers of w64^n2 in registers, 2 every twiddle
// as powers (default: +6% on B200, fewer shared-memory wavefronts and no spills,
// profiles/r01_s2_ab2d.txt); BF_UNROLL = chunks per thread in flight in the column/row-b stages.
#ifndef BF_TW_POW
#define BF_TW_POW 2
#endif
#ifndef BF_UNROLL
#define BF_UNROLL 1
#endif
constexpr int kUnroll = BF_UNROLL;

// x[j] *= w^(+-j) for j = 1..7 with w = (wr, wi) = w64^t: powers by repeated multiplication
// (6 complex multiplies; error ~ j ulp).
template <bool INV>
__device__ __forceinline__ void twiddle_pow(double (&xr)[8], double (&xi)[8], double wr, double wi) {
  if (INV) wi = -wi;
  double pr = wr, pi = wi;
#pragma unroll
  for (int j = 1; j < 8; ++j) {
    cmul(xr[j], xi[j], pr, pi);
    if (j < 7) {
      const double t = pr * wr - pi * wi;
      pi = fma(pr, wi, pi * wr);
      pr = t;
    }
  }
}

// twiddle x[j] *= w64^(+-t j), j = 1..7; tw[8 j + t] = w64^(j t) (shared, 1 KB): a warp-uniform
// t is a broadcast, t = lane & 7 hits 8 distinct 16-byte chunks per quarter-warp.
template <bool INV>
__device__ __forceinline__ void twiddle_chunk(double (&xr)[8], double (&xi)[8], const double2* tw, int t) {
#pragma unroll
  for (int j = 1; j < 8; ++j) {
    const double2 w = tw[8 * j + t];
    cmul(xr[j], xi[j], w.x, INV ? -w.y : w.y);
  }
}

struct Geom {
  int64_t o0, oa1, ob1;
  bool has_b;
};
__device__ __forceinline__ Geom geom(const Fft2dArgs& a, int64_t p) {
  // pair indices and tile counts fit 32 bits (the plan's pair count is far below 2^31)
  const int npr = (int)a.npr, pi = (int)p;
  const int t0 = pi / npr, pj = pi - t0 * npr;
  Geom g;
  g.o0 = (int64_t)t0 * a.S + a.bd.shift;
  g.oa1 = (int64_t)2 * pj * a.S + a.bd.shift;
  g.ob1 = g.oa1 + a.S;
  g.has_b = 2 * pj + 1 < a.nt1;
  return g;
}

// Row of chunk u in the row stages R1/R4 (n2 = lane & 7): bits 0-1 <- warp & 3, bit 2 <- lane
// bit 3, bit 3 <- lane bit 4, bits 4-5 <- (warp >> 2) + 2 u.
__device__ __forceinline__ int row_of(int warp, int lane, int u) {
  return (warp & 3) | (((lane >> 3) & 1) << 2) | (((lane >> 4) & 1) << 3) | (((warp >> 2) + 2 * u) << 4);
}

// TMA refill of a group buffer with pair p: eight 64 x 16 boxes (OOB -> 0).
__device__ __forceinline__ void issue_pair(const Fft2dArgs& a, const CUtensorMap* tm, const Geom& g, double* dR,
                                           uint64_t* bar) {
  const int y = (int)(g.o0 - a.win.g0);
  tma::mbar_expect_tx(bar, (g.has_b ? 2u : 1u) * PLANE * 8u);
#pragma unroll
  for (int b = 0; b < 4; ++b) tma::load_2d(dR + b * 1024, tm, (int)g.oa1 + 16 * b, y, bar);
  if (g.has_b)
#pragma unroll
    for (int b = 0; b < 4; ++b) tma::load_2d(dR + PLANE + b * 1024, tm, (int)g.ob1 + 16 * b, y, bar);
}

// Barrier of one 256-thread group (ids 1, 2; id 0 is __syncthreads).
__device__ __forceinline__ void group_sync(int grp) { asm volatile("bar.sync %0, %1;\n" ::"r"(grp + 1), "r"(NT) : "memory"); }

// The seven stages over the pair in (sR, sI) by group `grp`; returns after R4's shared reads
// (the buffer may be refilled) with the TMA refill of `next` issued, then stores the window.
template <bool TMA>
__device__ __forceinline__ void tile_stages(double* sR, double* sI, const double* sSr, const double* sSi,
                                            const double2* tw, const Fft2dArgs& a, const Geom& g, int warp,
                                            int lane, int grp, const CUtensorMap* tm, uint64_t* bar, bool has_next,
                                            const Geom& gn) {
  const int S = a.S, h = a.h;
  // ---- R1: rows, stage a; chunk (r, n2), n2 = lane & 7; a half-warp covers rows r0, r0 + 4
  // (8-byte words ((8 n1 + n2) & 15) ^ 2 (r & 7): the two rows land in opposite bank halves) ----
#pragma unroll kUnroll
  for (int u = 0; u < 2; ++u) {
    const int r = row_of(warp, lane, u), n2 = lane & 7;
    double xr[8], xi[8];
#pragma unroll
    for (int n1 = 0; n1 < 8; ++n1) {
      const int o = wd(r, 8 * n1 + n2);
      xr[n1] = sR[o];
      xi[n1] = sI[o];
    }
    fft8<false>(xr, xi);
    if (BF_TW_POW >= 1) {
      const double2 w = tw[8 + n2];   // w64^n2
      twiddle_pow<false>(xr, xi, w.x, w.y);
    } else {
      twiddle_chunk<false>(xr, xi, tw, n2);
    }
#pragma unroll
    for (int k1 = 0; k1 < 8; ++k1) {
      const int o = wd(r, 8 * k1 + n2);
      sR[o] = xr[k1];
      sI[o] = xi[k1];
    }
  }
  group_sync(grp);
  // ---- R2: rows, stage b; chunk (r, k1): columns 8 k1 + n2 (4 x 16-byte words) ----
#pragma unroll kUnroll
  for (int u = 0; u < 2; ++u) {
    const int task = warp + NW * u, r = lane + 32 * (task & 1), k1 = task >> 1;
    double xr[8], xi[8];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int o = wd(r, 8 * k1 + 2 * j);
      const double2 vr = *reinterpret_cast<const double2*>(sR + o);
      const double2 vi = *reinterpret_cast<const double2*>(sI + o);
      xr[2 * j] = vr.x; xr[2 * j + 1] = vr.y; xi[2 * j] = vi.x; xi[2 * j + 1] = vi.y;
    }
    fft8<false>(xr, xi);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int o = wd(r, 8 * k1 + 2 * j);
      *reinterpret_cast<double2*>(sR + o) = make_double2(xr[2 * j], xr[2 * j + 1]);
      *reinterpret_cast<double2*>(sI + o) = make_double2(xi[2 * j], xi[2 * j + 1]);
    }
  }
  group_sync(grp);
  // ---- C1: columns, stage a; chunk (c, n2): rows 8 n1 + n2 ----
#pragma unroll kUnroll
  for (int u = 0; u < 2; ++u) {
    const int task = warp + NW * u, c = lane + 32 * (task & 1), n2 = task >> 1;
    double xr[8], xi[8];
#pragma unroll
    for (int n1 = 0; n1 < 8; ++n1) {
      const int o = wd(8 * n1 + n2, c);
      xr[n1] = sR[o];
      xi[n1] = sI[o];
    }
    fft8<false>(xr, xi);
    if (BF_TW_POW >= 2) {
      const double2 w = tw[8 + n2];
      twiddle_pow<false>(xr, xi, w.x, w.y);
    } else {
      twiddle_chunk<false>(xr, xi, tw, n2);
    }
#pragma unroll
    for (int k1 = 0; k1 < 8; ++k1) {
      const int o = wd(8 * k1 + n2, c);
      sR[o] = xr[k1];
      sI[o] = xi[k1];
    }
  }
  group_sync(grp);
  // ---- C2: columns, stage b, * S_T, inverse stage b; chunk (c, k1): rows 8 k1 + n2 ----
#pragma unroll kUnroll
  for (int u = 0; u < 2; ++u) {
    const int task = warp + NW * u, c = lane + 32 * (task & 1), k1 = task >> 1;
    double xr[8], xi[8];
#pragma unroll
    for (int n2 = 0; n2 < 8; ++n2) {
      const int o = wd(8 * k1 + n2, c);
      xr[n2] = sR[o];
      xi[n2] = sI[o];
    }
    fft8<false>(xr, xi);   // slot k2: frequency k1 + 8 k2 at position 8 k1 + k2
#pragma unroll
    for (int k2 = 0; k2 < 8; ++k2) {
      const int so = (8 * k1 + k2) * L + c;
      cmul(xr[k2], xi[k2], sSr[so], sSi[so]);
    }
    fft8<true>(xr, xi);    // slot n2
    if (BF_TW_POW >= 2) {
      const double2 w = tw[8 + k1];
      twiddle_pow<true>(xr, xi, w.x, w.y);
    } else {
      twiddle_chunk<true>(xr, xi, tw, k1);
    }
#pragma unroll
    for (int n2 = 0; n2 < 8; ++n2) {
      const int o = wd(8 * k1 + n2, c);
      sR[o] = xr[n2];
      sI[o] = xi[n2];
    }
  }
  group_sync(grp);
  // ---- C3: columns, inverse stage a; chunk (c, n2): rows 8 k1 + n2 -> rows 8 n1 + n2 (S kept) ----
#pragma unroll kUnroll
  for (int u = 0; u < 2; ++u) {
    const int task = warp + NW * u, c = lane + 32 * (task & 1), n2 = task >> 1;
    double xr[8], xi[8];
#pragma unroll
    for (int k1 = 0; k1 < 8; ++k1) {
      const int o = wd(8 * k1 + n2, c);
      xr[k1] = sR[o];
      xi[k1] = sI[o];
    }
    fft8<true>(xr, xi);
#pragma unroll
    for (int n1 = 0; n1 < 8; ++n1) {
      const int rr = 8 * n1 + n2;
      if (rr >= h && rr < h + S) {
        const int o = wd(rr, c);
        sR[o] = xr[n1];
        sI[o] = xi[n1];
      }
    }
  }
  group_sync(grp);
  const int nrb = (S + 31) >> 5;   // blocks of 32 output rows
  // ---- R3: the S output rows, inverse stage b; chunk (r, k1) ----
  for (int task = warp; task < 8 * nrb; task += NW) {
    const int i = 32 * (task % nrb) + lane, k1 = task / nrb;
    if (i < S) {
      const int r = h + i;
      double xr[8], xi[8];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int o = wd(r, 8 * k1 + 2 * j);
        const double2 vr = *reinterpret_cast<const double2*>(sR + o);
        const double2 vi = *reinterpret_cast<const double2*>(sI + o);
        xr[2 * j] = vr.x; xr[2 * j + 1] = vr.y; xi[2 * j] = vi.x; xi[2 * j + 1] = vi.y;
      }
      fft8<true>(xr, xi);
      if (BF_TW_POW >= 2) {
        const double2 w = tw[8 + k1];
        twiddle_pow<true>(xr, xi, w.x, w.y);
      } else {
        twiddle_chunk<true>(xr, xi, tw, k1);
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int o = wd(r, 8 * k1 + 2 * j);
        *reinterpret_cast<double2*>(sR + o) = make_double2(xr[2 * j], xr[2 * j + 1]);
        *reinterpret_cast<double2*>(sI + o) = make_double2(xi[2 * j], xi[2 * j + 1]);
      }
    }
  }
  group_sync(grp);
  // ---- R4: the S output rows, inverse stage a; chunk (h + i, n2), the R1 lane map over i ->
  // store the window; both chunks are read before the buffer is released for the refill ----
  double yr[2][8], yi[2][8];
#pragma unroll
  for (int u = 0; u < 2; ++u) {
    const int i = row_of(warp, lane, u), n2 = lane & 7;
    if (i < S) {
#pragma unroll
      for (int k1 = 0; k1 < 8; ++k1) {
        const int o = wd(h + i, 8 * k1 + n2);
        yr[u][k1] = sR[o];
        yi[u][k1] = sI[o];
      }
    }
  }
  if (TMA) tma::fence_proxy_async();   // the buffer is refilled by TMA after the barrier
  group_sync(grp);
  if (TMA && warp == 0 && lane == 0 && has_next) issue_pair(a, tm, gn, sR, bar);
#pragma unroll
  for (int u = 0; u < 2; ++u) {
    const int i = row_of(warp, lane, u), n2 = lane & 7;
    const int64_t c0 = g.o0 + h + i;
    if (i >= S || c0 >= a.bd.lim0 || c0 < a.win.w_lo || c0 >= a.win.w_hi) continue;
    fft8<true>(yr[u], yi[u]);
    double* drow = a.dst + (c0 - a.win.g0) * a.n1;
#pragma unroll
    for (int n1 = 0; n1 < 8; ++n1) {
      const int cc = 8 * n1 + n2;
      if (cc >= h && cc < h + S) {
        int64_t c1 = g.oa1 + cc;
        if (c1 < a.bd.lim1) drow[c1] = yr[u][n1];
        c1 = g.ob1 + cc;
        if (g.has_b && c1 < a.bd.lim1) drow[c1] = yi[u][n1];
      }
    }
  }
}

template <bool TMA, bool WRAP = false>
__global__ void __launch_bounds__(2 * NT, 1) fft2d_bf_kernel(const Fft2dArgs a, const __grid_constant__ CUtensorMap tm) {
  extern __shared__ unsigned char smem_raw[];
  const uint32_t mis = tma::smem_addr(smem_raw) & (kAlign - 1);
  double* base = reinterpret_cast<double*>(smem_raw + (mis ? kAlign - mis : 0));   // stays in the shared window
  const double* sSr = base + 4 * PLANE;
  const double* sSi = sSr + PLANE;
  double2* tw = reinterpret_cast<double2*>(base + 6 * PLANE);
  __shared__ __align__(8) uint64_t bar[3];
  const int grp = threadIdx.x >> 8, tid = threadIdx.x & (NT - 1), warp = tid >> 5, lane = tid & 31;
  double* sR = base + grp * 2 * PLANE;
  double* sI = sR + PLANE;
  if (threadIdx.x == 0) {
    tma::mbar_init(&bar[0], 1);
    tma::mbar_init(&bar[1], 1);
    tma::mbar_init(&bar[2], 1);
  }
  if (threadIdx.x < L) {   // tw[8 j + t] = w64^(j t) from the plan's w64^m table
    const int m = ((threadIdx.x >> 3) * (threadIdx.x & 7)) & 63;
    tw[threadIdx.x] = make_double2(a.Fre[m], a.Fim[m]);
  }
  __syncthreads();
  if (threadIdx.x == 0) {   // S_T once per launch (position order, re | im planes contiguous)
    tma::mbar_expect_tx(&bar[2], 2u * PLANE * 8u);
    tma::load_bulk(base + 4 * PLANE, a.Sre, PLANE * 8u, &bar[2]);
    tma::load_bulk(base + 5 * PLANE, a.Sim, PLANE * 8u, &bar[2]);
  }
  const int64_t stride = 2 * (int64_t)gridDim.x;
  const int64_t p0 = a.win.p_begin + 2 * (int64_t)blockIdx.x + grp;
  if (TMA && tid == 0 && p0 < a.win.p_end) issue_pair(a, &tm, geom(a, p0), sR, &bar[grp]);
  tma::mbar_wait(&bar[2], 0);

  uint32_t parity = 0;
  for (int64_t p = p0; p < a.win.p_end; p += stride) {
    const Geom g = geom(a, p);
    if (TMA) {
      tma::mbar_wait(&bar[grp], parity);
      parity ^= 1;
      if (!g.has_b) {
        for (int e = tid; e < PLANE; e += NT) sI[e] = 0.0;
        group_sync(grp);
      }
    } else {
      for (int e = tid; e < 2 * PLANE; e += NT) {
        const int t = e >> 12, r = (e >> 6) & 63, c = e & 63;
        int64_t g0 = g.o0 + r, g1 = (t ? g.ob1 : g.oa1) + c;
        if (WRAP) { g0 = wrap_index(g0, a.n0); g1 = wrap_index(g1, a.n1); }
        const int64_t lg0 = g0 - a.win.g0;
        const bool valid = (t == 0 || g.has_b) && g0 < a.n0 && lg0 >= 0 && lg0 < a.win.gn && g1 >= 0 && g1 < a.n1;
        cp_async8((t ? sI : sR) + wd(r, c), valid ? a.src + lg0 * a.n1 + g1 : a.src, valid);
      }
      asm volatile("cp.async.commit_group;\n" ::);
      asm volatile("cp.async.wait_all;\n" ::: "memory");
      group_sync(grp);
    }
    const bool has_next = p + stride < a.win.p_end;
    const Geom gn = geom(a, has_next ? p + stride : p);
    tile_stages<TMA>(sR, sI, sSr, sSi, tw, a, g, warp, lane, grp, &tm, &bar[grp], has_next, gn);
  }
}

}  // namespace

// Two group buffers + S_T + the w64 table.
size_t fused2d_bf_smem(bool) { return (size_t)6 * PLANE * sizeof(double) + 64 * 16 + kAlign; }

cudaError_t fused2d_bf_configure(int* max_blocks) {
  const int st = (int)fused2d_bf_smem(true), sc = (int)fused2d_bf_smem(false);
  cudaError_t e = cudaFuncSetAttribute(fft2d_bf_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, st);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(fft2d_bf_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sc);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft2d_bf_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sc);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft2d_bf_kernel<true>, 2 * NT, st);
}

cudaError_t launch_fused2d_bf(const Fft2dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s) {
  static const CUtensorMap none = {};
  if (tm)
    fft2d_bf_kernel<true><<<grid, 2 * NT, fused2d_bf_smem(true), s>>>(a, *tm);
  else if (a.bd.wrap)
    fft2d_bf_kernel<false, true><<<grid, 2 * NT, fused2d_bf_smem(false), s>>>(a, none);
  else
    fft2d_bf_kernel<false><<<grid, 2 * NT, fused2d_bf_smem(false), s>>>(a, none);
  return cudaGetLastError();
}

}  // namespace fstencil
