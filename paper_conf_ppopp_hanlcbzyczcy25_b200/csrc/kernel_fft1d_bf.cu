// Fused 1D FFT-stencil tile kernel, long factored tile L = 4096 = 64 x 64, with butterflies on
// the FP64 ALU (sm_100a): the default 1D engine.
//
// Same pass as kernel_fft1d_ct.cu (the four-step form of §3.2.1's reshaping, L208-L218, on a
// 4096-cell overlap-save tile; Double-layer Filling Eq. 9; temporal fusion Eq. 10):
//     n = a + 64 b,  k = c + 64 d
//     X[c + 64 d] = sum_a w64^(a d) w4096^(a c) sum_b x[a + 64 b] w64^(b c)
// with the tile held as a 64 x 64 plane (row b, column a) and each DFT-64 split 64 = 4 x 16 as
// in kernel_fft2d_bf.cu (position 16 k0 + k' <-> frequency k0 + 4 k').  The w4096 twiddle sits
// between the column and the row transform, so the stage-1 passes cannot serve both axes at
// once (as they do in 2D) -- seven in-place shared-memory passes per pair:
//   P1 column stage 1 (4 x 4 blocks: DFT-4 over the row digit, * w64^(rr c0))
//   P2 column stage 2 (DFT-16 down a column segment) * w4096^(a c)
//   P3 row stage 1    (4 x 4 blocks: DFT-4 over the column digit, * w64^(cc d0))
//   P4 row stage 2 (DFT-16 along a row segment), * S_T, inverse DFT-16
//   P5 row inverse stage 1, P6 * conj w4096 + column inverse stage 2, P7 column inverse
//   stage 1 -> store the S valid cells [h, h + S) of each tile (Eq. 7, reading Q4).
// w4096^(a (c0 + 4 c')) = w4096^(a c0) (w4096^(4 a))^c' is formed by register powers from a
// 256-entry table.  Layout, bank analysis, TMA staging (the tile as four 64 x 16 boxes of the
// grid viewed as rows of 64 cells; used when tile origins and the grid are 64-aligned) and the
// two-group CTA organisation are those of kernel_fft2d_bf.cu.  S_T is staged in shared memory
// transposed ([column position][row position], interleaved) so P4's lanes (consecutive rows)
// read consecutive 16-byte words.
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
constexpr int kTw4096 = 256;   // w4096^m, m < 256

__device__ __forceinline__ int wd(int r, int c) { return ((c >> 4) << 10) | (r << 4) | ((c & 15) ^ ((r & 7) << 1)); }

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

using radix::cmul;
using radix::dft4;
using radix::fft16;

struct Geom {
  int64_t oa, ob;   // tile origins (cell of plane element (0, 0))
  bool has_b;
};
__device__ __forceinline__ Geom geom(const Fft1dArgs& a, int64_t p) {
  Geom g;
  g.oa = 2 * p * a.S + a.bd.shift;
  g.ob = g.oa + a.S;
  g.has_b = 2 * p + 1 < a.ntiles;
  return g;
}

// TMA refill: the grid as rows of 64 cells, a tile = rows (o - g0) / 64 .. + 63, four 64 x 16 boxes.
__device__ __forceinline__ void issue_pair(const Fft1dArgs& a, const CUtensorMap* tm, const Geom& g, double* dR,
                                           uint64_t* bar) {
  tma::mbar_expect_tx(bar, (g.has_b ? 2u : 1u) * PLANE * 8u);
  const int ya = (int)((g.oa - a.win.g0) >> 6), yb = (int)((g.ob - a.win.g0) >> 6);
#pragma unroll
  for (int b = 0; b < 4; ++b) tma::load_2d(dR + b * 1024, tm, 16 * b, ya, bar);
  if (g.has_b)
#pragma unroll
    for (int b = 0; b < 4; ++b) tma::load_2d(dR + PLANE + b * 1024, tm, 16 * b, yb, bar);
}

__device__ __forceinline__ void group_sync(int grp) { asm volatile("bar.sync %0, %1;\n" ::"r"(grp + 1), "r"(NT) : "memory"); }

__device__ __forceinline__ void load_block(const double* sR, const double* sI, int rr, int cc, double (&xr)[4][4],
                                           double (&xi)[4][4]) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int o = wd(16 * i + rr, 16 * j + cc);
      xr[i][j] = sR[o];
      xi[i][j] = sI[o];
    }
}
__device__ __forceinline__ void store_block(double* sR, double* sI, int rr, int cc, const double (&xr)[4][4],
                                            const double (&xi)[4][4]) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int o = wd(16 * i + rr, 16 * j + cc);
      sR[o] = xr[i][j];
      sI[o] = xi[i][j];
    }
}

// Column stage 1 on a 4 x 4 block: DFT-4 over i for every j, [i][j] *= w64^(+-rr i).
template <bool INV>
__device__ __forceinline__ void col_stage1(double (&xr)[4][4], double (&xi)[4][4], const double2* tw64, int rr) {
  if (INV) {   // conj twiddle first, then the inverse DFT-4
#pragma unroll
    for (int i = 1; i < 4; ++i) {
      const double2 w = tw64[(rr * i) & 63];
#pragma unroll
      for (int j = 0; j < 4; ++j) cmul(xr[i][j], xi[i][j], w.x, -w.y);
    }
  }
#pragma unroll
  for (int j = 0; j < 4; ++j)
    dft4<INV>(xr[0][j], xi[0][j], xr[1][j], xi[1][j], xr[2][j], xi[2][j], xr[3][j], xi[3][j]);
  if (!INV) {
#pragma unroll
    for (int i = 1; i < 4; ++i) {
      const double2 w = tw64[(rr * i) & 63];
#pragma unroll
      for (int j = 0; j < 4; ++j) cmul(xr[i][j], xi[i][j], w.x, w.y);
    }
  }
}

// Row stage 1 on a 4 x 4 block: DFT-4 over j for every i, [i][j] *= w64^(+-cc j).
template <bool INV>
__device__ __forceinline__ void row_stage1(double (&xr)[4][4], double (&xi)[4][4], const double2* tw64, int cc) {
  if (INV) {
#pragma unroll
    for (int j = 1; j < 4; ++j) {
      const double2 w = tw64[(cc * j) & 63];
#pragma unroll
      for (int i = 0; i < 4; ++i) cmul(xr[i][j], xi[i][j], w.x, -w.y);
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
    dft4<INV>(xr[i][0], xi[i][0], xr[i][1], xi[i][1], xr[i][2], xi[i][2], xr[i][3], xi[i][3]);
  if (!INV) {
#pragma unroll
    for (int j = 1; j < 4; ++j) {
      const double2 w = tw64[(cc * j) & 63];
#pragma unroll
      for (int i = 0; i < 4; ++i) cmul(xr[i][j], xi[i][j], w.x, w.y);
    }
  }
}

// x[c'] *= (base * step^c')^(+-1), c' = 0..15 (register powers; base = w4096^(a c0), step = w4096^(4 a)).
template <bool INV>
__device__ __forceinline__ void twiddle4096(double (&xr)[16], double (&xi)[16], double2 base, double2 step) {
  double wr = base.x, wi = INV ? -base.y : base.y;
  const double sr = step.x, si = INV ? -step.y : step.y;
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    cmul(xr[k], xi[k], wr, wi);
    if (k < 15) cmul(wr, wi, sr, si);
  }
}

template <bool TMA, bool PEER>
__device__ __forceinline__ void tile_passes(double* sR, double* sI, const double* sS, const double2* tw64,
                                            const double2* tw4k, const Fft1dArgs& a, const Geom& g, int warp,
                                            int lane, int grp, const CUtensorMap* tm, uint64_t* bar, bool has_next,
                                            const Geom& gn) {
  const int S = a.S, h = a.h;
  const int rr = (warp << 1) | (lane >> 4), cc = lane & 15;     // block classes (P1, P3, P5, P7)
  const int rc = lane + ((warp & 1) << 5), blk = warp >> 1;      // segment passes (P2, P4, P6)
  double br[4][4], bi[4][4];
  // ---- P1: column stage 1 ----
  load_block(sR, sI, rr, cc, br, bi);
  col_stage1<false>(br, bi, tw64, rr);
  store_block(sR, sI, rr, cc, br, bi);
  group_sync(grp);
  // ---- P2: column stage 2 (column a = rc, rows 16 c0 + m, c0 = blk) * w4096^(a c) ----
  {
    double xr[16], xi[16];
#pragma unroll
    for (int m = 0; m < 16; ++m) {
      const int o = wd(16 * blk + m, rc);
      xr[m] = sR[o];
      xi[m] = sI[o];
    }
    fft16<false>(xr, xi);   // slot c': c = blk + 4 c'
    twiddle4096<false>(xr, xi, tw4k[rc * blk], tw4k[4 * rc]);
#pragma unroll
    for (int m = 0; m < 16; ++m) {
      const int o = wd(16 * blk + m, rc);
      sR[o] = xr[m];
      sI[o] = xi[m];
    }
  }
  group_sync(grp);
  // ---- P3: row stage 1 ----
  load_block(sR, sI, rr, cc, br, bi);
  row_stage1<false>(br, bi, tw64, cc);
  store_block(sR, sI, rr, cc, br, bi);
  group_sync(grp);
  // ---- P4: row stage 2 (row rc, columns 16 d0 + m, d0 = blk), * S_T, inverse ----
  {
    const int base = (blk << 10) | (rc << 4), s = rc & 7;
    double xr[16], xi[16];
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const int o = base + ((c ^ s) << 1);
      const double2 vr = *reinterpret_cast<const double2*>(sR + o);
      const double2 vi = *reinterpret_cast<const double2*>(sI + o);
      xr[2 * c] = vr.x; xr[2 * c + 1] = vr.y;
      xi[2 * c] = vi.x; xi[2 * c + 1] = vi.y;
    }
    fft16<false>(xr, xi);   // slot d': column position 16 blk + d'
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      const double2 sv = *reinterpret_cast<const double2*>(sS + ((((16 * blk + k) << 6) + rc) << 1));
      cmul(xr[k], xi[k], sv.x, sv.y);
    }
    fft16<true>(xr, xi);
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const int o = base + ((c ^ s) << 1);
      *reinterpret_cast<double2*>(sR + o) = make_double2(xr[2 * c], xr[2 * c + 1]);
      *reinterpret_cast<double2*>(sI + o) = make_double2(xi[2 * c], xi[2 * c + 1]);
    }
  }
  group_sync(grp);
  // ---- P5: row inverse stage 1 ----
  load_block(sR, sI, rr, cc, br, bi);
  row_stage1<true>(br, bi, tw64, cc);
  store_block(sR, sI, rr, cc, br, bi);
  group_sync(grp);
  // ---- P6: * conj w4096^(a c), column inverse stage 2 ----
  {
    double xr[16], xi[16];
#pragma unroll
    for (int m = 0; m < 16; ++m) {
      const int o = wd(16 * blk + m, rc);
      xr[m] = sR[o];
      xi[m] = sI[o];
    }
    twiddle4096<true>(xr, xi, tw4k[rc * blk], tw4k[4 * rc]);
    fft16<true>(xr, xi);
#pragma unroll
    for (int m = 0; m < 16; ++m) {
      const int o = wd(16 * blk + m, rc);
      sR[o] = xr[m];
      sI[o] = xi[m];
    }
  }
  group_sync(grp);
  // ---- P7: column inverse stage 1 -> store (read, release, compute) ----
  load_block(sR, sI, rr, cc, br, bi);
  if (TMA) tma::fence_proxy_async();
  group_sync(grp);
  if (TMA && warp == 0 && lane == 0 && has_next) issue_pair(a, tm, gn, sR, bar);
  col_stage1<true>(br, bi, tw64, rr);
  // tile offsets l = a + 64 b stored: [h, h + S) within the grid limit and the rank's window
  const int64_t hi_c = min(a.bd.lim0, a.win.w_hi);
  const int la0 = (int)max((int64_t)h, a.win.w_lo - g.oa), la1 = (int)min((int64_t)(h + S), hi_c - g.oa);
  const int lb0 = (int)max((int64_t)h, a.win.w_lo - g.ob);
  const int lb1 = g.has_b ? (int)min((int64_t)(h + S), hi_c - g.ob) : 0;
  double* da = a.dst + (g.oa - a.win.g0);
  double* db = a.dst + (g.ob - a.win.g0);
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int l = 16 * j + cc + 64 * (16 * i + rr);   // cell offset a + 64 b within the tile
      if (l >= la0 && l < la1) da[l] = br[i][j];
      if (l >= lb0 && l < lb1) db[l] = bi[i][j];
      if (PEER) {   // boundary cells of a peer-transport rank: also into the neighbour's halo
        const int64_t c = g.oa + l, d = g.ob + l;
        if (l >= la0 && l < la1) {
          if (c < a.peer.lo_end) a.peer.lo[c - a.peer.lo_g0] = br[i][j];
          else if (c >= a.peer.hi_begin) a.peer.hi[c - a.peer.hi_g0] = br[i][j];
        }
        if (l >= lb0 && l < lb1) {
          if (d < a.peer.lo_end) a.peer.lo[d - a.peer.lo_g0] = bi[i][j];
          else if (d >= a.peer.hi_begin) a.peer.hi[d - a.peer.hi_g0] = bi[i][j];
        }
      }
    }
}

// PEER: boundary cells of a peer-transport rank are also stored into the neighbour (a.peer).
template <bool TMA, bool WRAP = false, bool PEER = false>
__global__ void __launch_bounds__(2 * NT, 1) fft1d_bf_kernel(const Fft1dArgs a, const __grid_constant__ CUtensorMap tm) {
  extern __shared__ unsigned char smem_raw[];
  const uint32_t mis = tma::smem_addr(smem_raw) & (kAlign - 1);
  double* base = reinterpret_cast<double*>(smem_raw + (mis ? kAlign - mis : 0));
  double* sS = base + 4 * PLANE;                                         // [column pos][row pos], (re, im)
  double2* tw64 = reinterpret_cast<double2*>(base + 6 * PLANE);          // w64^m
  double2* tw4k = tw64 + L;                                              // w4096^m, m < 256
  __shared__ __align__(8) uint64_t bar[2];
  const int grp = threadIdx.x >> 8, tid = threadIdx.x & (NT - 1), warp = tid >> 5, lane = tid & 31;
  double* sR = base + grp * 2 * PLANE;
  double* sI = sR + PLANE;
  if (threadIdx.x == 0) {
    tma::mbar_init(&bar[0], 1);
    tma::mbar_init(&bar[1], 1);
  }
  if (threadIdx.x < L) tw64[threadIdx.x] = make_double2(a.Fre[threadIdx.x], a.Fim[threadIdx.x]);
  if (threadIdx.x < kTw4096) tw4k[threadIdx.x] = make_double2(a.tw[2 * threadIdx.x], a.tw[2 * threadIdx.x + 1]);
  for (int e = threadIdx.x; e < PLANE; e += 2 * NT)   // once per launch
    *reinterpret_cast<double2*>(sS + 2 * e) = make_double2(__ldg(a.Sre + e), __ldg(a.Sim + e));
  __syncthreads();
  const int64_t np = (a.ntiles + 1) / 2;
  const int64_t stride = 2 * (int64_t)gridDim.x;
  const int64_t p_end = min(a.win.p_end, np);
  const int64_t p0 = a.win.p_begin + 2 * (int64_t)blockIdx.x + grp;
  if (TMA && tid == 0 && p0 < p_end) issue_pair(a, &tm, geom(a, p0), sR, &bar[grp]);

  uint32_t parity = 0;
  for (int64_t p = p0; p < p_end; p += stride) {
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
        const int t = e >> 12, l = e & (PLANE - 1);
        int64_t c = (t ? g.ob : g.oa) + l;
        if (WRAP) c = wrap_index(c, a.n);
        const int64_t lc = c - a.win.g0;
        const bool valid = (t == 0 || g.has_b) && c >= 0 && c < a.n && lc >= 0 && lc < a.win.gn;
        cp_async8((t ? sI : sR) + wd(l >> 6, l & 63), valid ? a.src + lc : a.src, valid);
      }
      asm volatile("cp.async.commit_group;\n" ::);
      asm volatile("cp.async.wait_all;\n" ::: "memory");
      group_sync(grp);
    }
    const bool has_next = p + stride < p_end;
    const Geom gn = geom(a, has_next ? p + stride : p);
    tile_passes<TMA, PEER>(sR, sI, sS, tw64, tw4k, a, g, warp, lane, grp, &tm, &bar[grp], has_next, gn);
  }
}

}  // namespace

// Two group buffers + S_T + the w64 and w4096 tables.
size_t fused1d_bf_smem() { return (size_t)6 * PLANE * sizeof(double) + (L + kTw4096) * 16 + kAlign; }

cudaError_t fused1d_bf_configure(int* max_blocks) {
  const int sm = (int)fused1d_bf_smem();
  cudaError_t e = cudaFuncSetAttribute(fft1d_bf_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(fft1d_bf_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft1d_bf_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft1d_bf_kernel<true, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft1d_bf_kernel<false, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft1d_bf_kernel<true>, 2 * NT, sm);
}

cudaError_t launch_fused1d_bf(const Fft1dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s) {
  static const CUtensorMap none = {};
  if (a.peer.lo || a.peer.hi) {   // boundary cells of a peer-transport rank (never periodic)
    if (tm)
      fft1d_bf_kernel<true, false, true><<<grid, 2 * NT, fused1d_bf_smem(), s>>>(a, *tm);
    else
      fft1d_bf_kernel<false, false, true><<<grid, 2 * NT, fused1d_bf_smem(), s>>>(a, none);
    return cudaGetLastError();
  }
  if (tm)
    fft1d_bf_kernel<true><<<grid, 2 * NT, fused1d_bf_smem(), s>>>(a, *tm);
  else if (a.bd.wrap)
    fft1d_bf_kernel<false, true><<<grid, 2 * NT, fused1d_bf_smem(), s>>>(a, none);
  else
    fft1d_bf_kernel<false><<<grid, 2 * NT, fused1d_bf_smem(), s>>>(a, none);
  return cudaGetLastError();
}

}  // namespace fstencil
