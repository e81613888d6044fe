// Fused 2D FFT-stencil tile kernel with register-resident butterflies on the FP64 ALU
// (sm_100a): the default 2D engine.
//
// Same fused pass and tile geometry as kernel_fft2d_ct.cu (Algorithm 1 L252-L258 on
// 64 x 64 overlap-save tiles, Double-layer Filling Eq. 9, temporal fusion Eq. 10, Stitching
// Eq. 7).  Each length-64 axis DFT is the Cooley-Tukey factorisation 64 = 4 x 16 (§3.2.1's
// reshaping, L208-L218), n = 16 n2 + m, k = k0 + 4 k':
//   X[k0 + 4 k'] = sum_m w16^(m k') w64^(m k0) sum_n2 w4^(n2 k0) x[16 n2 + m]
// evaluated with butterflies in registers (fft_radix.cuh) instead of DFT GEMMs on DMMA (B200's
// DMMA and DFMA peaks are equal and shared, profiles/r01_fp64_shared.txt, Q20).
//
// Five in-place shared-memory passes per tile pair; a thread owns 16 complex values per pass:
//   P1 (thread = row class rr, column class cc; the 4 x 4 block rows 16 i + rr, columns
//      16 j + cc): DFT-4 over i and over j, * w64^(rr k0r) w64^(cc k0c)   [both axes, stage 1]
//   P2 (thread = row r, column block b): DFT-16 over the 16 columns 16 b + m   [axis 1, stage 2]
//   P3 (thread = column c, row block b): DFT-16 over the rows 16 b + m, * S_T, inverse DFT-16
//                                                                           [axis 0, stage 2]
//   P4 (thread = row r, column block b): inverse DFT-16                      [axis 1, stage 2]
//   P5 (as P1): * conj twiddles, inverse DFT-4 over j and i -> store the S x S window.
// After P2/P3 position 16 k0 + k' of an axis holds frequency k0 + 4 k' (S_T is stored in that
// position order by the plan).  Doing stage 1 of both axes in one pass (4 x 4 register blocks)
// needs 5 passes where a thread-per-chunk radix-8 design needs 7: shared-memory traffic, which
// binds this kernel, drops by ~25%.
// Shared layout: four 64 x 16 column blocks, each the TMA SWIZZLE_128B image of one box:
//   word(r, c) = 1024 (c >> 4) + 16 r + ((c & 15) ^ 2 (r & 7)).
// Bank check (8-byte words: a half-warp per wavefront; 16-byte: a quarter-warp): P1/P5/P3 give
// a half-warp 16 consecutive columns of one block and one row -> words (c & 15) ^ 2 (r & 7)
// distinct; P2/P4 read a row block as 16-byte words, chunk ((c & 15) >> 1) ^ (r & 7), with 8
// consecutive rows per quarter-warp -> distinct.  S_T (interleaved re/im, 16-byte words,
// consecutive columns per lane) and the w64 table sit in shared memory, staged once per launch.
//
// One CTA per SM = two independent 256-thread groups, each transforming its own sequence of
// tile pairs in its own 64 KB buffer (named barriers); a group releases its buffer after P5's
// reads and its next pair's eight TMA boxes (64 x 16, SWIZZLE_128B, OOB -> 0) land while it
// finishes the inverse and the stores.  The cp.async path (periodic wrap-around, or a pitch TMA
// cannot describe) loads the same layout synchronously.
//
// Six variants measured slower on B200 (twiddle powers in registers, combined twiddles,
// warp-local row passes, S_T in tensor memory, a ping-pong schedule of the two groups,
// interleaved complex words after P1, profiles/r01_s3_ab2d.txt) were removed
// from this file in round 2; they are in git history (commit b1c0b88, BF_* macros).
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

// The row swizzle of the TMA SWIZZLE_128B image (r & 7), kept by every later pass.
__device__ __forceinline__ int wn(int r, int c) { return wd(r, c); }

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

using radix::cmul;
using radix::dft4;
using radix::fft16;

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

// TMA refill of a group buffer with one pair: eight 64 x 16 boxes (OOB -> 0).
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

// The 4 x 4 block of P1/P5: element [i][j] at row 16 i + rr, column 16 j + cc.
template <bool TMA_LAYOUT>
__device__ __forceinline__ void load_block(const double* sR, const double* sI, int rr, int cc, double (&xr)[4][4],
                                           double (&xi)[4][4]) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int o = TMA_LAYOUT ? wd(16 * i + rr, 16 * j + cc) : wn(16 * i + rr, 16 * j + cc);
      xr[i][j] = sR[o];
      xi[i][j] = sI[o];
    }
}

// DFT-4 over i (axis 0) for every j and over j (axis 1) for every i.
template <bool INV>
__device__ __forceinline__ void dft4x4(double (&xr)[4][4], double (&xi)[4][4]) {
#pragma unroll
  for (int j = 0; j < 4; ++j)
    dft4<INV>(xr[0][j], xi[0][j], xr[1][j], xi[1][j], xr[2][j], xi[2][j], xr[3][j], xi[3][j]);
#pragma unroll
  for (int i = 0; i < 4; ++i)
    dft4<INV>(xr[i][0], xi[i][0], xr[i][1], xi[i][1], xr[i][2], xi[i][2], xr[i][3], xi[i][3]);
}

// Shared twiddle table layout: w64^m sits at 16-byte word kTwPos[m], a permutation of 0..63
// chosen (by a colouring search) so that the column twiddles w64^(cc i) of a quarter-warp
// (cc = 8q..8q+7, i = 1, 2, 3) fall in eight different bank slots: with the natural layout
// i = 2 hit four slots twice each (the 2-way conflicts ncu counted, ~8 % of the kernel's
// shared-memory wavefronts).  The row twiddles w64^(rr i) are one address per
// half-warp (broadcast).
__constant__ unsigned char kTwPos[64] = {0, 2, 5, 4, 6, 3, 1, 7, 11, 13, 12, 8, 10, 9, 15, 14, 18, 16, 19, 24, 20, 23, 21, 32, 40, 48, 22, 26, 31, 56, 17, 25, 33, 27, 41, 49, 28, 57, 34, 29, 42, 50, 30, 58, 35, 39, 43, 51, 59, 36, 44, 52, 60, 37, 45, 53, 61, 38, 46, 54, 62, 47, 55, 63};

// element [i][j] *= w64^(+-(rr i + cc j)) (conjugate if INV): a row and a column twiddle, all
// six powers from the shared w64^m table (prow / pcol: the thread's table words of w64^(rr i) and
// w64^(cc i), i = 1..3, looked up once per launch, one byte each).
template <bool INV>
__device__ __forceinline__ void twiddle4x4(double (&xr)[4][4], double (&xi)[4][4], const double2* tw,
                                           uint32_t prow, uint32_t pcol) {
  double2 pr[4], pc[4];
#pragma unroll
  for (int i = 1; i < 4; ++i) {   // byte i - 1 of prow / pcol: the word of w64^(rr i) / w64^(cc i)
    pr[i] = tw[(prow >> (8 * i - 8)) & 63];
    pc[i] = tw[(pcol >> (8 * i - 8)) & 63];
  }
#pragma unroll
  for (int i = 1; i < 4; ++i) {
    const double wi = INV ? -pr[i].y : pr[i].y;
#pragma unroll
    for (int j = 0; j < 4; ++j) cmul(xr[i][j], xi[i][j], pr[i].x, wi);
  }
#pragma unroll
  for (int j = 1; j < 4; ++j) {
    const double wi = INV ? -pc[j].y : pc[j].y;
#pragma unroll
    for (int i = 0; i < 4; ++i) cmul(xr[i][j], xi[i][j], pc[j].x, wi);
  }
}

// P2/P4: the 16 columns 16 b + m of row r as 16-byte words (chunk (m >> 1) ^ (r & 7)).
__device__ __forceinline__ void row_load(const double* sR, const double* sI, int r, int b, double (&xr)[16],
                                         double (&xi)[16]) {
  const int base = (b << 10) | (r << 4), s = r & 7;
#pragma unroll
  for (int c = 0; c < 8; ++c) {
    const int o = base + ((c ^ s) << 1);
    const double2 vr = *reinterpret_cast<const double2*>(sR + o);
    const double2 vi = *reinterpret_cast<const double2*>(sI + o);
    xr[2 * c] = vr.x; xr[2 * c + 1] = vr.y;
    xi[2 * c] = vi.x; xi[2 * c + 1] = vi.y;
  }
}
__device__ __forceinline__ void row_store(double* sR, double* sI, int r, int b, const double (&xr)[16],
                                          const double (&xi)[16]) {
  const int base = (b << 10) | (r << 4), s = r & 7;
#pragma unroll
  for (int c = 0; c < 8; ++c) {
    const int o = base + ((c ^ s) << 1);
    *reinterpret_cast<double2*>(sR + o) = make_double2(xr[2 * c], xr[2 * c + 1]);
    *reinterpret_cast<double2*>(sI + o) = make_double2(xi[2 * c], xi[2 * c + 1]);
  }
}
// P3: the 16 rows 16 blk + m of column rc (8-byte words).
__device__ __forceinline__ void col_load(const double* sR, const double* sI, int rc, int blk, double (&xr)[16],
                                         double (&xi)[16]) {
#pragma unroll
  for (int m = 0; m < 16; ++m) {
    const int o = wn(16 * blk + m, rc);
    xr[m] = sR[o];
    xi[m] = sI[o];
  }
}
__device__ __forceinline__ void col_store(double* sR, double* sI, int rc, int blk, const double (&xr)[16],
                                          const double (&xi)[16]) {
#pragma unroll
  for (int m = 0; m < 16; ++m) {
    const int o = wn(16 * blk + m, rc);
    sR[o] = xr[m];
    sI[o] = xi[m];
  }
}
__device__ __forceinline__ void block_store(double* sR, double* sI, int rr, int cc, const double (&xr)[4][4],
                                            const double (&xi)[4][4]) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int o = wn(16 * i + rr, 16 * j + cc);
      sR[o] = xr[i][j];
      sI[o] = xi[i][j];
    }
}

// The five passes over the pair in (sR, sI) by group `grp`, whose tile data are in place (the
// caller waited for them); releases the buffer (TMA refill of the group's next pair `gnext`)
// after P5's reads, then stores the window.
template <bool TMA>
__device__ __forceinline__ void tile_passes(double* sR, double* sI, const double* sS, const double2* tw,
                                            const Fft2dArgs& a, const Geom& g, int warp, int lane, int grp,
                                            const CUtensorMap* tm, uint64_t* bar, bool has_next, const Geom& gnext,
                                            uint32_t prow, uint32_t pcol) {
  const int S = a.S, h = a.h;
  const int rr = (warp << 1) | (lane >> 4), cc = lane & 15;     // P1/P5 block classes
  const int rc = lane + ((warp & 1) << 5), blk = warp >> 1;      // P3 column, row block
  const int r2 = rc, b2 = blk;                                  // P2/P4 row and column block
  double xr[16], xi[16];
  {
    // ---- P1: stage 1 of both axes ----
    double br[4][4], bi[4][4];
    load_block<true>(sR, sI, rr, cc, br, bi);
    dft4x4<false>(br, bi);
    twiddle4x4<false>(br, bi, tw, prow, pcol);
    block_store(sR, sI, rr, cc, br, bi);
  }
  // ---- P2: axis 1, DFT-16 along row r2, block b2 ----
  group_sync(grp);
  row_load(sR, sI, r2, b2, xr, xi);
  fft16<false>(xr, xi);
  // ---- P3: axis 0 DFT-16 down column rc in row block blk, * S_T, inverse DFT-16 ----
  row_store(sR, sI, r2, b2, xr, xi);
  group_sync(grp);
  col_load(sR, sI, rc, blk, xr, xi);
  fft16<false>(xr, xi);   // slot k': position 16 blk + k' <-> frequency blk + 4 k'
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    const double2 sv = *reinterpret_cast<const double2*>(sS + ((((16 * blk + k) << 6) + rc) << 1));
    cmul(xr[k], xi[k], sv.x, sv.y);
  }
  fft16<true>(xr, xi);
  // ---- P4: axis 1 inverse DFT-16 ----
  col_store(sR, sI, rc, blk, xr, xi);
  group_sync(grp);
  row_load(sR, sI, r2, b2, xr, xi);
  fft16<true>(xr, xi);
  // ---- P5: conj twiddles, inverse stage 1 of both axes (after the buffer's release), store ----
  row_store(sR, sI, r2, b2, xr, xi);
  group_sync(grp);
  double br[4][4], bi[4][4];
  load_block<false>(sR, sI, rr, cc, br, bi);
  if (TMA) tma::fence_proxy_async();   // the buffer is refilled by TMA after the barrier
  group_sync(grp);
  if (TMA && warp == 0 && lane == 0 && has_next) issue_pair(a, tm, gnext, sR, bar);
  twiddle4x4<true>(br, bi, tw, prow, pcol);
  dft4x4<true>(br, bi);
  // column predicates once per pass (valid window [h, h + S), grid limit, tile b present), in
  // 32-bit arithmetic: every column coordinate and limit is < 2^31 (plan: extents < 2^31)
  const int ca = (int)g.oa1 + cc, cb = (int)g.ob1 + cc, lim1 = (int)a.bd.lim1;
  bool va[4], vb[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int c = 16 * j + cc;
    const bool in = c >= h && c < h + S;
    va[j] = in && ca + 16 * j < lim1;
    vb[j] = in && g.has_b && cb + 16 * j < lim1;
  }
  // rows [r_lo, r_hi) of the tile (clamped into [h, h + S] before narrowing)
  const int r_lo = (int)min((int64_t)(h + S), max((int64_t)h, max(a.win.w_lo, (int64_t)0) - g.o0));
  const int r_hi = (int)max((int64_t)h, min((int64_t)(h + S), min(a.bd.lim0, a.win.w_hi) - g.o0));
  double* dbase = a.dst + (g.o0 - a.win.g0) * a.n1;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int r = 16 * i + rr;
    if (r < r_lo || r >= r_hi) continue;
    double* drow = dbase + (int64_t)r * a.n1;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (va[j]) drow[ca + 16 * j] = br[i][j];
      if (vb[j]) drow[cb + 16 * j] = bi[i][j];
    }
  }
}

template <bool TMA, bool WRAP = false>
__global__ void __launch_bounds__(2 * NT, 1) fft2d_bf_kernel(const Fft2dArgs a, const __grid_constant__ CUtensorMap tm) {
  extern __shared__ unsigned char smem_raw[];
  const uint32_t mis = tma::smem_addr(smem_raw) & (kAlign - 1);
  double* base = reinterpret_cast<double*>(smem_raw + (mis ? kAlign - mis : 0));   // stays in the shared window
  double* sS = base + 4 * PLANE;                                  // S_T interleaved (re, im), position order
  double2* tw = reinterpret_cast<double2*>(base + 6 * PLANE);    // w64^m
  __shared__ __align__(8) uint64_t bar[2];
  const int grp = threadIdx.x >> 8, tid = threadIdx.x & (NT - 1), warp = tid >> 5, lane = tid & 31;
  double* sR = base + grp * 2 * PLANE;
  double* sI = sR + PLANE;
  if (threadIdx.x == 0) {
    tma::mbar_init(&bar[0], 1);
    tma::mbar_init(&bar[1], 1);
  }
  if (threadIdx.x < L) tw[kTwPos[threadIdx.x]] = make_double2(a.Fre[threadIdx.x], a.Fim[threadIdx.x]);
  // table words of this thread's P1/P5 twiddles (rr, cc as in tile_passes), one byte per power
  uint32_t prow = 0, pcol = 0;
  {
    const int rr = (warp << 1) | (lane >> 4), cc = lane & 15;
#pragma unroll
    for (int i = 1; i < 4; ++i) {
      prow |= (uint32_t)kTwPos[(rr * i) & 63] << (8 * i - 8);
      pcol |= (uint32_t)kTwPos[(cc * i) & 63] << (8 * i - 8);
    }
  }
  for (int e = threadIdx.x; e < PLANE; e += 2 * NT)   // once per launch
    *reinterpret_cast<double2*>(sS + 2 * e) = make_double2(__ldg(a.Sre + e), __ldg(a.Sim + e));
  __syncthreads();
  const int64_t stride = 2 * (int64_t)gridDim.x;
  const int64_t p0 = a.win.p_begin + 2 * (int64_t)blockIdx.x + grp;
  if (TMA && tid == 0 && p0 < a.win.p_end) issue_pair(a, &tm, geom(a, p0), sR, &bar[grp]);

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
    const Geom gnext = geom(a, has_next ? p + stride : p);
    tile_passes<TMA>(sR, sI, sS, tw, a, g, warp, lane, grp, &tm, &bar[grp], has_next, gnext, prow, pcol);
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
