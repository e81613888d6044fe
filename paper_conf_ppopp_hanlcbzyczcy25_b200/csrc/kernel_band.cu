// Boundary-band and fixed-ring kernels (sm_100a).
//
// The paper never states a boundary condition (reading Q2); the product keeps a fixed ring
// of width r.  A T-step FFT pass reproduces the direct stencil only on the exact region
// [h, n_a - h) of every axis (reading Q5): cells of the band r <= c_a < h (and the mirror
// band) feel the fixed ring within T steps.  This kernel recomputes the band by t direct
// steps (PAPER.md L93 definition) in shared memory: one CTA per band block loads the block
// grown by r*t on every side (clipped to the grid), steps t times -- ring cells held,
// cells whose neighbourhood leaves the loaded region held (they lie outside the dependency
// cone of every cell written) -- and writes the block.  Blocks partition the band exactly
// (plan.cpp), so every band cell is written once per pass and never overlaps the fused
// kernel's exact-region writes.
#include "kernels.cuh"

#ifndef BAND_LEAN
#define BAND_LEAN 1   // 0: per-cell ring test and index recomputation (the session-2 loop)
#endif
#ifndef BAND_CPASYNC
#define BAND_CPASYNC 1   // 0: synchronous region loads (round-2 kernel, ablation)
#endif
#ifndef BAND_TAPREG
#define BAND_TAPREG 1   // 0: taps always read from shared memory (ablation)
#endif

namespace fstencil {
namespace {

__global__ void __launch_bounds__(kBandThreads) band_kernel(const BandArgs a) {
  extern __shared__ double sb[];
  const int* blk = a.blocks + 8 * blockIdx.x;
  int64_t lo[3], hi[3], rl[3], D[3], off[3] = {0, 0, 0};
  off[a.oax] = a.g0;   // buffers start at global outer-axis row g0
#pragma unroll
  for (int q = 0; q < 3; ++q) {
    lo[q] = blk[q];
    hi[q] = blk[3 + q];
    if (q == a.oax) { lo[q] = max(lo[q], a.clip_lo); hi[q] = min(hi[q], a.clip_hi); }
    const int64_t gq = a.active[q] ? (int64_t)a.r * a.t : 0;
    int64_t l = max((int64_t)0, lo[q] - gq), u = min(a.n[q], hi[q] + gq);
    if (q == a.oax) { l = max(l, a.g0); u = min(u, a.g0 + a.gn); }
    rl[q] = l;
    D[q] = u - l;
  }
  if (hi[a.oax] <= lo[a.oax]) return;   // block outside the clip rows (whole CTA)
  const int64_t vol = D[0] * D[1] * D[2];
  double* b0 = sb;
  double* b1 = sb + vol;
  for (int64_t e = threadIdx.x; e < vol; e += blockDim.x) {
    const int64_t i2 = e % D[2], i1 = (e / D[2]) % D[1], i0 = e / (D[1] * D[2]);
    b0[e] = a.src[((rl[0] + i0 - off[0]) * a.n[1] + (rl[1] + i1 - off[1])) * a.n[2] + (rl[2] + i2 - off[2])];
  }
  __syncthreads();
  const int r = a.r, wd = 2 * r + 1;
  const int lo0 = a.active[0] ? -r : 0, lo1 = a.active[1] ? -r : 0, lo2 = a.active[2] ? -r : 0;
  const int hi0 = -lo0, hi1 = -lo1, hi2 = -lo2;
  for (int s = 0; s < a.t; ++s) {
    for (int64_t e = threadIdx.x; e < vol; e += blockDim.x) {
      const int64_t i2 = e % D[2], i1 = (e / D[2]) % D[1], i0 = e / (D[1] * D[2]);
      const int64_t ii[3] = {i0, i1, i2};
      bool keep = false;
#pragma unroll
      for (int q = 0; q < 3; ++q) {
        if (!a.active[q]) continue;
        const int64_t c = rl[q] + ii[q];
        keep |= (c < r) || (c >= a.n[q] - r);                 // fixed ring
        keep |= (ii[q] < r) || (ii[q] + r >= D[q]);           // region edge
      }
      double v;
      if (keep) {
        v = b0[e];
      } else {
        v = 0.0;
        int k = 0;
        for (int o0 = lo0; o0 <= hi0; ++o0)
          for (int o1 = lo1; o1 <= hi1; ++o1)
            for (int o2 = lo2; o2 <= hi2; ++o2, ++k) {
              const double wv = __ldg(a.w + k);
              v = fma(wv, b0[((i0 + o0) * D[1] + (i1 + o1)) * D[2] + (i2 + o2)], v);
            }
      }
      b1[e] = v;
    }
    __syncthreads();
    double* t = b0; b0 = b1; b1 = t;
  }
  (void)wd;
  const int64_t O1 = hi[1] - lo[1], O2 = hi[2] - lo[2];
  const int64_t ovol = (hi[0] - lo[0]) * O1 * O2;
  for (int64_t e = threadIdx.x; e < ovol; e += blockDim.x) {
    const int64_t j2 = e % O2, j1 = (e / O2) % O1, j0 = e / (O1 * O2);
    const int64_t c0 = lo[0] + j0, c1 = lo[1] + j1, c2 = lo[2] + j2;
    a.dst[((c0 - off[0]) * a.n[1] + (c1 - off[1])) * a.n[2] + (c2 - off[2])] =
        b0[((c0 - rl[0]) * D[1] + (c1 - rl[1])) * D[2] + (c2 - rl[2])];
  }
}

// Faster band kernel: the block's nonzero taps are compacted into shared memory with their
// flattened region offsets; at step s only the dependency cone of the output block is
// updated (distance >= r*s from every region edge that is not the grid boundary -- the
// cells outside it are never read again), and threads map to (row, column) of the region
// without per-cell divisions.  Same definition and result as band_kernel.
constexpr int kMaxTaps = 512;

// x / d for 0 <= x < 2^20, d >= 1 (block-geometry indices): a float reciprocal estimate (relative
// error ~2^-21, so at most one off) and one correction step -- ~9 instructions instead of the
// ~25 of a 32-bit integer division; a 3D band block does ~16 of them per warp (ncu: the
// per-block index setup was ~40 % of the band kernel's instructions, profiles/r02_band_async_ncu.txt).
#ifndef BAND_FDIV
#define BAND_FDIV 1   // 0: integer division (ablation)
#endif
__device__ __forceinline__ int fdiv(int x, int d) {
#if BAND_FDIV
  int q = __float2int_rz(__fdividef((float)x, (float)d));
  const int r = x - q * d;
  q += (r >= d) - (r < 0);
  return q;
#else
  return x / d;
#endif
}

// NTH = 256, (256, 6): at most 40 registers (one band CTA fits beside the DMMA engines' fused
// CTAs); NTH = 1024 for the 1D band, whose two blocks run t (~1000) sequential steps on SMs
// the fused kernel leaves free (capi.cu), so per-step latency is what counts.
// NTAPS > 0: the stencil has exactly NTAPS nonzero taps (host-counted); the lean cone loop then
// keeps offsets and weights in registers, fully unrolled (no shared-memory tap loads, no loop).
// PEER: the launch holds boundary rows of a peer-transport rank; their cells are also stored into the
// neighbour's halo rows (a.peer) -- a separate instantiation, the store loop of the others is unchanged.
template <int NTH, int NTAPS = 0, bool PEER = false>
__global__ void __launch_bounds__(NTH, NTH == 256 ? 6 : 1) band_cone_kernel(const BandArgs a) {
  extern __shared__ double sb[];
  __shared__ int s_off[kMaxTaps];
  __shared__ double s_w[kMaxTaps];
  __shared__ int s_ntaps;
  const int* blk = a.blocks + 8 * blockIdx.x;
  int64_t lo[3], hi[3], rl[3], off[3] = {0, 0, 0};
  int D[3], clo[3], chi[3];
  bool open_lo[3], open_hi[3];
  off[a.oax] = a.g0;
#pragma unroll
  for (int q = 0; q < 3; ++q) {
    lo[q] = blk[q];
    hi[q] = blk[3 + q];
    if (q == a.oax) { lo[q] = max(lo[q], a.clip_lo); hi[q] = min(hi[q], a.clip_hi); }
    const int64_t gq = a.active[q] ? (int64_t)a.r * a.t : 0;
    int64_t l = max((int64_t)0, lo[q] - gq), u = min(a.n[q], hi[q] + gq);
    if (q == a.oax) { l = max(l, a.g0); u = min(u, a.g0 + a.gn); }
    rl[q] = l;
    D[q] = (int)(u - l);
    open_lo[q] = a.active[q] && l > 0;               // cells below were not loaded
    open_hi[q] = a.active[q] && u < a.n[q];
  }
  if (hi[a.oax] <= lo[a.oax]) return;   // block outside the clip rows (whole CTA)
  const int r = a.r, wd = 2 * r + 1;
  // Tap table: the nonzero weights in offset-cube order (the summation order of every cell, so
  // results stay bitwise equal to the reference band kernel) with their flattened region
  // offsets.  Warp 0 builds it 32 weights at a time (ballot + prefix count): one thread's loop
  // of dependent global loads cost microseconds per block, and a 3D band is tens of thousands
  // of small blocks (profiles/r02_band3d.txt).
  const int W1 = a.active[1] ? wd : 1, W2 = a.active[2] ? wd : 1;
  const int nw = (a.active[0] ? wd : 1) * W1 * W2;
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    int base = 0;
    for (int k0 = 0; k0 < nw; k0 += 32) {
      const int k = k0 + lane;
      const double wv = k < nw ? a.w[k] : 0.0;
      const unsigned m = __ballot_sync(0xffffffffu, wv != 0.0);
      if (wv != 0.0) {
        const int pos = base + __popc(m & ((1u << lane) - 1u));
        if (pos < kMaxTaps) {
          const int kq = fdiv(k, W2), i2 = k - kq * W2, i0 = fdiv(kq, W1), i1 = kq - i0 * W1;
          const int o0 = a.active[0] ? i0 - r : 0, o1 = a.active[1] ? i1 - r : 0, o2 = a.active[2] ? i2 - r : 0;
          s_off[pos] = (o0 * D[1] + o1) * D[2] + o2;
          s_w[pos] = wv;
        }
      }
      base += __popc(m);
    }
    if (lane == 0) s_ntaps = min(base, kMaxTaps);
  }
  const int vol = D[0] * D[1] * D[2];
  double* b0 = sb;
  double* b1 = sb + vol;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5, ny = NTH / 32;
  {
    // region load, flattened over all threads (thin faces have rows of a few cells: a warp per
    // row left most lanes idle); (i0, i1, i2) advanced by carries
    const int D12 = D[1] * D[2];
    int i0 = fdiv(threadIdx.x, D12), i1 = fdiv(threadIdx.x - i0 * D12, D[2]), i2 = threadIdx.x - i0 * D12 - i1 * D[2];
    const int d0 = fdiv(NTH, D12), d1 = fdiv(NTH - d0 * D12, D[2]), d2 = NTH - d0 * D12 - d1 * D[2];
    const double* src0 = a.src + ((rl[0] - off[0]) * a.n[1] + (rl[1] - off[1])) * a.n[2] + (rl[2] - off[2]);
    for (int e = threadIdx.x; e < vol; e += NTH) {
      const double* gp = src0 + ((int64_t)i0 * a.n[1] + i1) * a.n[2] + i2;
      if (BAND_CPASYNC) {
        // asynchronous 8-byte copies: a thread's ~14 region loads are all in flight at once
        // (the synchronous loop waited one global-load latency per cell: ncu long_scoreboard)
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"((unsigned)__cvta_generic_to_shared(b0 + e)),
                     "l"(gp));
      } else {
        const double v = *gp;
        b0[e] = v;
        if (BAND_LEAN) b1[e] = v;   // the fixed ring lives in both buffers
      }
      i2 += d2;
      i1 += d1;
      i0 += d0;
      if (i2 >= D[2]) { i2 -= D[2]; ++i1; }
      if (i1 >= D[1]) { i1 -= D[1]; ++i0; }
    }
    if (BAND_CPASYNC) {
      asm volatile("cp.async.commit_group;\n" ::);
      asm volatile("cp.async.wait_all;\n" ::: "memory");
      // a thread's own copies are visible to it after the wait: the fixed ring goes to b1 too
      if (BAND_LEAN)
        for (int e = threadIdx.x; e < vol; e += NTH) b1[e] = b0[e];
    }
  }
  __syncthreads();
  const int ntaps = s_ntaps;
  // fixed-ring bounds in region-local coordinates (inactive axes never hit)
  int rlo[3], rhi[3];
#pragma unroll
  for (int q = 0; q < 3; ++q) {
    rlo[q] = a.active[q] ? (int)(r - rl[q]) : -(1 << 30);
    rhi[q] = a.active[q] ? (int)(a.n[q] - r - rl[q]) : (1 << 30);
  }
#ifndef BAND_ROWS
#define BAND_ROWS 0   // 1: a warp per cone row for 2D / 3D wide rows (measured slower, ablation)
#endif
  const bool rows_ok = BAND_ROWS && a.active[1] && a.active[2];   // 2D and 3D (not 1D)
  for (int s = 1; s <= a.t; ++s) {
#pragma unroll
    for (int q = 0; q < 3; ++q) {
      clo[q] = open_lo[q] ? r * s : 0;
      chi[q] = D[q] - (open_hi[q] ? r * s : 0);
    }
    const int W0 = chi[0] - clo[0], W1 = chi[1] - clo[1], W2 = chi[2] - clo[2];
    if (rows_ok && W2 >= 16) {
      // 2D / 3D blocks whose cone rows (axis 2) are >= 16 cells: a warp per cone row, lanes
      // along the row; the ring test is per row plus a column range, the cell index one add --
      // the flattened form below spends ~50 integer instructions per FMA on index bookkeeping
      // (ncu, profiles/r01_s3_band2d_ncu.txt), yet this form measured slower (band 95 -> 114 us
      // per Heat-2D launch, profiles/r01_s3_ab_band.txt), so it is an ablation only.
      for (int row = ty; row < W0 * W1; row += ny) {
        const int k0 = row / W1, k1 = row - k0 * W1;
        const int i0 = clo[0] + k0, i1 = clo[1] + k1;
        const bool ring_row = i0 < rlo[0] || i0 >= rhi[0] || i1 < rlo[1] || i1 >= rhi[1];
        const int c_lo = ring_row ? W2 : max(0, rlo[2] - clo[2]), c_hi = ring_row ? W2 : min(W2, rhi[2] - clo[2]);
        const int rowbase = (i0 * D[1] + i1) * D[2] + clo[2];
        for (int k2 = tx; k2 < W2; k2 += 32) {
          const int e = rowbase + k2;
          double v;
          if (k2 < c_lo || k2 >= c_hi) {
            v = b0[e];                                      // fixed ring
          } else {
            v = 0.0;
#pragma unroll 4
            for (int k = 0; k < ntaps; ++k) v = fma(s_w[k], b0[e + s_off[k]], v);
          }
          b1[e] = v;
        }
      }
      __syncthreads();
      double* t = b0; b0 = b1; b1 = t;
      continue;
    }
    if (BAND_LEAN) {
      // The cone box clipped to the interior (ring cells sit unchanged in both buffers, so no
      // per-cell ring test) and the cell index advanced incrementally with the carries: ~3x
      // fewer integer instructions per cell than the loop below (which ncu showed issue-bound
      // at ~50 integer instructions per FMA).  Same cells, same tap order: bitwise equal.
      int lo3[3], w3[3];
#pragma unroll
      for (int q = 0; q < 3; ++q) {
        lo3[q] = max(clo[q], rlo[q]);
        w3[q] = min(chi[q], rhi[q]) - lo3[q];
      }
      if (w3[0] > 0 && w3[1] > 0 && w3[2] > 0) {
        const int V12 = w3[1] * w3[2], nc = w3[0] * V12;
        int j0 = fdiv(threadIdx.x, V12), j1 = fdiv(threadIdx.x - j0 * V12, w3[2]);
        int j2 = threadIdx.x - j0 * V12 - j1 * w3[2];
        const int e0 = fdiv(NTH, V12), e1 = fdiv(NTH - e0 * V12, w3[2]);
        const int e2 = NTH - e0 * V12 - e1 * w3[2];
        const int D12 = D[1] * D[2];
        const int de = e2 + e1 * D[2] + e0 * D12;       // index step per NTH cells, before carries
        const int c2 = D[2] - w3[2], c1 = (D[1] - w3[1]) * D[2];
        int e = (lo3[0] + j0) * D12 + (lo3[1] + j1) * D[2] + lo3[2] + j2;
        constexpr int NR = NTAPS > 0 ? NTAPS : 1;
        double wr[NR];
        int orr[NR];
#pragma unroll
        for (int k = 0; k < NR; ++k) {
          wr[k] = NTAPS > 0 ? s_w[k] : 0.0;
          orr[k] = NTAPS > 0 ? s_off[k] : 0;
        }
        for (int f = threadIdx.x; f < nc; f += NTH) {
          double v = 0.0;
          if (NTAPS > 0) {
#pragma unroll
            for (int k = 0; k < NR; ++k) v = fma(wr[k], b0[e + orr[k]], v);
          } else {
#pragma unroll 4
            for (int k = 0; k < ntaps; ++k) v = fma(s_w[k], b0[e + s_off[k]], v);
          }
          b1[e] = v;
          j2 += e2;
          j1 += e1;
          j0 += e0;
          e += de;
          if (j2 >= w3[2]) { j2 -= w3[2]; ++j1; e += c2; }
          if (j1 >= w3[1]) { j1 -= w3[1]; ++j0; e += c1; }
        }
      }
      __syncthreads();
      double* t = b0; b0 = b1; b1 = t;
      continue;
    }
    // cone box of this step, flattened over all threads (no idle lanes on narrow faces);
    // the (k0, k1, k2) decomposition is advanced by carries, not recomputed by divisions
    const int W12 = W1 * W2, ncone = W0 * W12;
    int k0 = fdiv(threadIdx.x, W12), k1 = fdiv(threadIdx.x - k0 * W12, W2);
    int k2 = threadIdx.x - k0 * W12 - k1 * W2;
    const int d0 = fdiv(NTH, W12), d1 = fdiv(NTH - d0 * W12, W2);
    const int d2 = NTH - d0 * W12 - d1 * W2;
    for (int f = threadIdx.x; f < ncone; f += NTH) {
      const int i0 = clo[0] + k0, i1 = clo[1] + k1, i2 = clo[2] + k2;
      const int e = (i0 * D[1] + i1) * D[2] + i2;
      double v;
      if (i0 < rlo[0] || i0 >= rhi[0] || i1 < rlo[1] || i1 >= rhi[1] || i2 < rlo[2] || i2 >= rhi[2]) {
        v = b0[e];                                          // fixed ring
      } else {
        v = 0.0;
#pragma unroll 4
        for (int k = 0; k < ntaps; ++k) v = fma(s_w[k], b0[e + s_off[k]], v);
      }
      b1[e] = v;
      k2 += d2;
      k1 += d1;
      k0 += d0;
      if (k2 >= W2) { k2 -= W2; ++k1; }
      if (k1 >= W1) { k1 -= W1; ++k0; }
    }
    __syncthreads();
    double* t = b0; b0 = b1; b1 = t;
  }
  // output store, flattened like the load (a face block of axis 2 has one-cell rows)
  const int O0 = (int)(hi[0] - lo[0]), O1 = (int)(hi[1] - lo[1]), O2 = (int)(hi[2] - lo[2]);
  const int O12 = O1 * O2, ovol = O0 * O12;
  int j0 = fdiv(threadIdx.x, O12), j1 = fdiv(threadIdx.x - j0 * O12, O2), j2 = threadIdx.x - j0 * O12 - j1 * O2;
  const int f0 = fdiv(NTH, O12), f1 = fdiv(NTH - f0 * O12, O2), f2 = NTH - f0 * O12 - f1 * O2;
  double* dst0 = a.dst + ((lo[0] - off[0]) * a.n[1] + (lo[1] - off[1])) * a.n[2] + (lo[2] - off[2]);
  const double* sb0 = b0 + ((lo[0] - rl[0]) * D[1] + (lo[1] - rl[1])) * D[2] + (lo[2] - rl[2]);
  // peer transport: cells of the rank's boundary rows also go to the neighbour's halo rows
  for (int e = threadIdx.x; e < ovol; e += NTH) {
    const double v = sb0[(j0 * D[1] + j1) * D[2] + j2];
    dst0[((int64_t)j0 * a.n[1] + j1) * a.n[2] + j2] = v;
    if (PEER) {
      int64_t c[3] = {lo[0] + j0, lo[1] + j1, lo[2] + j2};
      const int64_t row = c[a.oax];
      double* pb = row < a.peer.lo_end ? a.peer.lo : row >= a.peer.hi_begin ? a.peer.hi : nullptr;
      if (pb) {
        c[a.oax] = row - (row < a.peer.lo_end ? a.peer.lo_g0 : a.peer.hi_g0);
        pb[(c[0] * a.n[1] + c[1]) * a.n[2] + c[2]] = v;
      }
    }
    j2 += f2;
    j1 += f1;
    j0 += f0;
    if (j2 >= O2) { j2 -= O2; ++j1; }
    if (j1 >= O1) { j1 -= O1; ++j0; }
  }
  (void)tx;
  (void)ty;
  (void)ny;
}

__global__ void box_copy_kernel(const BoxCopyArgs a) {
  const int64_t L0 = a.hi[0] - a.lo[0], L1 = a.hi[1] - a.lo[1], L2 = a.hi[2] - a.lo[2];
  const int64_t vol = L0 * L1 * L2;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < vol; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j2 = e % L2, j1 = (e / L2) % L1, j0 = e / (L1 * L2);
    int64_t c[3] = {a.lo[0] + j0, a.lo[1] + j1, a.lo[2] + j2};
    int64_t d[3] = {c[0], c[1], c[2]};
    c[a.oax] -= a.src_off;
    d[a.oax] -= a.dst_off;
    const double v = a.src[(c[0] * a.n[1] + c[1]) * a.n[2] + c[2]];
    const int64_t di = (d[0] * a.n[1] + d[1]) * a.n[2] + d[2];
    if (a.dst0) a.dst0[di] = v;
    if (a.dst1) a.dst1[di] = v;
  }
}

}  // namespace

// The max-dynamic-shared-memory attribute belongs to the function, not to a plan: set it to
// the device limit once (minus each kernel's static shared memory) so plans of different
// band sizes coexist, and refuse a plan whose band region does not fit.
cudaError_t band_configure(size_t smem) {
  int dev = 0, optin = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  if (e != cudaSuccess) return e;
  cudaFuncAttributes fa;
  if ((e = cudaFuncGetAttributes(&fa, band_kernel)) != cudaSuccess) return e;
  const size_t lim0 = (size_t)optin - fa.sharedSizeBytes;
  if ((e = cudaFuncSetAttribute(band_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lim0)) != cudaSuccess)
    return e;
  if ((e = cudaFuncGetAttributes(&fa, band_cone_kernel<256>)) != cudaSuccess) return e;
  const size_t lim1 = (size_t)optin - fa.sharedSizeBytes;
  if ((e = cudaFuncSetAttribute(band_cone_kernel<256, 5>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lim1)) !=
      cudaSuccess ||
      (e = cudaFuncSetAttribute(band_cone_kernel<256, 7>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lim1)) !=
      cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(band_cone_kernel<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lim1)) !=
      cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(band_cone_kernel<256, 5, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)lim1)) != cudaSuccess ||
      (e = cudaFuncSetAttribute(band_cone_kernel<256, 7, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)lim1)) != cudaSuccess ||
      (e = cudaFuncSetAttribute(band_cone_kernel<256, 0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)lim1)) != cudaSuccess ||
      (e = cudaFuncSetAttribute(band_cone_kernel<1024, 0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)lim1)) != cudaSuccess ||
      (e = cudaFuncSetAttribute(band_cone_kernel<64, 0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)lim1)) != cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(band_cone_kernel<1024>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lim1)) !=
      cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(band_cone_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lim1)) !=
      cudaSuccess)
    return e;
  return smem <= lim0 && smem <= lim1 ? cudaSuccess : cudaErrorInvalidValue;
}

template <bool PEER>
void launch_cone(const BandArgs& a, size_t smem, cudaStream_t s, bool one_d) {
  // 1D: 1024 threads for the long bands of deep-fusion plans (t ~ 1000 sequential steps over
  // thousands of cells); a 64-thread CTA when the region is small (e.g. configs[0]: 23 cells,
  // where 32 mostly idle warps spent ~150 issue slots each per step: 15 us vs ~3 us)
  if (one_d && a.region_cells > 512)
    band_cone_kernel<1024, 0, PEER><<<a.nblocks, 1024, smem, s>>>(a);
  else if (one_d)
    band_cone_kernel<64, 0, PEER><<<a.nblocks, 64, smem, s>>>(a);
  else
    // register-resident taps for 5- and 7-point stars (9 taps spill at the 40-register budget
    // and measured 0.4% slower, profiles/r01_s3_ab_band_tapreg.txt)
    switch (BAND_LEAN && BAND_TAPREG ? a.ntaps : 0) {
      case 5: band_cone_kernel<256, 5, PEER><<<a.nblocks, kBandThreads, smem, s>>>(a); break;
      case 7: band_cone_kernel<256, 7, PEER><<<a.nblocks, kBandThreads, smem, s>>>(a); break;
      default: band_cone_kernel<256, 0, PEER><<<a.nblocks, kBandThreads, smem, s>>>(a);
    }
}

cudaError_t launch_band(const BandArgs& a, size_t smem, cudaStream_t s) {
  if (a.nblocks <= 0) return cudaSuccess;
  int taps = 1;
  for (int q = 0; q < 3; ++q) taps *= a.active[q] ? 2 * a.r + 1 : 1;
  const bool one_d = a.active[0] + a.active[1] + a.active[2] == 1;
  if (taps <= kMaxTaps && !a.reference) {
    if (a.peer.lo || a.peer.hi)
      launch_cone<true>(a, smem, s, one_d);
    else
      launch_cone<false>(a, smem, s, one_d);
  } else {
    band_kernel<<<a.nblocks, kBandThreads, smem, s>>>(a);
  }
  return cudaGetLastError();
}

cudaError_t launch_box_copy(const BoxCopyArgs& a, cudaStream_t s) {
  const int64_t vol = (a.hi[0] - a.lo[0]) * (a.hi[1] - a.lo[1]) * (a.hi[2] - a.lo[2]);
  if (vol <= 0) return cudaSuccess;
  int64_t grid = (vol + 255) / 256;
  if (grid > 4096) grid = 4096;
  box_copy_kernel<<<(int)grid, 256, 0, s>>>(a);
  return cudaGetLastError();
}

}  // namespace fstencil
