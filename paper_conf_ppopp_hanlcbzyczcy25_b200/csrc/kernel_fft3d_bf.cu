// Fused 3D FFT-stencil tile kernel with register-resident radix-4 FFTs on the FP64 ALU
// (sm_100a).  One thread owns one whole 16-point line per pass.
//
// Same fused pass as kernel_fft3d_ct.cu (Algorithm 1 L252-L258 on 16^3 overlap-save
// tiles, Double-layer Filling Eq. 9, temporal fusion Eq. 10, Stitching Eq. 7; 3D handled axis
// by axis as in §3.2.1), with each length-16 axis DFT evaluated as a 4 x 4 Cooley-Tukey
// FFT in registers (fft_radix.cuh: 160 FP64 instructions per line) instead of DFT-8 GEMMs on
// the tensor pipe (kernel_fft3d_ct.cu: 8 DMMA.8x8x4 = 2048 FMA per 4 lines, i.e. ~512 FP64
// pipe operations per line on a pipe B200 shares between DMMA and DFMA).
//
// Per tile pair, five shared-memory passes, each thread reading one line and rewriting it in
// place (no intra-pass exchange):
//   P1 forward axis 2 | P2 forward axis 1 | P3 forward axis 0, * S_T, inverse axis 0 (writes
//   only the S output planes) | P4 inverse axis 1 on those planes (writes only the S output
//   rows) | P5 inverse axis 2 on the S x S output rows -> store the S^3 window.
// Shared layout: the tiles land as the TMA SWIZZLE_128B image of two dense 16^3 boxes (Re and
// Im planes; element (l0, l1, l2) at word 256 l0 + 16 l1 + (l2 ^ 2 (l1 & 7))); P1 reads each
// row from both planes (16-byte words, lanes l1 = 0..7 per quarter-warp: conflict-free) and
// rewrites it in place in an interleaved complex layout (cofs below) that every later pass
// reads and writes as one 16-byte word per element.  S_T is staged once per launch in shared
// memory, interleaved, natural [k0][k1][k2] order.
#include "fft_radix.cuh"
#include "kernels.cuh"
#include "tma.cuh"

namespace fstencil {
namespace {

constexpr int L = 16;
constexpr int PLANE = L * L * L;
constexpr int NT = 256;                 // threads per CTA: one per line of a full pass
constexpr int kAlign = 1024;            // SWIZZLE_128B destinations are 1024-byte aligned

__device__ __forceinline__ int wofs(int l0, int l1, int l2) { return (l0 << 8) | (l1 << 4) | (l2 ^ ((l1 & 7) << 1)); }

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

// Row lines (along l2) at row (l0, l1): 16-byte chunk c holds l2 = 2c, 2c + 1 at chunk c ^ (l1 & 7).
__device__ __forceinline__ void load_row(const double* sR, const double* sI, int l0, int l1, double (&xr)[16],
                                         double (&xi)[16]) {
  const int base = (l0 << 8) | (l1 << 4), s = l1 & 7;
#pragma unroll
  for (int c = 0; c < 8; ++c) {
    const int o = base + ((c ^ s) << 1);
    const double2 r = *reinterpret_cast<const double2*>(sR + o);
    const double2 i = *reinterpret_cast<const double2*>(sI + o);
    xr[2 * c] = r.x; xr[2 * c + 1] = r.y;
    xi[2 * c] = i.x; xi[2 * c + 1] = i.y;
  }
}
// Interleaved complex layout used after P1 (double2 (re, im) per element, one 16-byte word):
// element (l0, l1, l2) of a group buffer sits in region l2 >> 3 (the bytes of the Re / Im
// plane's row (l0, l1)), 16-byte chunk (l2 & 7) ^ (l1 & 7) of that row.  P1 converts each row
// in place (a thread owns both planes' 128-byte rows of its row); every later access is one
// 16-byte word per element, conflict-free per quarter-warp (lanes = 8 consecutive l2 or l1).
__device__ __forceinline__ int cofs(int l0, int l1, int l2) {
  return ((l2 >> 3) << 12) | (l0 << 8) | (l1 << 4) | (((l2 & 7) ^ (l1 & 7)) << 1);
}
__device__ __forceinline__ double2 ldc(const double* b, int o) { return *reinterpret_cast<const double2*>(b + o); }
__device__ __forceinline__ void stc(double* b, int o, double re, double im) {
  *reinterpret_cast<double2*>(b + o) = make_double2(re, im);
}

// Barrier of one 256-thread group (ids 1, 2; id 0 is __syncthreads).
__device__ __forceinline__ void group_sync(int grp) { asm volatile("bar.sync %0, %1;\n" ::"r"(grp + 1), "r"(NT) : "memory"); }

// 256-bit global store (sm_100): four doubles at a 32-byte aligned address, one whole sector.
__device__ __forceinline__ void st256(double* p, double a, double b, double c, double d) {
  asm volatile("st.global.v4.f64 [%0], {%1, %2, %3, %4};\n" ::"l"(p), "d"(a), "d"(b), "d"(c), "d"(d) : "memory");
}

struct PairGeom {
  int64_t o0, o1, oa2, ob2;
  bool has_b;
};
// p is the launch's traversal index in [p_begin, p_end) (whole outer tile rows): in natural order
// it is the pair index itself; with blk0 > 0 the launch visits blocks of blk0 outer tile rows x
// blk1 tile lines (all pairs of each line), block rows in order, so the tiles whose halo planes
// / rows overlap are transformed close together in time and the overlap is re-read from L2 (a
// 1024^3 outer tile row of 16-plane tiles is 134 MB, more than the 126 MB L2: in natural order the
// next row's four overlapping planes come back from HBM).
__device__ __forceinline__ PairGeom pair_geom(const Fft3dArgs& a, int64_t p) {
  // pair / tile indices fit 32 bits (the plan's pair count is far below 2^31)
  const int S = a.S, npr = (int)a.npr, nt1 = (int)a.nt1;
  int t0, t1, pj;
  if (a.blk0 > 0) {
    const int ppu = nt1 * npr, u0 = (int)(a.win.p_begin / ppu), nu = (int)((a.win.p_end - a.win.p_begin) / ppu);
    const int q = (int)(p - a.win.p_begin);
    const int b0 = q / (a.blk0 * ppu);                       // block row (outer tile rows)
    const int s0 = min(a.blk0, nu - b0 * a.blk0);            // its height (last one partial)
    const int q1 = q - b0 * a.blk0 * ppu;
    const int b1 = q1 / (s0 * a.blk1 * npr);                 // block within the row (tile lines)
    const int s1 = min(a.blk1, nt1 - b1 * a.blk1);
    const int q2 = q1 - b1 * s0 * a.blk1 * npr;
    pj = q2 % npr;
    const int r = q2 / npr;                                  // (t0, t1) within the block, t1 fastest
    t0 = u0 + b0 * a.blk0 + r / s1;
    t1 = b1 * a.blk1 + r % s1;
  } else {
    const int pi = (int)p;
    const int line = pi / npr;
    pj = pi - line * npr;
    t0 = line / nt1;
    t1 = line - t0 * nt1;
  }
  PairGeom g;
  g.o0 = (int64_t)t0 * S + a.bd.shift;
  g.o1 = (int64_t)t1 * S + a.bd.shift;
  g.oa2 = (int64_t)2 * pj * S + a.bd.shift;
  g.ob2 = g.oa2 + S;
  g.has_b = 2 * pj + 1 < a.nt2;
  return g;
}

// One CTA per SM = two independent 256-thread groups, each transforming its own sequence of
// tile pairs in its own 64 KB buffer (the other group's work hides a group's TMA latency and
// barrier waits); S_T (64 KB) is staged once and shared: 192 KB.  Thread t of a group owns
// line (t >> 4, t & 15) of every pass, so a warp's P1 rows and P2 lines lie in the same two
// l0-planes (P1 -> P2 needs only __syncwarp), and likewise P4 -> P5 on the output planes.
// TMA = false: cp.async loads (periodic wrap-around, or a pitch TMA cannot describe).
// PEER: the launch holds boundary rows of a peer-transport rank (a.peer, kernels.cuh): its output
// rows within h of the slab edge are stored into the neighbour's buffer too (a separate
// instantiation, so the single-GPU kernel's code and registers are untouched).
template <bool TMA, bool WRAP = false, bool PEER = false>
__global__ void __launch_bounds__(2 * NT, 1) fft3d_bf_kernel(const Fft3dArgs a, const __grid_constant__ CUtensorMap tm) {
  extern __shared__ unsigned char smem_raw[];
  const uint32_t mis = tma::smem_addr(smem_raw) & (kAlign - 1);
  double* base = reinterpret_cast<double*>(smem_raw + (mis ? kAlign - mis : 0));   // stays in the shared window
  double* sS = base + 4 * PLANE;   // S_T interleaved (re, im), natural [k0][k1][k2]
  __shared__ __align__(8) uint64_t bar[2];
  const int grp = threadIdx.x >> 8, tid = threadIdx.x & (NT - 1);
  const int hi = tid >> 4, lo = tid & 15;
  const int S = a.S, h = a.h;
  double* sR = base + grp * 2 * PLANE;
  double* sI = sR + PLANE;
  if (threadIdx.x == 0) {
    tma::mbar_init(&bar[0], 1);
    tma::mbar_init(&bar[1], 1);
  }
  for (int e = threadIdx.x; e < PLANE; e += 2 * NT) stc(sS, 2 * e, __ldg(a.Sre + e), __ldg(a.Sim + e));   // once per launch
  __syncthreads();
  const int64_t stride = 2 * (int64_t)gridDim.x;
  const int64_t p0 = a.win.p_begin + 2 * (int64_t)blockIdx.x + grp;
  // TMA box origins of a group's next pair (x = axis 2 of tile a, y, z, x of tile b or -1), computed
  // by the issuing thread at the top of an iteration, when few registers are live: the refill is
  // issued mid-transform, with the 32 line registers live
  __shared__ int nxt[2][4];
  auto prepare = [&](int64_t p) {
    const PairGeom g = pair_geom(a, p);
    nxt[grp][0] = (int)g.oa2;
    nxt[grp][1] = (int)g.o1;
    nxt[grp][2] = (int)(g.o0 - a.win.g0);
    nxt[grp][3] = g.has_b ? (int)g.ob2 : INT32_MIN;
  };
  auto issue = [&]() {
    const int x = nxt[grp][0], y = nxt[grp][1], z = nxt[grp][2], xb = nxt[grp][3];
    tma::mbar_expect_tx(&bar[grp], (xb != INT32_MIN ? 2u : 1u) * PLANE * 8u);
    tma::load_3d(sR, &tm, x, y, z, &bar[grp]);
    if (xb != INT32_MIN) tma::load_3d(sI, &tm, xb, y, z, &bar[grp]);
  };
  if (TMA && tid == 0 && p0 < a.win.p_end) {
    prepare(p0);
    issue();
  }

  // iteration count form of the pair loop (measured ~1-2 % faster than `for (p = p0; p < end;
  // p += stride)`, same work: the compiler schedules the counted loop better)
  const int64_t nmine = p0 < a.win.p_end ? (a.win.p_end - p0 + stride - 1) / stride : 0;
  uint32_t parity = 0;
  for (int64_t it = 0; it < nmine; ++it) {
    const int64_t p = p0 + it * stride;
    const PairGeom g = pair_geom(a, p);
    if (TMA) {
      if (tid == 0 && p + stride < a.win.p_end) prepare(p + stride);
      tma::mbar_wait(&bar[grp], parity);
      parity ^= 1;
      if (!g.has_b) {
        for (int e = tid; e < PLANE; e += NT) sI[e] = 0.0;
        group_sync(grp);
      }
    } else {
      for (int e = tid; e < 2 * PLANE; e += NT) {
        const int t = e >> 12, l0 = (e >> 8) & 15, l1 = (e >> 4) & 15, l2 = e & 15;
        int64_t g0 = g.o0 + l0, g1 = g.o1 + l1, g2 = (t ? g.ob2 : g.oa2) + l2;
        if (WRAP) { g0 = wrap_index(g0, a.n0); g1 = wrap_index(g1, a.n1); g2 = wrap_index(g2, a.n2); }
        const int64_t lg0 = g0 - a.win.g0;
        const bool valid = (t == 0 || g.has_b) && g0 < a.n0 && lg0 >= 0 && lg0 < a.win.gn && g1 >= 0 && g1 < a.n1 &&
                           g2 >= 0 && g2 < a.n2;
        cp_async8((t ? sI : sR) + wofs(l0, l1, l2), valid ? a.src + (lg0 * a.n1 + g1) * a.n2 + g2 : a.src, valid);
      }
      asm volatile("cp.async.commit_group;\n" ::);
      asm volatile("cp.async.wait_all;\n" ::: "memory");
      group_sync(grp);
    }
    double xr[16], xi[16];
    // ---- P1: forward axis 2 (thread = row (l0, l1) = (hi, lo)); TMA planes -> interleaved ----
    load_row(sR, sI, hi, lo, xr, xi);
    radix::fft16<false>(xr, xi);
#pragma unroll
    for (int l2 = 0; l2 < 16; ++l2) stc(sR, cofs(hi, lo, l2), xr[l2], xi[l2]);
    __syncwarp();
    // ---- P2: forward axis 1 (thread = (l0, l2) = (hi, lo)); same planes as the warp's P1 rows ----
#pragma unroll
    for (int l1 = 0; l1 < 16; ++l1) {
      const double2 v = ldc(sR, cofs(hi, l1, lo));
      xr[l1] = v.x;
      xi[l1] = v.y;
    }
    radix::fft16<false>(xr, xi);
#pragma unroll
    for (int l1 = 0; l1 < 16; ++l1) stc(sR, cofs(hi, l1, lo), xr[l1], xi[l1]);
    group_sync(grp);
    // ---- P3: forward axis 0, * S_T, inverse axis 0 (thread = (k1, k2) = (hi, lo)) ----
    {
      const int b = cofs(0, hi, lo);
#pragma unroll
      for (int l0 = 0; l0 < 16; ++l0) {
        const double2 v = ldc(sR, b + (l0 << 8));
        xr[l0] = v.x;
        xi[l0] = v.y;
      }
      radix::fft16<false>(xr, xi);
#pragma unroll
      for (int k0 = 0; k0 < 16; ++k0) {
        const double2 sv = ldc(sS, ((k0 << 8) + tid) << 1);
        radix::cmul(xr[k0], xi[k0], sv.x, sv.y);
      }
      radix::fft16<true>(xr, xi);
#pragma unroll
      for (int l0 = 0; l0 < 16; ++l0)
        if (l0 >= h && l0 < h + S) stc(sR, b + (l0 << 8), xr[l0], xi[l0]);
    }
    group_sync(grp);
    // ---- P4: inverse axis 1 on the S output planes (thread = (l0 - h, l2)) ----
    if (hi < S) {
#pragma unroll
      for (int l1 = 0; l1 < 16; ++l1) {
        const double2 v = ldc(sR, cofs(h + hi, l1, lo));
        xr[l1] = v.x;
        xi[l1] = v.y;
      }
    }
    if (hi < S) radix::fft16<true>(xr, xi);
    if (hi < S) {
#pragma unroll
      for (int l1 = 0; l1 < 16; ++l1)
        if (l1 >= h && l1 < h + S) stc(sR, cofs(h + hi, l1, lo), xr[l1], xi[l1]);
    }
    __syncwarp();
    // ---- P5: inverse axis 2 on the output rows (thread = (l0 - h, l1 - h)), same planes as P4 ----
    const bool p5 = hi < S && lo < S;
    if (p5) {
#pragma unroll
      for (int l2 = 0; l2 < 16; ++l2) {
        const double2 v = ldc(sR, cofs(h + hi, h + lo, l2));
        xr[l2] = v.x;
        xi[l2] = v.y;
      }
    }
    // the buffer is free: order this thread's shared accesses before the next TMA write, then
    // refill it while the last transform and the stores run
    if (TMA) tma::fence_proxy_async();
    group_sync(grp);
    if (TMA && tid == 0 && p + stride < a.win.p_end) issue();
    if (p5) {
      const int l0 = h + hi, l1 = h + lo;
      radix::fft16<true>(xr, xi);
      const int64_t c0 = g.o0 + l0, c1 = g.o1 + l1;
      if (!(c0 >= a.bd.lim0 || c0 < a.win.w_lo || c0 >= a.win.w_hi || c1 >= a.bd.lim1)) {
        double* drow = a.dst + ((c0 - a.win.g0) * a.n1 + c1) * a.n2;
        // 16-byte stores of (l2, l2 + 1) when the row and window are aligned
        const bool vec = ((g.oa2 | h | a.n2 | S) & 1) == 0 && (reinterpret_cast<uintptr_t>(a.dst) & 15) == 0 &&
                         g.oa2 + h + S <= a.bd.lim2 && (!g.has_b || g.ob2 + h + S <= a.bd.lim2);
        if (vec) {
#pragma unroll
          for (int l2 = 0; l2 < 16; l2 += 2) {
            if ((a.st32 >> l2) & 1) {   // whole 32-byte sectors (launch mask, see Fft3dArgs)
              st256(drow + g.oa2 + l2, xr[l2], xr[l2 + 1], xr[l2 + 2], xr[l2 + 3]);
              if (g.has_b) st256(drow + g.ob2 + l2, xi[l2], xi[l2 + 1], xi[l2 + 2], xi[l2 + 3]);
            } else if ((a.st16 >> l2) & 1) {
              *reinterpret_cast<double2*>(drow + g.oa2 + l2) = make_double2(xr[l2], xr[l2 + 1]);
              if (g.has_b) *reinterpret_cast<double2*>(drow + g.ob2 + l2) = make_double2(xi[l2], xi[l2 + 1]);
            }
          }
        } else {
#pragma unroll
          for (int l2 = 0; l2 < 16; ++l2)
            if (l2 >= h && l2 < h + S) {
              int64_t c2 = g.oa2 + l2;
              if (c2 < a.bd.lim2) drow[c2] = xr[l2];
              c2 = g.ob2 + l2;
              if (g.has_b && c2 < a.bd.lim2) drow[c2] = xi[l2];
            }
        }
        if (PEER) {   // the same cells into the neighbour's halo row (NVLink stores)
          double* prow = c0 < a.peer.lo_end ? a.peer.lo + ((c0 - a.peer.lo_g0) * a.n1 + c1) * a.n2
                       : c0 >= a.peer.hi_begin ? a.peer.hi + ((c0 - a.peer.hi_g0) * a.n1 + c1) * a.n2
                                               : nullptr;
          if (prow) {
#pragma unroll
            for (int l2 = 0; l2 < 16; ++l2)
              if (l2 >= h && l2 < h + S) {
                int64_t c2 = g.oa2 + l2;
                if (c2 < a.bd.lim2) prow[c2] = xr[l2];
                c2 = g.ob2 + l2;
                if (g.has_b && c2 < a.bd.lim2) prow[c2] = xi[l2];
              }
          }
        }
      }
    }
  }
}

}  // namespace

// Two group buffers + S_T.
size_t fused3d_bf_smem(bool) { return (size_t)6 * PLANE * sizeof(double) + kAlign; }

cudaError_t fused3d_bf_configure(int* max_blocks) {
  const int st = (int)fused3d_bf_smem(true), sc = (int)fused3d_bf_smem(false);
  cudaError_t e = cudaFuncSetAttribute(fft3d_bf_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, st);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(fft3d_bf_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sc);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft3d_bf_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sc);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft3d_bf_kernel<true, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, st);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft3d_bf_kernel<false, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sc);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft3d_bf_kernel<true>, 2 * NT, st);
}

cudaError_t launch_fused3d_bf(const Fft3dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s) {
  static const CUtensorMap none = {};
  if (a.peer.lo || a.peer.hi) {   // boundary rows of a peer-transport rank (never periodic)
    if (tm)
      fft3d_bf_kernel<true, false, true><<<grid, 2 * NT, fused3d_bf_smem(true), s>>>(a, *tm);
    else
      fft3d_bf_kernel<false, false, true><<<grid, 2 * NT, fused3d_bf_smem(false), s>>>(a, none);
    return cudaGetLastError();
  }
  if (tm)
    fft3d_bf_kernel<true><<<grid, 2 * NT, fused3d_bf_smem(true), s>>>(a, *tm);
  else if (a.bd.wrap)
    fft3d_bf_kernel<false, true><<<grid, 2 * NT, fused3d_bf_smem(false), s>>>(a, none);
  else
    fft3d_bf_kernel<false><<<grid, 2 * NT, fused3d_bf_smem(false), s>>>(a, none);
  return cudaGetLastError();
}

}  // namespace fstencil
