// Whole-run kernel for small 1D grids (sm_100a): every pass of one fftstencil_run in ONE launch
// of ONE thread-block cluster (8 CTAs on 8 SMs), the grid resident in shared memory.
//
// A grid of a few thousand cells (BASELINE configs[0]: Heat-1D, 4096 cells, T = 8, 64 steps)
// gives each fused pass ~50 tile pairs: the per-pass kernels of the normal driver (fused tile
// kernel, band kernel, events, ring copies) are launch-latency bound (~20 us per pass for ~4 us
// of work), and a single CTA is bound by one SM's FP64 tensor pipe (51 pairs x 32 DMMA).  Here
// every CTA of the cluster keeps the whole grid (2 buffers, <= 128 KB) in its shared memory:
//   load in -> buffers A and B (B keeps the fixed ring);
//   per pass t in {T, ..., T, steps mod T}: CTA c's warps transform its share of the tile pairs
//     exactly as kernel_fft1d.cu does (PFA 8 x 7 = 56-cell tiles, CRT map, four chained 8x8
//     complex DMMA GEMMs with the powered spectrum S_t between them: PAPER.md §3.2.1
//     L212-L218, Alg. 1, Eq. 10), reading its own copy of the current buffer
//     and storing every output into the other buffer of ALL 8 CTAs (distributed shared memory);
//     the first / last CTA's spare warp recomputes the band cells [r, h) / [n-h, n-r) by t direct
//     steps over their dependency cones (reading Q5) and stores them the same way; cluster
//     barrier (release / acquire); swap;
//   CTA 0 stores the final buffer to out (in == out is fine: every CTA read all of in before
//   the first cluster barrier).
// Tiles write exactly the exact region [h, n-h), the band the rest of the interior, the ring
// never changes, so every cell of the destination buffer is defined after each pass.
#include <cooperative_groups.h>

#include "device_common.cuh"
#include "kernels.cuh"

namespace fstencil {
namespace {

using dev::cgemm8;

namespace cg = cooperative_groups;

constexpr int kCtas = 8;                   // cluster size (portable maximum)
constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;

// Remote (distributed shared memory) addresses: rb[k] = the buffer's shared::cluster address in
// CTA k (mapa once per launch); st.shared::cluster stores v to element i of it in every CTA.
struct RemoteBuf {
  uint32_t rb[kCtas];
};
__device__ __forceinline__ RemoteBuf remote(const double* b) {
  RemoteBuf r;
  const uint32_t a = (uint32_t)__cvta_generic_to_shared(b);
#pragma unroll
  for (int k = 0; k < kCtas; ++k) asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r.rb[k]) : "r"(a), "r"(k));
  return r;
}
__device__ __forceinline__ void bcast(const RemoteBuf& d, int i, double v) {
#pragma unroll
  for (int k = 0; k < kCtas; ++k)
    asm volatile("st.shared::cluster.f64 [%0], %1;" ::"r"(d.rb[k] + 8u * (uint32_t)i), "d"(v) : "memory");
}
// Cluster barrier with release / acquire at cluster scope (orders the shared::cluster stores;
// no GPU-scope fence as cooperative_groups' cluster.sync() emits for generic stores).
__device__ __forceinline__ void cluster_barrier() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;\n" ::: "memory");
}

// t direct steps of one band side in scratch (a, b: 2 x R doubles); lower side: cells
// [0, R) with the ring [0, r); upper side: cells [n - R, n) with the ring [n - r, n).
__device__ void band_side(const RemoteBuf& dst, const Small1dArgs& A, const double* w, const double* src, double* a,
                          double* b, int t, bool upper, int lane) {
  const int r = A.r, h = A.h, n = (int)A.n;
  const int R = min(h + r * t, n);
  const int base = upper ? n - R : 0;
  for (int i = lane; i < R; i += 32) a[i] = src[base + i];
  __syncwarp();
  for (int s = 1; s <= t; ++s) {
    // local cells updated at step s: the cone shrinks from the open side
    const int lo = upper ? r * s : r, hi = upper ? R - r : R - r * s;
    for (int i = lane; i < R; i += 32) {
      double v = a[i];
      if (i >= lo && i < hi) {
        v = 0.0;
        for (int o = -r; o <= r; ++o) v = fma(w[o + r], a[i + o], v);
      }
      b[i] = v;
    }
    __syncwarp();
    double* tmp = a; a = b; b = tmp;
  }
  // band cells: lower [r, h), upper [n - h, n - r)
  const int c0 = upper ? n - h : r, c1 = upper ? n - r : h;
  for (int c = c0 + lane; c < c1; c += 32) bcast(dst, c, a[c - base]);
}

__global__ void __cluster_dims__(kCtas, 1, 1) __launch_bounds__(kThreads, 1) small1d_run_kernel(const Small1dArgs A) {
  const int rank = (int)cg::this_cluster().block_rank();
  extern __shared__ double sm[];
  __shared__ double s_w[2 * kSmall1dMaxR + 1];
  const int n = (int)A.n;
  if (threadIdx.x <= 2 * A.r) s_w[threadIdx.x] = A.w[threadIdx.x];
  double* bufA = sm;
  double* bufB = sm + n;
  double* scratch = sm + 2 * n;                         // band: 2 x Rmax
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;
  for (int i = threadIdx.x; i < n; i += kThreads) {
    const double v = A.in[i];
    bufA[i] = v;
    bufB[i] = v;                                        // the ring of the second buffer
  }
  const RemoteBuf remA = remote(bufA), remB = remote(bufB);
  cluster_barrier();   // every CTA's buffers are loaded before any CTA stores into them

  // DFT fragments and tile positions for the launch (kernel_fft1d.cu's layout)
  double f1r[2], f1i[2], f2r[2], f2i[2];
  int pos[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const int c = 2 * q + j;
    f1r[j] = A.Fre[g * 8 + c];
    f1i[j] = A.Fim[g * 8 + c];
    f2r[j] = A.Fre[(8 + g) * 8 + c];
    f2i[j] = A.Fim[(8 + g) * 8 + c];
    pos[j] = A.crt[g * 8 + c];
  }
  // spectrum fragments of S_T and of the remainder pass's S_rem, for the launch
  double sTr[2], sTi[2], sRr[2], sRi[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    sTr[j] = A.Sre_T[g * 8 + 2 * q + j];
    sTi[j] = A.Sim_T[g * 8 + 2 * q + j];
    sRr[j] = A.Sre_rem[g * 8 + 2 * q + j];
    sRi[j] = A.Sim_rem[g * 8 + 2 * q + j];
  }
  const int L = A.L, S = A.S, h = A.h;
  const int64_t npairs = (A.ntiles + 1) / 2;
  const int64_t per = (npairs + kCtas - 1) / kCtas;
  const int64_t p_lo = min(npairs, rank * per), p_hi = min(npairs, p_lo + per);
  for (int64_t pass = 0; pass < A.passes; ++pass) {
    const bool last_rem = pass == A.passes - 1 && A.rem > 0;
    const int t = last_rem ? A.rem : A.T;
    const bool even = (pass & 1) == 0;
    const double* src = even ? bufA : bufB;
    const RemoteBuf& dst = even ? remB : remA;
    // band: the last warp of CTA 0 (lower side) and of CTA kCtas - 1 (upper side)
    if (warp == kWarps - 1 && (rank == 0 || rank == kCtas - 1)) {
      const bool upper = rank == kCtas - 1;
      band_side(dst, A, s_w, src, scratch, scratch + A.rmax, t, upper, lane);
    }
    double sr[2], si[2];
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      sr[j] = last_rem ? sRr[j] : sTr[j];
      si[j] = last_rem ? sRi[j] : sTi[j];
    }
    // this CTA's pairs [p_lo, p_hi), one per warp and round
    for (int64_t p = p_lo + warp; p < p_hi; p += kWarps) {
      const int oa = (int)(2 * p * S), ob = oa + S;    // cell of tile position 0
      const bool has_b = 2 * p + 1 < A.ntiles;
      double xr[2], xi[2];
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        xr[j] = 0.0;
        xi[j] = 0.0;
        if (pos[j] >= 0) {
          const int xa = oa + pos[j], xb = ob + pos[j];
          if (xa < n) xr[j] = src[xa];
          if (has_b && xb < n) xi[j] = src[xb];
        }
      }
      double m1r[2], m1i[2], m2r[2], m2i[2];
      cgemm8<false>(f2r, f2i, xr, xi, m1r, m1i);
      cgemm8<false>(f1r, f1i, m1r, m1i, m2r, m2i);
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const double re = m2r[j] * sr[j] - m2i[j] * si[j];
        const double im = m2r[j] * si[j] + m2i[j] * sr[j];
        m2r[j] = re;
        m2i[j] = im;
      }
      cgemm8<true>(f2r, f2i, m2r, m2i, m1r, m1i);
      cgemm8<true>(f1r, f1i, m1r, m1i, m2r, m2i);
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int l = pos[j];
        if (l >= h && l < L - h) {                     // valid window, exact region [h, n - h)
          const int xa = oa + l, xb = ob + l;
          if (xa < n - h) bcast(dst, xa, m2r[j]);
          if (has_b && xb < n - h) bcast(dst, xb, m2i[j]);
        }
      }
    }
    cluster_barrier();   // every CTA's destination buffer is complete
  }
  if (rank == 0) {
    const double* fin = (A.passes & 1) ? bufB : bufA;
    for (int i = threadIdx.x; i < n; i += kThreads) A.out[i] = fin[i];
  }
}

}  // namespace

size_t small1d_smem(int64_t n, int rmax) { return (size_t)(2 * n + 2 * rmax) * sizeof(double); }

cudaError_t small1d_configure() {
  return cudaFuncSetAttribute(small1d_run_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)small1d_smem(kSmall1dMaxCells, kSmall1dMaxBand));
}

cudaError_t launch_small1d(const Small1dArgs& a, cudaStream_t s) {
  small1d_run_kernel<<<kCtas, kThreads, small1d_smem(a.n, a.rmax), s>>>(a);
  return cudaGetLastError();
}

}  // namespace fstencil
