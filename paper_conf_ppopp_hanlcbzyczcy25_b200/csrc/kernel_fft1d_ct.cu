// Fused 1D FFT-stencil tile kernel with a LONG factored tile: L = 4096 = 64 x 64 (sm_100a).
//
// The paper's 1D path reshapes a length-N DFT into a 2D one (§3.2.1) with the
// prime-factor map so that no twiddles are needed (kernel_fft1d.cu, N = 8 x 7).  A tile
// of 56 cells, however, spends most of itself on the halo once T grows (S = 56 - 2rT), and
// the paper's own unrestricted temporal fusion (§4) wants T large: the cost per
// cell-step is ~ (DFT work per cell) x L / ((L - 2rT) T), minimised at T = L / (4r).  On
// B200 the tile that fits three CTAs per SM is 4096 complex (64 KB for the pair), so this
// kernel takes the Cooley-Tukey form of the same reshaping (four-step FFT):
//     n = a + 64 b,  k = c + 64 d        (a, b, c, d in [0, 64))
//     X[c + 64 d] = sum_a w64^(a d) . w4096^(a c) . sum_b x[a + 64 b] w64^(b c)
// i.e. DFT-64 down every column (b -> c), twiddle w4096^(a c), DFT-64 along every row
// (a -> d); each DFT-64 is itself CT 8 x 8 on the tensor cores (ct_line.cuh).  The inverse
// (conj(F), 1/L folded into S_T, L258 / reading Q7) runs the same steps backwards.
// Per tile pair (Double-layer Filling Eq. 9: Re = tile 2p, Im = tile 2p + 1):
//   load      x[o + a + 64 b] -> plane[b][a]  (natural row-major, XOR-swizzled)
//   phase 1   64 columns a:  DFT-64 over b (-> c at row c), * w4096^(a c)        in place
//   phase 2   64 rows c:     DFT-64 over a (-> d), * S_T[c + 64 d] (Eq. 10),
//                            iDFT-64 over d (-> a)                                in place
//   phase 3   64 columns a:  * w4096^(-a c), iDFT-64 over c (-> b)                in place
//   store     the S valid cells [h, h + S) of each tile (Eq. 7, reading Q4)
// Every phase reads and rewrites exactly its own line's words, so three CTA barriers are the
// only synchronisation; the swizzle makes both line patterns bank-conflict free.
#include "ct_line.cuh"
#include "kernels.cuh"

namespace fstencil {
namespace {

using namespace ct;

constexpr int PLANE = L * L;   // 4096 = the 1D tile length
constexpr int kThreads = 256;

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

template <bool CONJ>
__device__ __forceinline__ void cmul(double (&cr)[1][2], double (&ci)[1][2], const double2 (&w)[2]) {
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const double wi = CONJ ? -w[j].y : w[j].y;
    const double r = cr[0][j] * w[j].x - ci[0][j] * wi;
    const double i = cr[0][j] * wi + ci[0][j] * w[j].x;
    cr[0][j] = r;
    ci[0][j] = i;
  }
}

template <bool WRAP>   // WRAP: periodic boundary (wrap-around tile loads)
__global__ void __maxnreg__(72) fft1d_ct_kernel(const Fft1dArgs a) {
  extern __shared__ __align__(128) double smem[];
  double* sR = smem;           // tile 2p   (Re), then the transform's real parts
  double* sI = smem + PLANE;   // tile 2p+1 (Im)
  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31, g = lane >> 2, q = lane & 3;
  constexpr int NW = kThreads / 32;

  double fr[2], fi[2], tr[2], ti[2];   // F8 (row g, column 2q + j) and w64^(g (2q + j))
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const int c = 2 * q + j;
    fr[j] = a.Fre[g * 8 + c];
    fi[j] = a.Fim[g * 8 + c];
    tr[j] = a.Fre[64 + g * 8 + c];
    ti[j] = a.Fim[64 + g * 8 + c];
  }
  int cl[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) cl[j] = 16 * q + 8 * j + g;
  const double2* tw = reinterpret_cast<const double2*>(a.tw);   // w4096^(a c) at [a][c]
  const int S = a.S, h = a.h;
  const int64_t g0 = a.win.g0, g1 = a.win.g0 + a.win.gn;

  for (int64_t p = a.win.p_begin + blockIdx.x; p < a.win.p_end; p += gridDim.x) {
    const int64_t oa = 2 * p * S + a.bd.shift, ob = oa + S;   // global cell of tile position 0
    const bool has_b = 2 * p + 1 < a.ntiles;
    __syncthreads();   // the previous pair's store has read the planes
    // ---- load the halo'd pair (OOB -> 0): x[o + a + 64 b] -> plane[b][a] ----
    for (int e = tid; e < 2 * PLANE; e += kThreads) {
      const int t = e >> 12, n = e & (PLANE - 1);
      int64_t x = (t ? ob : oa) + n;
      if (WRAP) x = wrap_index(x, a.n);
      const bool valid = (t == 0 || has_b) && x >= 0 && x < a.n && x >= g0 && x < g1;
      cp_async8((t ? sI : sR) + sw(n >> 6, n & 63), valid ? a.src + (x - g0) : a.src, valid);
    }
    asm volatile("cp.async.commit_group;\n" ::);
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    __syncthreads();

    // ---- phase 1: columns a, DFT-64 over b -> c (row c = cl[j]), * w4096^(a c) ----
    for (int col = warp; col < L; col += NW) {
      double br[1][2], bi[1][2], c1r[1][2], c1i[1][2], c2r[1][2], c2i[1][2];
      double2 w[2];
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        br[0][j] = sR[sw(cl[j], col)];
        bi[0][j] = sI[sw(cl[j], col)];
        w[j] = __ldg(tw + col * 64 + cl[j]);
      }
      broute_n<false, 1>(c1r, c1i, fr, fi, br, bi);
      twiddle_n<false, 1>(c1r, c1i, tr, ti);
      aroute_n<false, 1>(c2r, c2i, c1r, c1i, fr, fi);
      cmul<false>(c2r, c2i, w);
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        sR[sw(cl[j], col)] = c2r[0][j];
        sI[sw(cl[j], col)] = c2i[0][j];
      }
    }
    __syncthreads();

    // ---- phase 2: rows c, DFT-64 over a -> d, * S_T[c + 64 d], iDFT-64 over d -> a ----
    for (int row = warp; row < L; row += NW) {
      double br[1][2], bi[1][2], c1r[1][2], c1i[1][2], c2r[1][2], c2i[1][2];
      const double2 sr = __ldg(reinterpret_cast<const double2*>(a.Sre + row * 64 + g * 8 + 2 * q));
      const double2 si = __ldg(reinterpret_cast<const double2*>(a.Sim + row * 64 + g * 8 + 2 * q));
      const double s_r[2] = {sr.x, sr.y}, s_i[2] = {si.x, si.y};
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        br[0][j] = sR[sw(row, cl[j])];
        bi[0][j] = sI[sw(row, cl[j])];
      }
      broute_n<false, 1>(c1r, c1i, fr, fi, br, bi);
      twiddle_n<false, 1>(c1r, c1i, tr, ti);
      aroute_n<false, 1>(c2r, c2i, c1r, c1i, fr, fi);   // d = cl[j]
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const double r = c2r[0][j] * s_r[j] - c2i[0][j] * s_i[j];
        const double i = c2r[0][j] * s_i[j] + c2i[0][j] * s_r[j];
        c2r[0][j] = r;
        c2i[0][j] = i;
      }
      broute_n<true, 1>(c1r, c1i, fr, fi, c2r, c2i);
      twiddle_n<true, 1>(c1r, c1i, tr, ti);
      aroute_n<true, 1>(c2r, c2i, c1r, c1i, fr, fi);    // a = cl[j]
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        sR[sw(row, cl[j])] = c2r[0][j];
        sI[sw(row, cl[j])] = c2i[0][j];
      }
    }
    __syncthreads();

    // ---- phase 3: columns a, * w4096^(-a c), iDFT-64 over c -> b ----
    for (int col = warp; col < L; col += NW) {
      double br[1][2], bi[1][2], c1r[1][2], c1i[1][2], c2r[1][2], c2i[1][2];
      double2 w[2];
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        br[0][j] = sR[sw(cl[j], col)];
        bi[0][j] = sI[sw(cl[j], col)];
        w[j] = __ldg(tw + col * 64 + cl[j]);
      }
      cmul<true>(br, bi, w);
      broute_n<true, 1>(c1r, c1i, fr, fi, br, bi);
      twiddle_n<true, 1>(c1r, c1i, tr, ti);
      aroute_n<true, 1>(c2r, c2i, c1r, c1i, fr, fi);    // b = cl[j]
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        sR[sw(cl[j], col)] = c2r[0][j];
        sI[sw(cl[j], col)] = c2i[0][j];
      }
    }
    __syncthreads();

    // ---- store the valid window of both tiles (coalesced; row-pattern shared reads) ----
    for (int e = tid; e < 2 * S; e += kThreads) {
      const int t = e >= S;
      if (t && !has_b) break;
      const int n = h + (t ? e - S : e);
      const int64_t x = (t ? ob : oa) + n;
      if (x < a.bd.lim0 && x >= a.win.w_lo && x < a.win.w_hi)
        a.dst[x - g0] = (t ? sI : sR)[sw(n >> 6, n & 63)];
    }
  }
}

}  // namespace

size_t fused1d_ct_smem() { return (size_t)2 * PLANE * sizeof(double); }

cudaError_t fused1d_ct_configure(int* max_blocks) {
  const int smem = (int)fused1d_ct_smem();
  cudaError_t e = cudaFuncSetAttribute(fft1d_ct_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft1d_ct_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft1d_ct_kernel<false>, kThreads, smem);
}

cudaError_t launch_fused1d_ct(const Fft1dArgs& a, int grid, cudaStream_t s) {
  const size_t smem = fused1d_ct_smem();
  if (a.bd.wrap)
    fft1d_ct_kernel<true><<<grid, kThreads, smem, s>>>(a);
  else
    fft1d_ct_kernel<false><<<grid, kThreads, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace fstencil
