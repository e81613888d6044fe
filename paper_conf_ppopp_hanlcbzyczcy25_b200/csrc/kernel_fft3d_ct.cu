// Fused 3D FFT-stencil tile kernel with FACTORED DFTs: 16 = 8 x 2 per axis (sm_100a).
//
// Same fused pass as kernel_fft3d.cu (Algorithm 1 L252-L258 on 16^3 overlap-save
// tiles, Double-layer Filling Eq. 9, temporal fusion Eq. 10, Stitching Eq. 7; 3D handled
// axis by axis as in §3.2.1), but each length-16 axis DFT is factored (§3.2.1's
// reshaping idea, L208-L218; Cooley-Tukey 16 = 8 x 2):
//   forward  X[ka + 8 kb] = sum_lb (-1)^(lb kb) w16^(ka lb) sum_la w8^(la ka) x[2 la + lb]
//   inverse  x[2 la + lb] = sum_ka w8^-(la ka) w16^-(ka lb) sum_kb (-1)^(lb kb) X[ka + 8 kb]
// The DFT-8 runs on the FP64 tensor cores over a group of 4 lines at once: the B operand is
// 8 x 8 with k = la and n = 2 m + lb (m = line of the group), so in the C fragment
// (row g, columns 2q + j) a thread holds both lb of one line -- the twiddle and the DFT-2
// are thread-local.  Per axis and element: 64 DMMA flops + 8 ALU flops instead of the
// dense 128 (kernel_fft3d.cu).  F_8 and the twiddles live in registers.
// Per tile pair, five shared-memory passes (each warp owns 4 lines; a group is read and
// rewritten in place):
//   P1 forward axis 2 | P2 forward axis 1 | P3 forward axis 0, * S_T, inverse axis 0 |
//   P4 inverse axis 1 on the S output planes | P5 inverse axis 2 on the S x S output rows
//   -> store the S^3 window.
// Shared layout: dense [l0][l1][l2] with l2 XOR-swizzled by a GF(2)-linear f(l0, l1) (parity
// masks 0x45, 0x86, 0xbd, 0xd7 of l0 | l1 << 4, found by search and checked exhaustively;
// evaluated as T0[l0] ^ T1[l1] from two packed 4-bit tables): every fragment pattern of the
// five passes is conflict-free per half-warp (8-byte accesses are served 16 lanes at a
// time), i.e. the optimal 2 wavefronts per 32 doubles,
// 64 KB for both planes -> 3 CTAs / SM.  f permutes words within a 16-element row only, so
// with TMA the tiles land as two dense 16^3 boxes and P1 (whose groups own whole rows)
// reads them unswizzled and rewrites its rows swizzled in place.
#include "ct_line.cuh"
#include "kernels.cuh"
#include "tma.cuh"

namespace fstencil {
namespace {

using dev::dmma;

constexpr int L = 16;   // (ct::L = 64 is the 2D line; unused here)
constexpr int PLANE = L * L * L;
constexpr int NWC = 8;

// f(l0, l1) = T0[l0] ^ T1[l1] (f is GF(2)-linear); the 16 x 4-bit tables packed in 64 bits.
__device__ __forceinline__ int swz(int l0, int l1) {
  constexpr unsigned long long kT0 = 0xc16b3e94852f7ad0ull, kT1 = 0xf3b76a2e1d5984c0ull;
  return (int)(((kT0 >> (4 * l0)) ^ (kT1 >> (4 * l1))) & 15ull);
}
__device__ __forceinline__ int off3(int l0, int l1, int l2) { return (l0 << 8) | (l1 << 4) | (l2 ^ swz(l0, l1)); }

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

// The 4 lines of a group: MODE 0 -> lines along l2 (l0 = a, l1 = b + m); MODE 1 -> along l1
// (l0 = a, l2 = b + m); MODE 2 -> along l0 (l1 = a, l2 = b + m).  DENSE: unswizzled offsets
// (the TMA staging layout, P1 reads only).
template <int MODE, bool DENSE = false>
struct Lines {
  int a, b;
  __device__ __forceinline__ int at(int m, int p) const {
    int l0, l1, l2;
    if (MODE == 0) { l0 = a; l1 = b + m; l2 = p; }
    else if (MODE == 1) { l0 = a; l1 = p; l2 = b + m; }
    else { l0 = p; l1 = a; l2 = b + m; }
    return DENSE ? (l0 << 8) | (l1 << 4) | l2 : off3(l0, l1, l2);
  }
};

// C = F8' . B (B-route of ct_line.cuh, one group; 4M unless FFTSTENCIL_CMUL3_3D)
template <bool CONJ>
__device__ __forceinline__ void cgemm(double (&cr)[2], double (&ci)[2], const double (&fr)[2], const double (&fi)[2],
                                      const double (&br)[2], const double (&bi)[2]) {
  double r[1][2], i[1][2];
  const double b_r[1][2] = {{br[0], br[1]}}, b_i[1][2] = {{bi[0], bi[1]}};
  ct::broute_n<CONJ, 1, FFTSTENCIL_CMUL3_3D != 0>(r, i, fr, fi, b_r, b_i);
  cr[0] = r[0][0]; cr[1] = r[0][1]; ci[0] = i[0][0]; ci[1] = i[0][1];
}

struct Regs {
  double fr[2], fi[2];     // F8[g][2q + j]
  double twr, twi;         // w16^g (forward, lb = 1)
  double itr[2], iti[2];   // conj(w16^(2q + j)) (inverse, lb = 1)
};

// Forward DFT-16 of the 4 lines read through `rd`; result (natural k order) written back
// through `wr` (same words), optionally multiplied by the spectrum (S_T at [q][g][j]).
template <class RD, class WR>
__device__ __forceinline__ void fwd_group(double* sR, double* sI, const RD& rd, const WR& wr, const Regs& rg, int g,
                                          int q, const double* spr, const double* spi) {
  double br[2], bi[2], cr[2], ci[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const int o = rd.at(g >> 1, 4 * q + 2 * j + (g & 1));
    br[j] = sR[o];
    bi[j] = sI[o];
  }
  cgemm<false>(cr, ci, rg.fr, rg.fi, br, bi);       // C[ka = g][2q + lb]
  const double tr = cr[1] * rg.twr - ci[1] * rg.twi, ti = cr[1] * rg.twi + ci[1] * rg.twr;
  double xr[2] = {cr[0] + tr, cr[0] - tr}, xi[2] = {ci[0] + ti, ci[0] - ti};   // k = g, g + 8
  if (spr) {
    const double2 s_r = __ldg(reinterpret_cast<const double2*>(spr));
    const double2 s_i = __ldg(reinterpret_cast<const double2*>(spi));
    const double a0 = xr[0] * s_r.x - xi[0] * s_i.x, b0 = xr[0] * s_i.x + xi[0] * s_r.x;
    const double a1 = xr[1] * s_r.y - xi[1] * s_i.y, b1 = xr[1] * s_i.y + xi[1] * s_r.y;
    xr[0] = a0; xi[0] = b0; xr[1] = a1; xi[1] = b1;
  }
  __syncwarp();   // the group is rewritten in place with another thread-to-word map
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const int o = wr.at(q, g + 8 * j);
    sR[o] = xr[j];
    sI[o] = xi[j];
  }
}

// Inverse DFT-16 (unnormalised; 1/16^3 is in S_T) of the 4 lines; returns the C fragment
// (line q, positions 2g + j) in cr/ci; writes it back in place if `store`.
template <class LN>
__device__ __forceinline__ void inv_group(double* sR, double* sI, const LN& ln, const Regs& rg, int g, int q,
                                          bool store, double (&cr)[2], double (&ci)[2]) {
  double br[2], bi[2];
  const int lb = g & 1;
#pragma unroll
  for (int j = 0; j < 2; ++j) {          // B[ka = 2q + j][n = g]: line g >> 1, lb = g & 1
    const int o0 = ln.at(g >> 1, 2 * q + j), o1 = ln.at(g >> 1, 2 * q + j + 8);
    const double ar = sR[o0], ai = sI[o0], xr = sR[o1], xi = sI[o1];
    double zr = lb ? ar - xr : ar + xr, zi = lb ? ai - xi : ai + xi;
    if (lb) {
      const double t = zr * rg.itr[j] - zi * rg.iti[j];
      zi = zr * rg.iti[j] + zi * rg.itr[j];
      zr = t;
    }
    br[j] = zr;
    bi[j] = zi;
  }
  cgemm<true>(cr, ci, rg.fr, rg.fi, br, bi);         // C[la = g][2q + lb] -> position 2g + j of line q
  if (store) {
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      const int o = ln.at(q, 2 * g + j);
      sR[o] = cr[j];
      sI[o] = ci[j];
    }
  }
}

template <bool TMA, bool WRAP = false>   // WRAP: periodic boundary (cp.async path only)
__global__ void __maxnreg__(72) fft3d_ct_kernel(const Fft3dArgs a, const __grid_constant__ CUtensorMap tm) {
  extern __shared__ __align__(128) double smem[];
  double* sR = smem;
  double* sI = smem + PLANE;
  __shared__ __align__(8) uint64_t bar;
  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31, g = lane >> 2, q = lane & 3;
  if (TMA && tid == 0) tma::mbar_init(&bar, 1);
  uint32_t parity = 0;
  Regs rg;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    rg.fr[j] = a.Fre[g * 8 + 2 * q + j];
    rg.fi[j] = a.Fim[g * 8 + 2 * q + j];
    rg.itr[j] = a.Fre[64 + 2 * q + j];
    rg.iti[j] = -a.Fim[64 + 2 * q + j];
  }
  rg.twr = a.Fre[64 + g];
  rg.twi = a.Fim[64 + g];
  const int S = a.S, h = a.h;
  const int G1 = (S + 3) >> 2;   // line groups of the last inverse pass

  for (int64_t p = a.win.p_begin + blockIdx.x; p < a.win.p_end; p += gridDim.x) {
    const int64_t line = p / a.npr, pj = p - line * a.npr;
    const int64_t t0 = line / a.nt1, t1 = line - t0 * a.nt1;
    const int64_t o0 = t0 * S + a.bd.shift, o1 = t1 * S + a.bd.shift, oa2 = 2 * pj * S + a.bd.shift, ob2 = oa2 + S;
    const bool has_b = 2 * pj + 1 < a.nt2;
    if (TMA) tma::fence_proxy_async();
    __syncthreads();
    if (TMA) {
      // ---- load the halo'd pair: two dense 16^3 TMA boxes (OOB -> 0) ----
      if (tid == 0) {
        tma::mbar_expect_tx(&bar, (has_b ? 2u : 1u) * PLANE * 8u);
        tma::load_3d(sR, &tm, (int)oa2, (int)o1, (int)(o0 - a.win.g0), &bar);
        if (has_b) tma::load_3d(sI, &tm, (int)ob2, (int)o1, (int)(o0 - a.win.g0), &bar);
      }
      if (!has_b)
        for (int e = tid; e < PLANE; e += NWC * 32) sI[e] = 0.0;
      tma::mbar_wait(&bar, parity);
      parity ^= 1;
    } else {
      // ---- load the halo'd pair (8-byte cp.async into the swizzled layout, OOB = 0) ----
      for (int e = tid; e < 2 * PLANE; e += NWC * 32) {
        const int t = e >> 12, l0 = (e >> 8) & 15, l1 = (e >> 4) & 15, l2 = e & 15;
        int64_t g0 = o0 + l0, g1 = o1 + l1, g2 = (t ? ob2 : oa2) + l2;
        if (WRAP) { g0 = wrap_index(g0, a.n0); g1 = wrap_index(g1, a.n1); g2 = wrap_index(g2, a.n2); }
        const int64_t lg0 = g0 - a.win.g0;
        const bool valid = (t == 0 || has_b) && g0 < a.n0 && lg0 >= 0 && lg0 < a.win.gn && g1 >= 0 && g1 < a.n1 &&
                           g2 >= 0 && g2 < a.n2;
        cp_async8((t ? sI : sR) + off3(l0, l1, l2), valid ? a.src + (lg0 * a.n1 + g1) * a.n2 + g2 : a.src, valid);
      }
      asm volatile("cp.async.commit_group;\n" ::);
      asm volatile("cp.async.wait_all;\n" ::: "memory");
    }
    __syncthreads();
    // ---- P1: forward axis 2 (lines along l2; TMA: read the dense rows, write swizzled) ----
    for (int grp = warp; grp < 64; grp += NWC) {
      const Lines<0, TMA> rd{grp >> 2, (grp & 3) * 4};
      const Lines<0> wr{grp >> 2, (grp & 3) * 4};
      fwd_group(sR, sI, rd, wr, rg, g, q, nullptr, nullptr);
    }
    __syncthreads();
    // ---- P2: forward axis 1 (lines along l1) ----
    for (int grp = warp; grp < 64; grp += NWC) {
      const Lines<1> ln{grp >> 2, (grp & 3) * 4};
      fwd_group(sR, sI, ln, ln, rg, g, q, nullptr, nullptr);
    }
    __syncthreads();
    // ---- P3: forward axis 0, * S_T, inverse axis 0 (lines along l0 at fixed k1) ----
    for (int grp = warp; grp < 64; grp += NWC) {
      const int k1 = grp >> 2, k2b = (grp & 3) * 4;
      const Lines<2> ln{k1, k2b};
      const int64_t si = (((int64_t)k1 * 16 + k2b + q) * 8 + g) * 2;   // S_T at [k1][k2][g][j]
      fwd_group(sR, sI, ln, ln, rg, g, q, a.Sre + si, a.Sim + si);
      __syncwarp();
      double cr[2], ci[2];
      inv_group(sR, sI, ln, rg, g, q, true, cr, ci);
    }
    __syncthreads();
    // ---- P4: inverse axis 1 on the S output planes (lines along l1) ----
    for (int grp = warp; grp < 4 * S; grp += NWC) {
      const Lines<1> ln{h + (grp >> 2), (grp & 3) * 4};
      double cr[2], ci[2];
      inv_group(sR, sI, ln, rg, g, q, true, cr, ci);
    }
    __syncthreads();
    // ---- P5: inverse axis 2 on the S x S output rows (lines along l2), store the window ----
    for (int grp = warp; grp < S * G1; grp += NWC) {
      const int i0 = grp / G1, gi = grp - i0 * G1;
      const int l0 = h + i0;
      // the last group of a ragged S shifts back inside the tile (its overlap is recomputed
      // and stored twice with bitwise-identical values)
      const int off1 = S >= 4 ? min(4 * gi, S - 4) : 0;
      const int l1b = h + off1;
      const Lines<0> ln{l0, l1b};
      double cr[2], ci[2];
      inv_group(sR, sI, ln, rg, g, q, false, cr, ci);
      const int64_t c0 = o0 + l0, c1 = o1 + l1b + q;
      if (off1 + q >= S || c0 >= a.bd.lim0 || c0 < a.win.w_lo || c0 >= a.win.w_hi || c1 >= a.bd.lim1) continue;
      double* drow = a.dst + ((c0 - a.win.g0) * a.n1 + c1) * a.n2;
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int l2 = 2 * g + j;
        if (l2 >= h && l2 < h + S) {
          int64_t c2 = oa2 + l2;
          if (c2 < a.bd.lim2) drow[c2] = cr[j];
          c2 = ob2 + l2;
          if (has_b && c2 < a.bd.lim2) drow[c2] = ci[j];
        }
      }
    }
  }
}

}  // namespace

size_t fused3d_ct_smem() { return (size_t)2 * PLANE * sizeof(double); }

cudaError_t fused3d_ct_configure(int* max_blocks) {
  const size_t smem = fused3d_ct_smem();
  cudaError_t e = cudaFuncSetAttribute(fft3d_ct_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft3d_ct_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft3d_ct_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft3d_ct_kernel<true>, NWC * 32, smem);
}

cudaError_t launch_fused3d_ct(const Fft3dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s) {
  static const CUtensorMap none = {};
  if (tm)
    fft3d_ct_kernel<true><<<grid, NWC * 32, fused3d_ct_smem(), s>>>(a, *tm);
  else if (a.bd.wrap)
    fft3d_ct_kernel<false, true><<<grid, NWC * 32, fused3d_ct_smem(), s>>>(a, none);
  else
    fft3d_ct_kernel<false><<<grid, NWC * 32, fused3d_ct_smem(), s>>>(a, none);
  return cudaGetLastError();
}

}  // namespace fstencil
