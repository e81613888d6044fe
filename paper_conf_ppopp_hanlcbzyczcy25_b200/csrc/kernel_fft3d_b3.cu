// Fused 3D FFT-stencil tile kernel, three shared-memory passes per tile pair (sm_100a).
//
// The fused pass of PAPER.md Algorithm 1 (L252-L258) on 16^3 overlap-save tiles (Eq. 3/4,
// Stitching Eq. 7), two real tiles per complex tile (Double-layer Filling, Eq. 9), the T-step
// powered spectrum (Eq. 10), 3D handled axis by axis (§3.2.1).  Each length-16 axis DFT
// is Cooley-Tukey 16 = 4 x 4 on the FP64 ALU (fft_radix.cuh; reading Q20 for why
// not the FP64 tensor pipe on B200).
//
// Why three passes.  The line kernel (kernel_fft3d_bf.cu) gives a thread one 16-point line
// per pass, so the forward and inverse 3D transforms take five shared-memory round trips per
// pair and the kernel is bound by shared-memory traffic and its latency (ncu: 4.8 k wavefronts
// vs 3.7 k FP64 pipe cycles per pair, profiles/r01_s3_fft3d_bf_ncu.txt).  Here a PAIR of
// threads (lanes L and L ^ m of one warp, "A" and "B") holds 64 complex values, 32 each --
// enough for a whole 16-point line of one axis times the first radix-4 digit of another:
//   P1  (l0, c): rows l1 = 4 j + c, j = 0..3 of plane l0 (A: j = 0, 2; B: j = 1, 3) ->
//       FFT-16 along axis 2, DFT-4 over j -> k1a (axis 1, first stage), twiddle w16^(c k1a);
//   P2  (k1a, k2): all 16 l0 x 4 c (A: c = 0, 2; B: c = 1, 3) -> DFT-4 over c -> k1b (axis 1,
//       second stage; k1 = k1a + 4 k1b), FFT-16 along axis 0, * S_T, inverse FFT-16, inverse
//       DFT-4 over k1b -> c on the S output planes;
//   P3  (l0, c), l0 an output plane: inverse DFT-4 over k1a -> j (its twiddle is applied by P2
//       on the output planes), inverse FFT-16 along axis 2 on rows l1 = 4 j + c -> store.
// Each DFT-4 that spans a thread pair is two radix-2 stages: the first inside each thread,
// the second across the pair with one register-shuffle exchange of 16 complex values
// (a half-exchange: each lane keeps one radix-2 output and sends the other).  Per pair: two
// shared-memory exchanges instead of four (2.8 k wavefronts incl. the TMA image, vs 4.9 k),
// ~1 k shuffle instructions, ~260 k FP64 instructions.
//
// Lane-uniform arithmetic.  A and B run the same instruction stream: the first radix-2 uses
// a per-lane sign s (A: +1, B: -1, so B's sum and difference land in swapped registers and
// both lanes send register 1), the second is out0 = recv + T, out1 = recv - T with T = own
// (A) or -+i own (B, two selects).  A's out1 then carries a minus sign, which is folded into
// the next linear factor: the P1 twiddle, the P2 spectrum (S_T), the inverse twiddle P2 applies
// before its stores (P2's inverse), and the final store (P3's inverse).
//
// S_T lives in tensor memory: a P2 lane always owns the same (k1a, k2, c parity), so its 32
// spectrum values (128 32-bit columns of its TMEM lane) are written once per launch and read
// with tcgen05.ld in P2, off the shared-memory path.  Shared memory holds only the pair
// buffers: three independent 128-thread groups per CTA, one 64 KB buffer each (192 KB, one
// CTA per SM, 12 warps).  A group waits for its pair's TMA boxes (Re = tile 2j, Im = tile
// 2j + 1) and refills its buffer with the next pair once P3 has read it.
#include "fft_radix.cuh"
#include "kernels.cuh"
#include "tma.cuh"

namespace fstencil {
namespace {

constexpr int L = 16;
constexpr int PLANE = L * L * L;        // doubles per real tile
constexpr int GT = 128;                 // threads per group (one tile pair)
#ifndef B3_NG
#define B3_NG 3
#endif
constexpr int NG = B3_NG;               // groups per CTA
constexpr int NT = GT * NG;
constexpr int kAlign = 1024;            // SWIZZLE_128B destinations are 1024-byte aligned
constexpr uint32_t kTmemCols = 128;     // 32 complex S_T values per TMEM lane

using radix::cmul;
using radix::fft16;

// Exchange layout (P1 -> P2 -> P3), one 16-byte (re, im) word per element (l0, c, k1a, k2):
// word ((l0 * 4 + c) * 4 + k1a) * 16 + (k2 ^ g), g = 2 c + (k1a & 1).  A P2 quarter-warp is
// 8 consecutive k2 (distinct words mod 8); a P1 / P3 quarter-warp is (c = 0..3) x (A, B) of
// one l0, i.e. 8 distinct g: conflict-free both ways.
__device__ __forceinline__ int xofs(int l0, int c, int k1a, int k2) {
  return ((((l0 << 2) | c) << 2 | k1a) << 5) | ((k2 ^ ((c << 1) | (k1a & 1))) << 1);
}
__device__ __forceinline__ double2 ld2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ void st2(double* p, double re, double im) {
  *reinterpret_cast<double2*>(p) = make_double2(re, im);
}

__device__ __forceinline__ void group_sync(int grp) {
  asm volatile("bar.sync %0, %1;\n" ::"r"(grp + 1), "r"(GT) : "memory");
}

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

// ---- tensor memory: 16 consecutive 32-bit columns of this warp's lane quarter ----
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
        "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};\n" ::"r"(
          taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]),
      "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
      : "memory");
}
__device__ __forceinline__ double u2d(uint32_t lo, uint32_t hi) { return __hiloint2double((int)hi, (int)lo); }

// The two radix-2 stages of a DFT-4 spread over a lane pair (A holds inputs 0 and 2, B holds
// 1 and 3, in registers x0 = first, x1 = second), per element:
//   local:  r0 = x0 + s x1, r1 = x0 - s x1        (A: s = +1 -> E0, E1; B: s = -1 -> O1, O0)
//   swap:   recv = partner's r1                   (A receives O0, B receives E1)
//   cross:  T = A ? r0 : rot r0  (rot = -i forward, +i inverse),  x0 = recv + T,  x1 = recv - T
// -> A: x0 = X0, x1 = -X2;  B: x0 = X1, x1 = X3  (forward; the inverse likewise with w4^-1).
template <bool INV>
__device__ __forceinline__ void pair_dft4(double& x0r, double& x0i, double& x1r, double& x1i, double s, bool isB,
                                          int mask) {
  const double r0r = fma(s, x1r, x0r), r0i = fma(s, x1i, x0i);
  const double r1r = fma(-s, x1r, x0r), r1i = fma(-s, x1i, x0i);
  const double vr = __shfl_xor_sync(0xffffffffu, r1r, mask);
  const double vi = __shfl_xor_sync(0xffffffffu, r1i, mask);
  // -i (re, im) = (im, -re);  +i (re, im) = (-im, re)
  const double tr = isB ? (INV ? -r0i : r0i) : r0r;
  const double ti = isB ? (INV ? r0r : -r0r) : r0i;
  x0r = vr + tr;
  x0i = vi + ti;
  x1r = vr - tr;
  x1i = vi - ti;
}

struct PairGeom {   // tile origins (32-bit: extents are below 2^31)
  int o0, o1, oa2, ob2;
  bool has_b;
};
__device__ __forceinline__ PairGeom pair_geom(const Fft3dArgs& a, int64_t p) {
  // pair / tile indices fit 32 bits (the plan's pair count is far below 2^31)
  const int S = a.S, npr = (int)a.npr, nt1 = (int)a.nt1, pi = (int)p;
  const int line = pi / npr, pj = pi - line * npr;
  const int t0 = line / nt1, t1 = line - t0 * nt1;
  PairGeom g;
  g.o0 = t0 * S + a.bd.shift;
  g.o1 = t1 * S + a.bd.shift;
  g.oa2 = 2 * pj * S + a.bd.shift;
  g.ob2 = g.oa2 + S;
  g.has_b = 2 * pj + 1 < a.nt2;
  return g;
}

template <bool TMA, bool WRAP = false>
__global__ void __launch_bounds__(NT, 1) fft3d_b3_kernel(const Fft3dArgs a, const __grid_constant__ CUtensorMap tm) {
  extern __shared__ unsigned char smem_raw[];
  const uint32_t mis = tma::smem_addr(smem_raw) & (kAlign - 1);
  double* base = reinterpret_cast<double*>(smem_raw + (mis ? kAlign - mis : 0));
  __shared__ __align__(8) uint64_t bar[NG];
  __shared__ __align__(8) uint64_t fbar[NG];   // "buffer read by P3": one arrival per warp
  __shared__ uint32_t tmem_base;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int grp = threadIdx.x / GT, tid = threadIdx.x % GT, gw = tid >> 5;
  const int S = a.S, h = a.h;
  double* buf = base + grp * 2 * PLANE;
  double* sR = buf;
  double* sI = buf + PLANE;
  if (threadIdx.x == 0)
    for (int g = 0; g < NG; ++g) {
      tma::mbar_init(&bar[g], 1);
      tma::mbar_init(&fbar[g], GT / 32);
    }

  // ---- P1 / P3 role: c = tid & 3, pair member ab = bit 2 (partner lane ^ 4), l0 = tid >> 3 ----
  const int c = tid & 3, ab = (tid >> 2) & 1;
  const bool isB = ab != 0;
  const double sg = isB ? -1.0 : 1.0;
  // ---- P2 role: k1a = group warp, k2 = lane bits {0,1,2,4}, ab2 = lane bit 3 (partner ^ 8) ----
  const int k1a_2 = gw, k2_2 = (lane & 7) | ((lane >> 4) << 3), ab2 = (lane >> 3) & 1;
  const bool isB2 = ab2 != 0;
  const double sg2 = isB2 ? -1.0 : 1.0;

  // twiddles w16^m, m = 0..15 (the plan's table at Fre / Fim[64 + m]), read per pass from shared
  // memory rather than held in registers across the loop
  __shared__ double2 sw16[16];
  if (threadIdx.x < 16) sw16[threadIdx.x] = make_double2(__ldg(a.Fre + 64 + threadIdx.x), __ldg(a.Fim + 64 + threadIdx.x));

  // ---- S_T into tensor memory: lane (32 (warp & 3) + lane) holds, for its P2 role, at columns
  // 4 (16 slot + k0) + {re lo, re hi, im lo, im hi}: S_T[k0][k1a + 4 (ab2 + 2 slot)][k2]
  // (slot 1 of A lanes negated); group 0 writes, groups 1 and 2 share (same warp & 3) ----
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(tma::smem_addr(&tmem_base)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;\n");
  const uint32_t tmem_s = tmem_base + ((uint32_t)(32 * (warp & 3)) << 16);
  if (grp == 0) {
#pragma unroll 1
    for (int q = 0; q < 8; ++q) {   // 4 complex values (16 columns) per store
      uint32_t v[16];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int idx = 4 * q + e, slot = idx >> 4, k0 = idx & 15;
        const int sidx = (k0 << 8) | ((k1a_2 + 4 * (ab2 + 2 * slot)) << 4) | k2_2;
        const double f = (slot == 1 && !isB2) ? -1.0 : 1.0;
        const double re = f * __ldg(a.Sre + sidx), im = f * __ldg(a.Sim + sidx);
        v[4 * e] = (uint32_t)__double2loint(re);
        v[4 * e + 1] = (uint32_t)__double2hiint(re);
        v[4 * e + 2] = (uint32_t)__double2loint(im);
        v[4 * e + 3] = (uint32_t)__double2hiint(im);
      }
      tmem_st16(tmem_s + 16 * q, v);
    }
    asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;\n");

  // pair indices fit 32 bits (the plan's pair count is far below 2^31); 32-bit loop state
  // leaves the registers to the 64 complex values of a lane pair
  const int stride = NG * (int)gridDim.x;
  const int p0 = (int)a.win.p_begin + NG * (int)blockIdx.x + grp, pend = (int)a.win.p_end;
  auto issue = [&](int p) {
    const PairGeom g = pair_geom(a, p);
    // tile b is loaded even where the tile row has no tile 2j + 1: its outputs are not stored,
    // and with a real stencil the Re half does not depend on it (OOB boxes fill with zeros)
    tma::mbar_expect_tx(&bar[grp], 2u * PLANE * 8u);
    tma::load_3d(sR, &tm, g.oa2, g.o1, (int)(g.o0 - a.win.g0), &bar[grp]);
    tma::load_3d(sI, &tm, g.ob2, g.o1, (int)(g.o0 - a.win.g0), &bar[grp]);
  };
  if (TMA && tid == 0 && p0 < pend) issue(p0);
  uint32_t parity = 0;

#pragma unroll 1
  for (int p = p0; p < pend; p += stride) {
    if (TMA) {
      tma::mbar_wait(&bar[grp], parity);
      parity ^= 1;
    } else {
      group_sync(grp);   // the previous pair's P3 reads of this buffer are done
      const PairGeom g = pair_geom(a, p);
#pragma unroll 1
      for (int e = tid; e < 2 * PLANE; e += GT) {
        const int t = e >> 12, l0 = (e >> 8) & 15, l1 = (e >> 4) & 15, l2 = e & 15;
        int64_t g0 = (int64_t)g.o0 + l0, g1 = g.o1 + l1, g2 = (t ? g.ob2 : g.oa2) + l2;
        if (WRAP) { g0 = wrap_index(g0, a.n0); g1 = wrap_index(g1, a.n1); g2 = wrap_index(g2, a.n2); }
        const int64_t lg0 = g0 - a.win.g0;
        const bool valid = (t == 0 || g.has_b) && g0 < a.n0 && lg0 >= 0 && lg0 < a.win.gn && g1 >= 0 && g1 < a.n1 &&
                           g2 >= 0 && g2 < a.n2;
        // TMA image layout: element (l0, l1, l2) at 256 l0 + 16 l1 + (l2 ^ 2 (l1 & 7))
        cp_async8((t ? sI : sR) + ((l0 << 8) | (l1 << 4) | (l2 ^ ((l1 & 7) << 1))),
                  valid ? a.src + (lg0 * a.n1 + g1) * a.n2 + g2 : a.src, valid);
      }
      asm volatile("cp.async.commit_group;\n" ::);
      asm volatile("cp.async.wait_all;\n" ::: "memory");
      group_sync(grp);
    }
    // ---- P1: rows l1 = 4 (2 jj + ab) + c of plane l0 -> FFT along axis 2, DFT-4 over j ----
    {
      const int l0 = tid >> 3;
      double xr[2][16], xi[2][16];
#pragma unroll
      for (int jj = 0; jj < 2; ++jj) {
        // 16-byte chunk q of the row sits at chunk q ^ (l1 & 7) = q ^ (4 ab + c): the eight
        // lanes of a quarter-warp read eight different bank slots
        const int l1 = 4 * (2 * jj + ab) + c, rb = (l0 << 8) | (l1 << 4), sw = l1 & 7;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const int o = rb + ((q ^ sw) << 1);
          const double2 r = ld2(sR + o), i = ld2(sI + o);
          xr[jj][2 * q] = r.x;
          xr[jj][2 * q + 1] = r.y;
          xi[jj][2 * q] = i.x;
          xi[jj][2 * q + 1] = i.y;
        }
      }
      fft16<false>(xr[0], xi[0]);
      fft16<false>(xr[1], xi[1]);
      // twiddles w16^(c k1a) of this lane's k1a = ab, 2 + ab (slot 1 of A negated: pair_dft4)
      const double2 w0 = sw16[(c * ab) & 15], w1 = sw16[(c * (2 + ab)) & 15];
      const double f1 = isB ? 1.0 : -1.0;
#pragma unroll
      for (int k2 = 0; k2 < 16; ++k2) {
        pair_dft4<false>(xr[0][k2], xi[0][k2], xr[1][k2], xi[1][k2], sg, isB, 4);
        cmul(xr[0][k2], xi[0][k2], w0.x, w0.y);
        cmul(xr[1][k2], xi[1][k2], f1 * w1.x, f1 * w1.y);
      }
      group_sync(grp);   // every P1 read of the TMA image is done: rewrite the buffer in place
#pragma unroll
      for (int k2 = 0; k2 < 16; ++k2) {
        st2(buf + xofs(l0, c, ab, k2), xr[0][k2], xi[0][k2]);
        st2(buf + xofs(l0, c, 2 + ab, k2), xr[1][k2], xi[1][k2]);
      }
    }
    group_sync(grp);
    // ---- P2: (k1a, k2), c = ab2, 2 + ab2 -> DFT-4 over c, FFT along axis 0, * S_T, inverse ----
    {
      double zr[2][16], zi[2][16];   // [slot][l0 -> k0]
#pragma unroll
      for (int l0 = 0; l0 < 16; ++l0)
#pragma unroll
        for (int sl = 0; sl < 2; ++sl) {
          const double2 v = ld2(buf + xofs(l0, ab2 + 2 * sl, k1a_2, k2_2));
          zr[sl][l0] = v.x;
          zi[sl][l0] = v.y;
        }
#pragma unroll
      for (int l0 = 0; l0 < 16; ++l0) pair_dft4<false>(zr[0][l0], zi[0][l0], zr[1][l0], zi[1][l0], sg2, isB2, 8);
#pragma unroll
      for (int sl = 0; sl < 2; ++sl) {
        fft16<false>(zr[sl], zi[sl]);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          uint32_t v[16];
          tmem_ld16(tmem_s + 64 * sl + 16 * q, v);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const int k0 = 4 * q + e;
            cmul(zr[sl][k0], zi[sl][k0], u2d(v[4 * e], v[4 * e + 1]), u2d(v[4 * e + 2], v[4 * e + 3]));
          }
        }
        fft16<true>(zr[sl], zi[sl]);
      }
      // P3's inverse twiddles conj(w16^(c k1a)), applied here to the output planes only; A's
      // slot 1 (c = 2) carries -y (pair_dft4), folded into its twiddle
      const double2 w0 = sw16[(ab2 * k1a_2) & 15], w1 = sw16[((2 + ab2) * k1a_2) & 15];
      const double f2 = isB2 ? 1.0 : -1.0;
      const double u0r = w0.x, u0i = -w0.y, u1r = f2 * w1.x, u1i = -f2 * w1.y;
#pragma unroll
      for (int l0 = 0; l0 < 16; ++l0)
        if (l0 >= h && l0 < h + S) {
          pair_dft4<true>(zr[0][l0], zi[0][l0], zr[1][l0], zi[1][l0], sg2, isB2, 8);
          cmul(zr[0][l0], zi[0][l0], u0r, u0i);
          cmul(zr[1][l0], zi[1][l0], u1r, u1i);
          st2(buf + xofs(l0, ab2, k1a_2, k2_2), zr[0][l0], zi[0][l0]);
          st2(buf + xofs(l0, ab2 + 2, k1a_2, k2_2), zr[1][l0], zi[1][l0]);
        }
    }
    group_sync(grp);
    // ---- P3: (l0, c), l0 = h + tid / 8 an output plane: inverse DFT-4 over k1a -> j, inverse
    // FFT-16 along axis 2 on rows l1 = 4 j + c -> store ----
    {
      // lanes tid < 8 S own output planes; every warp runs the transforms (the pair shuffles need
      // whole warps, and a warp-uniform branch around them would make them collective
      // operations in divergent code), idle lanes read a valid slot and store nothing.  The
      // refill of the buffer waits on an mbarrier (one arrival per warp after its reads), so
      // only the issuing warp waits for the others.
      const bool act = tid < 8 * S;
      const int l0 = h + (tid >> 3);
      {
        double yr[2][16], yi[2][16];   // [slot: k1a = ab, 2 + ab -> j = ab, 2 + ab][k2 -> l2]
#pragma unroll
        for (int k2 = 0; k2 < 16; ++k2) {
          const double2 v0 = ld2(buf + xofs(l0 & 15, c, ab, k2)), v1 = ld2(buf + xofs(l0 & 15, c, 2 + ab, k2));
          yr[0][k2] = v0.x;
          yi[0][k2] = v0.y;
          yr[1][k2] = v1.x;
          yi[1][k2] = v1.y;
        }
        if (TMA) {
          // order this warp's shared reads before the next TMA write, report, and refill the
          // buffer (thread 0) while the inverse transforms and the stores run
          tma::fence_proxy_async();
          __syncwarp();
          if (lane == 0) tma::mbar_arrive(&fbar[grp]);
          if (tid == 0) {
            tma::mbar_wait(&fbar[grp], parity ^ 1);
            if (p + stride < pend) issue(p + stride);
          }
        }
        // (the inverse twiddles were applied by P2)
#pragma unroll
        for (int k2 = 0; k2 < 16; ++k2) pair_dft4<true>(yr[0][k2], yi[0][k2], yr[1][k2], yi[1][k2], sg, isB, 4);
        const PairGeom g = pair_geom(a, p);   // recomputed here: not held across the passes
        const int64_t c0 = g.o0 + l0;
        const bool row_ok = !(c0 >= a.bd.lim0 || c0 < a.win.w_lo || c0 >= a.win.w_hi);
        const bool vec = ((g.oa2 | h | a.n2 | S) & 1) == 0 && (reinterpret_cast<uintptr_t>(a.dst) & 15) == 0 &&
                         g.oa2 + h + S <= a.bd.lim2 && (!g.has_b || g.ob2 + h + S <= a.bd.lim2);
#pragma unroll
        for (int sl = 0; sl < 2; ++sl) {
          fft16<true>(yr[sl], yi[sl]);
          const double f = (sl == 1 && !isB) ? -1.0 : 1.0;   // A's slot 1 holds -row (pair_dft4)
          const int l1 = 4 * (ab + 2 * sl) + c;
          const int64_t c1 = g.o1 + l1;
          if (!act || !row_ok || l1 < h || l1 >= h + S || c1 >= a.bd.lim1) continue;
          double* drow = a.dst + ((c0 - a.win.g0) * a.n1 + c1) * a.n2;
          if (vec) {
#pragma unroll
            for (int l2 = 0; l2 < 16; l2 += 2)
              if (l2 >= h && l2 < h + S) {
                *reinterpret_cast<double2*>(drow + g.oa2 + l2) = make_double2(f * yr[sl][l2], f * yr[sl][l2 + 1]);
                if (g.has_b)
                  *reinterpret_cast<double2*>(drow + g.ob2 + l2) = make_double2(f * yi[sl][l2], f * yi[sl][l2 + 1]);
              }
          } else {
#pragma unroll
            for (int l2 = 0; l2 < 16; ++l2)
              if (l2 >= h && l2 < h + S) {
                int64_t c2 = g.oa2 + l2;
                if (c2 < a.bd.lim2) drow[c2] = f * yr[sl][l2];
                c2 = g.ob2 + l2;
                if (g.has_b && c2 < a.bd.lim2) drow[c2] = f * yi[sl][l2];
              }
          }
        }
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;\n");
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem_base), "r"(kTmemCols));
}

}  // namespace

// Three group buffers of one tile pair each (S_T is in tensor memory).
size_t fused3d_b3_smem() { return (size_t)NG * 2 * PLANE * sizeof(double) + kAlign; }

cudaError_t fused3d_b3_configure(int* max_blocks) {
  const int sm = (int)fused3d_b3_smem();
  cudaError_t e = cudaFuncSetAttribute(fft3d_b3_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(fft3d_b3_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft3d_b3_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e != cudaSuccess) return e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft3d_b3_kernel<true>, NT, sm);
  if (e == cudaSuccess && *max_blocks > 1) *max_blocks = 1;   // tensor-memory columns sized for one CTA per SM
  return e;
}

cudaError_t launch_fused3d_b3(const Fft3dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s) {
  static const CUtensorMap none = {};
  if (tm)
    fft3d_b3_kernel<true><<<grid, NT, fused3d_b3_smem(), s>>>(a, *tm);
  else if (a.bd.wrap)
    fft3d_b3_kernel<false, true><<<grid, NT, fused3d_b3_smem(), s>>>(a, none);
  else
    fft3d_b3_kernel<false><<<grid, NT, fused3d_b3_smem(), s>>>(a, none);
  return cudaGetLastError();
}

}  // namespace fstencil
