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
// Compile-time ablations (all 0 by default; each measured slower on B200, DESIGN.md §13,
// profiles/r01_s3_ab2d.txt): BF_TW_REG (twiddle powers in registers), BF_TW_COMB (combined
// twiddles), BF_WARP_LOCAL (warp-local row passes), BF_TMEM_S (S_T in tensor memory),
// BF_PINGPONG (the two groups alternate memory and compute phases), BF_CPLX (interleaved
// complex words after P1).  Build one with FFTSTENCIL_NVCC_DEFS="-DBF_...=1".
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

// BF_WARP_LOCAL = 1: P1 rewrites its rows in the layout wn (row swizzle gn below instead of the
// TMA's r & 7), and P2 / P4 give warp w exactly the eight rows 16 i + 2 w + e (i = 0..3,
// e = 0..1) its P1 / P5 blocks cover (lane = 8 b + 2 i + e, b = column block).  P1 -> P2 and
// P4 -> P5 then exchange data only inside a warp (__syncwarp instead of a group barrier: three
// group barriers per pair instead of five).  gn = i | e << 2 is distinct over a warp's eight
// rows, so a quarter-warp's eight 16-byte row-pass words stay conflict-free; the row and
// column segments of P1 / P3 / P5 are conflict-free under any row swizzle.
#ifndef BF_WARP_LOCAL
#define BF_WARP_LOCAL 0
#endif
__device__ __forceinline__ int gn(int r) { return BF_WARP_LOCAL ? (((r >> 4) & 3) | ((r & 1) << 2)) : (r & 7); }
__device__ __forceinline__ int wn(int r, int c) { return ((c >> 4) << 10) | (r << 4) | ((c & 15) ^ (gn(r) << 1)); }

// BF_CPLX = 1: after P1 every element is one 16-byte (re, im) word.  Row r's 64 complex values
// occupy exactly the bytes row r had in the two TMA planes (1 KB: four 128-byte segments per
// plane): columns 16 b + 0..7 in the Re plane's segment b, 16 b + 8..15 in the Im plane's, as
// 16-byte chunk (c & 7) ^ (r & 7).  A half-warp of P1 owns four whole rows, so it converts them
// in place after a __syncwarp.  Every later access moves one complex value per instruction
// (LDS.128 / STS.128): 176 shared-memory instructions per thread and pair instead of 240, the
// same wavefronts (a quarter-warp covers 8 chunks of one segment: 8 consecutive columns of a row
// in P1 / P3 / P5, 8 consecutive rows of a column chunk in P2 / P4 -> distinct banks).
#ifndef BF_CPLX
#define BF_CPLX 0
#endif
static_assert(!(BF_CPLX && BF_WARP_LOCAL), "BF_CPLX and BF_WARP_LOCAL are exclusive");
// double offset of element (r, c)'s (re, im) word from the group buffer base sR
__device__ __forceinline__ int wc(int r, int c) {
  return (((c >> 3) & 1) << 12) | ((c >> 4) << 10) | (r << 4) | (((c & 7) ^ (r & 7)) << 1);
}
__device__ __forceinline__ void ldc2(const double* b, int o, double& re, double& im) {
  const double2 v = *reinterpret_cast<const double2*>(b + o);
  re = v.x;
  im = v.y;
}
__device__ __forceinline__ void stc2(double* b, int o, double re, double im) {
  *reinterpret_cast<double2*>(b + o) = make_double2(re, im);
}

__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}

using radix::cmul;
using radix::dft4;
using radix::fft16;

// BF_TMEM_S = 1: S_T lives in tensor memory instead of shared memory (P3 reads it with
// tcgen05.ld, a data path of its own, taking 512 wavefronts per pair off shared memory).
// Per TMEM lane 32 (w & 3) + lane of a group-local warp w: the S values of P3 column
// rc = lane + 32 (w & 1), row block (w >> 1), set s = w >> 2 -> columns 64 s + 4 k + {re lo,
// re hi, im lo, im hi}, k = 0..15; both groups share them (128 columns).
#ifndef BF_TMEM_S
#define BF_TMEM_S 0
#endif

__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t (&v)[8]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
}
// 16 columns (4 complex S values) in one load, one wait (BF_TMEM_S = 2).
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
__device__ __forceinline__ double u2d(uint32_t lo, uint32_t hi) {
  return __hiloint2double((int)hi, (int)lo);
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

// BF_PINGPONG = 1: the two groups take turns at shared memory (the FA3 "ping-pong" schedule).
// Each pass of a group is a memory phase M (the previous pass's shared stores, the group
// barrier, this pass's shared loads) followed by a compute phase C (butterflies in registers);
// group g starts an M phase with bar.sync on barrier 3 + g and ends it -- once its loads have
// returned -- with bar.arrive on the other group's barrier, so one group's butterflies run
// while the other group moves data.  Group 0 skips the wait of its very first phase and group 1
// the arrive of its very last one (group 1, which may own one pair fewer, pads with turns that
// do no work), so the two barriers see matched sync / arrive counts.
#ifndef BF_PINGPONG
#define BF_PINGPONG 0
#endif
__device__ __forceinline__ void pp_begin(int grp, bool first_phase) {
  if (BF_PINGPONG && !(grp == 0 && first_phase))
    asm volatile("bar.sync %0, %1;\n" ::"r"(3 + grp), "r"(2 * NT) : "memory");
}
// a0..a3: loaded values, so the arrive waits for the phase's loads to return
// (BF_PINGPONG = 2: arrive as soon as the loads are issued)
__device__ __forceinline__ void pp_end(int grp, bool last_phase, double a0, double a1, double a2, double a3) {
  if (BF_PINGPONG == 1 && !(grp == 1 && last_phase))
    asm volatile("bar.arrive %0, %1;\n" ::"r"(4 - grp), "r"(2 * NT), "d"(a0), "d"(a1), "d"(a2), "d"(a3) : "memory");
  if (BF_PINGPONG == 2 && !(grp == 1 && last_phase))
    asm volatile("bar.arrive %0, %1;\n" ::"r"(4 - grp), "r"(2 * NT) : "memory");
}

// The 4 x 4 block of P1/P5: element [i][j] at row 16 i + rr, column 16 j + cc.
template <bool TMA_LAYOUT>
__device__ __forceinline__ void load_block(const double* sR, const double* sI, int rr, int cc, double (&xr)[4][4],
                                           double (&xi)[4][4]) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (BF_CPLX && !TMA_LAYOUT) {
        ldc2(sR, wc(16 * i + rr, 16 * j + cc), xr[i][j], xi[i][j]);
        continue;
      }
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

// element [i][j] *= w64^(+-(rr i + cc j)) (conjugate if INV).  BF_TW_REG = 1: two table loads
// (w64^rr, one address per half-warp; w64^cc, 16 consecutive words) and their squares and cubes
// formed in registers (16 FP64 instructions instead of four more lane-varying shared-memory
// loads, which conflict for j = 2); BF_TW_REG = 0: all six powers from the shared w64^m table.
#ifndef BF_TW_REG
#define BF_TW_REG 0
#endif
// BF_TW_COMB = 1: one multiply by the combined w64^(rr i + cc j) per element (15 complex
// multiplies, 15 table loads) instead of a row and a column twiddle (24 multiplies, 6 loads).
#ifndef BF_TW_COMB
#define BF_TW_COMB 0
#endif

__device__ __forceinline__ void powers3(double2 w, double2 (&p)[4]) {
  p[1] = w;
  p[2] = make_double2(fma(w.x, w.x, -w.y * w.y), 2.0 * (w.x * w.y));
  p[3] = make_double2(fma(w.x, p[2].x, -w.y * p[2].y), fma(w.x, p[2].y, w.y * p[2].x));
}

template <bool INV>
__device__ __forceinline__ void twiddle4x4(double (&xr)[4][4], double (&xi)[4][4], const double2* tw, int rr,
                                           int cc) {
  if (BF_TW_COMB) {
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (i | j) {
          const double2 w = tw[(rr * i + cc * j) & 63];
          cmul(xr[i][j], xi[i][j], w.x, INV ? -w.y : w.y);
        }
    return;
  }
  double2 pr[4], pc[4];
  if (BF_TW_REG) {
    powers3(tw[rr], pr);
    powers3(tw[cc], pc);
  } else {
#pragma unroll
    for (int i = 1; i < 4; ++i) {
      pr[i] = tw[(rr * i) & 63];
      pc[i] = tw[(cc * i) & 63];
    }
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

// P2/P4: the 16 columns 16 b + m of row r as 16-byte words (chunk (m >> 1) ^ gn(r)).
__device__ __forceinline__ void row_load(const double* sR, const double* sI, int r, int b, double (&xr)[16],
                                         double (&xi)[16]) {
  if (BF_CPLX) {
#pragma unroll
    for (int m = 0; m < 16; ++m) ldc2(sR, wc(r, 16 * b + m), xr[m], xi[m]);
    return;
  }
  const int base = (b << 10) | (r << 4), s = gn(r);
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
  if (BF_CPLX) {
#pragma unroll
    for (int m = 0; m < 16; ++m) stc2(sR, wc(r, 16 * b + m), xr[m], xi[m]);
    return;
  }
  const int base = (b << 10) | (r << 4), s = gn(r);
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
    if (BF_CPLX) {
      ldc2(sR, wc(16 * blk + m, rc), xr[m], xi[m]);
      continue;
    }
    const int o = wn(16 * blk + m, rc);
    xr[m] = sR[o];
    xi[m] = sI[o];
  }
}
__device__ __forceinline__ void col_store(double* sR, double* sI, int rc, int blk, const double (&xr)[16],
                                          const double (&xi)[16]) {
#pragma unroll
  for (int m = 0; m < 16; ++m) {
    if (BF_CPLX) {
      stc2(sR, wc(16 * blk + m, rc), xr[m], xi[m]);
      continue;
    }
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
      if (BF_CPLX) {
        stc2(sR, wc(16 * i + rr, 16 * j + cc), xr[i][j], xi[i][j]);
        continue;
      }
      const int o = wn(16 * i + rr, 16 * j + cc);
      sR[o] = xr[i][j];
      sI[o] = xi[i][j];
    }
}

// The five passes over the pair in (sR, sI) by group `grp`, whose tile data are in place (the
// caller waited for them in the first memory phase); releases the buffer (TMA refill of the
// group's next pair `gn`) after P5's reads, then stores the window.  M / C mark the memory and
// compute phases of the ping-pong schedule (BF_PINGPONG).
template <bool TMA, bool PEER>
__device__ __forceinline__ void tile_passes(double* sR, double* sI, const double* sS, const double2* tw,
                                            const Fft2dArgs& a, const Geom& g, int warp, int lane, int grp,
                                            const CUtensorMap* tm, uint64_t* bar, bool has_next, const Geom& gn,
                                            uint32_t tmem_s, bool last) {
  const int S = a.S, h = a.h;
  const int rr = (warp << 1) | (lane >> 4), cc = lane & 15;     // P1/P5 block classes
  const int rc = lane + ((warp & 1) << 5), blk = warp >> 1;      // P3 column, row block
  // P2/P4 row and column block (BF_WARP_LOCAL: the warp's P1/P5 rows)
  const int r2 = BF_WARP_LOCAL ? ((((lane & 7) >> 1) << 4) | (warp << 1) | (lane & 1)) : rc;
  const int b2 = BF_WARP_LOCAL ? (lane >> 3) : blk;
  double xr[16], xi[16];
  {
    // ---- P1 (M: loads) (C: stage 1 of both axes) ----
    double br[4][4], bi[4][4];
    load_block<true>(sR, sI, rr, cc, br, bi);
    pp_end(grp, false, br[0][0], bi[0][0], br[3][3], bi[3][3]);
    dft4x4<false>(br, bi);
    twiddle4x4<false>(br, bi, tw, rr, cc);
    // ---- P2 (M: P1 stores, barrier, loads) (C: axis 1, DFT-16 along row r2, block b2) ----
    pp_begin(grp, false);
    if (BF_WARP_LOCAL || BF_CPLX) __syncwarp();   // the warp's rows are rewritten in layout wn / wc
    block_store(sR, sI, rr, cc, br, bi);
  }
  if (BF_WARP_LOCAL) __syncwarp(); else group_sync(grp);
  row_load(sR, sI, r2, b2, xr, xi);
  pp_end(grp, false, xr[0], xi[0], xr[15], xi[15]);
  fft16<false>(xr, xi);
  // ---- P3 (M: P2 stores, barrier, loads) (C: axis 0 DFT-16 down column rc in row block blk,
  //      * S_T, inverse DFT-16) ----
  pp_begin(grp, false);
  row_store(sR, sI, r2, b2, xr, xi);
  group_sync(grp);
  col_load(sR, sI, rc, blk, xr, xi);
  pp_end(grp, false, xr[0], xi[0], xr[15], xi[15]);
  fft16<false>(xr, xi);   // slot k': position 16 blk + k' <-> frequency blk + 4 k'
  if (BF_TMEM_S == 2) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {   // 4 complex values per 16-column load
      uint32_t v[16];
      tmem_ld16(tmem_s + 16 * q, v);
#pragma unroll
      for (int e = 0; e < 4; ++e)
        cmul(xr[4 * q + e], xi[4 * q + e], u2d(v[4 * e], v[4 * e + 1]), u2d(v[4 * e + 2], v[4 * e + 3]));
    }
  } else if (BF_TMEM_S) {
#pragma unroll
    for (int q = 0; q < 8; ++q) {   // 2 complex values per 8-column load
      uint32_t v[8];
      tmem_ld8(tmem_s + 8 * q, v);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        cmul(xr[2 * q + e], xi[2 * q + e], u2d(v[4 * e], v[4 * e + 1]), u2d(v[4 * e + 2], v[4 * e + 3]));
    }
  } else {
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      const double2 sv = *reinterpret_cast<const double2*>(sS + ((((16 * blk + k) << 6) + rc) << 1));
      cmul(xr[k], xi[k], sv.x, sv.y);
    }
  }
  fft16<true>(xr, xi);
  // ---- P4 (M: P3 stores, barrier, loads) (C: axis 1 inverse DFT-16) ----
  pp_begin(grp, false);
  col_store(sR, sI, rc, blk, xr, xi);
  group_sync(grp);
  row_load(sR, sI, r2, b2, xr, xi);
  pp_end(grp, false, xr[0], xi[0], xr[15], xi[15]);
  fft16<true>(xr, xi);
  // ---- P5 (M: P4 stores, barrier, loads, release) (C: conj twiddles, inverse stage 1 of both
  //      axes, store the window) ----
  pp_begin(grp, false);
  row_store(sR, sI, r2, b2, xr, xi);
  if (BF_WARP_LOCAL) __syncwarp(); else group_sync(grp);
  double br[4][4], bi[4][4];
  load_block<false>(sR, sI, rr, cc, br, bi);
  if (TMA) tma::fence_proxy_async();   // the buffer is refilled by TMA after the barrier
  group_sync(grp);
  if (TMA && warp == 0 && lane == 0 && has_next) issue_pair(a, tm, gn, sR, bar);
  pp_end(grp, last, br[0][0], bi[0][0], br[3][3], bi[3][3]);
  twiddle4x4<true>(br, bi, tw, rr, cc);
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
    if (PEER) {   // boundary rows of a peer-transport rank: the same cells into the neighbour's halo row
      const int64_t c0 = g.o0 + r;
      double* prow = c0 < a.peer.lo_end ? a.peer.lo + (c0 - a.peer.lo_g0) * a.n1
                   : c0 >= a.peer.hi_begin ? a.peer.hi + (c0 - a.peer.hi_g0) * a.n1 : nullptr;
      if (prow) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          if (va[j]) prow[ca + 16 * j] = br[i][j];
          if (vb[j]) prow[cb + 16 * j] = bi[i][j];
        }
      }
    }
  }
}

// PEER: boundary rows of a peer-transport rank are also stored into the neighbour (a.peer,
// kernels.cuh); a separate instantiation, the single-GPU kernel is unchanged.
template <bool TMA, bool WRAP = false, bool PEER = false>
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
  if (threadIdx.x < L) tw[threadIdx.x] = make_double2(a.Fre[threadIdx.x], a.Fim[threadIdx.x]);
  __shared__ uint32_t tmem_base;
  uint32_t tmem_s = 0;
  if (BF_TMEM_S) {
    if (threadIdx.x < 32) {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;\n" ::"r"(tma::smem_addr(&tmem_base)));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n");
    // this thread's lane quadrant and column set (see BF_TMEM_S)
    tmem_s = tmem_base + ((uint32_t)(32 * (warp & 3)) << 16) + 64 * (warp >> 2);
    if (grp == 0) {   // group 0 fills the (shared) S values of its P3 lines
      const int rc = lane + ((warp & 1) << 5), blk = warp >> 1;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint32_t v[16];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int idx = ((16 * blk + 4 * q + e) << 6) + rc;
          const double re = __ldg(a.Sre + idx), im = __ldg(a.Sim + idx);
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
  } else {
    for (int e = threadIdx.x; e < PLANE; e += 2 * NT)   // once per launch
      *reinterpret_cast<double2*>(sS + 2 * e) = make_double2(__ldg(a.Sre + e), __ldg(a.Sim + e));
  }
  __syncthreads();
  if (BF_TMEM_S) asm volatile("tcgen05.fence::after_thread_sync;\n");
  const int64_t stride = 2 * (int64_t)gridDim.x;
  const int64_t p0 = a.win.p_begin + 2 * (int64_t)blockIdx.x + grp;
  if (TMA && tid == 0 && p0 < a.win.p_end) issue_pair(a, &tm, geom(a, p0), sR, &bar[grp]);

  // pairs of this group and of group 0 (which owns as many as group 1 or one more)
  const int64_t pb0 = a.win.p_begin + 2 * (int64_t)blockIdx.x;
  const int64_t n0 = pb0 < a.win.p_end ? (a.win.p_end - pb0 + stride - 1) / stride : 0;
  const int64_t nmine = p0 < a.win.p_end ? (a.win.p_end - p0 + stride - 1) / stride : 0;
  const int64_t niter = BF_PINGPONG ? n0 : nmine;
  uint32_t parity = 0;
  for (int64_t it = 0; it < niter; ++it) {
    const int64_t p = p0 + it * stride;
    const bool last = it == niter - 1;
    if (it >= nmine) {   // ping-pong turns without work (group 1)
#pragma unroll 1
      for (int k = 0; k < 5; ++k) {
        pp_begin(grp, false);
        pp_end(grp, last && k == 4, 0.0, 0.0, 0.0, 0.0);
      }
      continue;
    }
    const Geom g = geom(a, p);
    pp_begin(grp, it == 0);   // M of P1: the tile's arrival and P1's loads
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
    tile_passes<TMA, PEER>(sR, sI, sS, tw, a, g, warp, lane, grp, &tm, &bar[grp], has_next, gn, tmem_s, last);
  }
  if (BF_TMEM_S) {
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n");
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;\n" ::"r"(tmem_base));
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
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft2d_bf_kernel<true, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, st);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fft2d_bf_kernel<false, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sc);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(max_blocks, fft2d_bf_kernel<true>, 2 * NT, st);
}

cudaError_t launch_fused2d_bf(const Fft2dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s) {
  static const CUtensorMap none = {};
  if (a.peer.lo || a.peer.hi) {   // boundary rows of a peer-transport rank (never periodic)
    if (tm)
      fft2d_bf_kernel<true, false, true><<<grid, 2 * NT, fused2d_bf_smem(true), s>>>(a, *tm);
    else
      fft2d_bf_kernel<false, false, true><<<grid, 2 * NT, fused2d_bf_smem(false), s>>>(a, none);
    return cudaGetLastError();
  }
  if (tm)
    fft2d_bf_kernel<true><<<grid, 2 * NT, fused2d_bf_smem(true), s>>>(a, *tm);
  else if (a.bd.wrap)
    fft2d_bf_kernel<false, true><<<grid, 2 * NT, fused2d_bf_smem(false), s>>>(a, none);
  else
    fft2d_bf_kernel<false><<<grid, 2 * NT, fused2d_bf_smem(false), s>>>(a, none);
  return cudaGetLastError();
}

}  // namespace fstencil
