// Kernel argument blocks and launchers of the fused FFT-stencil path (sm_100a).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

namespace fstencil {

// Outer-axis window of one launch (multi-GPU decomposition).  The source
// and destination buffers hold global axis-0 rows [g0, g0 + gn); the launch processes
// tile pairs [p_begin, p_end) and writes only global axis-0 rows [w_lo, w_hi).  Input rows
// outside the buffer read as zero (they only influence rows the launch does not write).
// Single GPU: g0 = 0, gn = n0, [w_lo, w_hi) = [0, n0), all pairs.
struct Window {
  int64_t g0, gn;
  int64_t w_lo, w_hi;
  int64_t p_begin, p_end;
};

// Boundary handling of a launch (NEXT-2).  Fixed ring: wrap = 0, shift = 0, lim = n - h.
// Periodic: wrap = 1, shift = -h, lim = n.  Tile t covers cells t*S + shift + [0, L) (taken
// modulo n when wrapping, else zero outside the grid) and writes cells t*S + shift + h + l,
// l in [0, S), below lim on every axis.
struct Bound {
  int wrap;
  int shift;
  int64_t lim0, lim1, lim2;
};

// Fused halo push of the peer transport (capi.cu run_dist_peer): a launch that produces a rank's
// boundary rows also stores every cell of global outer-axis row c < lo_end into the lower
// neighbour's buffer `lo` (an IPC-mapped pointer; its row 0 is global row lo_g0) and of row
// c >= hi_begin into the upper neighbour's `hi` (row 0 = hi_g0), so the exchange is the pass's own
// stores over NVLink, tile by tile.  lo / hi null: no such neighbour, or a launch without them.
struct PeerStore {
  double* lo;
  double* hi;
  int64_t lo_end, lo_g0, hi_begin, hi_g0;
};

__host__ __device__ __forceinline__ int64_t wrap_index(int64_t x, int64_t n) {
  x %= n;
  return x < 0 ? x + n : x;
}

// Tile pairs (Double-layer Filling, Eq. 9): tiles are paired along the innermost tile axis
// within one row of tiles -- (.., 2j) with (.., 2j+1); an odd row count pairs the last tile
// with zeros.  Pairs never straddle an outer-axis tile row, so a decomposition into whole
// tile rows computes exactly the single-GPU pairs (bitwise-equal results).

// One fused pass of the 2D path over every tile pair (kernel_fft2d.cu).
struct Fft2dArgs {
  const double* src;
  double* dst;
  int64_t n0, n1;        // grid extents
  int h, S;              // halo r*T (tile geometry) and valid side L - 2h
  int64_t nt1;           // tiles along axis 1
  int64_t npr;           // pairs per tile row = ceil(nt1 / 2)
  Window win;
  Bound bd;
  const double* Fre;     // L x L forward DFT matrix, row-major, columns permuted (perm8)
  const double* Fim;
  const double* Sre;     // L x L powered spectrum of this pass, natural row-major
  const double* Sim;
  double* spec;          // unfused ablation only: [pair][re|im][k0][k1] spectrum in HBM
  PeerStore peer;        // multi-GPU peer transport: boundary rows also stored to the neighbours
};

// One fused pass of the 1D path: prime-factor 8 x 7 tile (kernel_fft1d.cu) or the
// factored 4096 = 64 x 64 tile (kernel_fft1d_ct.cu).
struct Fft1dArgs {
  const double* src;
  double* dst;
  int64_t n;
  int h, S, L;           // L = N1*N2 = 56 (PFA) or 4096 (factored)
  int64_t ntiles;        // pair p holds tiles 2p and 2p+1
  Window win;
  Bound bd;
  const double* Fre;     // 16 x 8: rows 0..7 F_N1, rows 8..15 F_N2 zero-padded
  const double* Fim;
  const double* Sre;     // 8 x 8 Ruritanian-ordered powered spectrum, zero-padded
  const double* Sim;
  const int* crt;        // PFA: 64 tile positions stored at (l1, l2), -1 = padding
  const double* tw;      // factored: w4096^(a c) at [a][c], interleaved (re, im)
  PeerStore peer;        // multi-GPU peer transport: boundary rows also stored to the neighbours
};

// One fused pass of the 3D path over every tile pair (kernel_fft3d.cu); 16^3 tiles.
struct Fft3dArgs {
  const double* src;
  double* dst;
  int64_t n0, n1, n2;
  int h, S;
  int64_t nt1, nt2;      // tiles along axes 1 and 2
  int64_t npr;           // pairs per (t0, t1) tile line = ceil(nt2 / 2)
  Window win;
  Bound bd;
  const double* Fre;     // 16 x 16 forward DFT matrix
  const double* Fim;
  const double* Sre;     // powered spectrum in [k1][k2][k0] order
  const double* Sim;
  // ALU kernel traversal order (kernel_fft3d_bf.cu pair_geom): blocks of blk0 outer tile rows x
  // blk1 tile lines, so the axis-0 / axis-1 halo overlap of neighbouring tiles is re-read from L2
  // instead of HBM; 0 = natural pair order.  Launch ranges are whole outer tile rows.
  int blk0, blk1;
  // ALU kernel output rows (vector path): bit l2 of st32 = 32-byte store of l2 .. l2 + 3, of st16 =
  // 16-byte store of l2, l2 + 1, for l2 in [h, h + S).  launch_fused sets st32 only when every
  // tile row starts 32-byte aligned (S, n2 multiples of 4, no shift, dst 32-byte aligned).
  int st32, st16;
  PeerStore peer;        // multi-GPU peer transport: boundary rows also stored to the neighbours
};

// Direct T-step recomputation of the boundary band (kernel_band.cu).
struct BandArgs {
  const double* src;
  double* dst;
  int64_t n[3];          // embedded extents (leading 1s)
  int active[3];
  int r, t;              // radius, steps of this pass
  const double* w;       // (2r+1)^ndim weights, offset-cube row-major
  const int* blocks;     // 8 ints per block: lo[3], hi[3], face, pad (global coordinates)
  int nblocks;
  int oax;               // embedded index of the outer axis (3 - ndim)
  int64_t g0, gn;        // buffers hold global outer-axis rows [g0, g0 + gn)
  int reference;         // 1: the first (unoptimised) band kernel, for ablation/tests
  int region_cells;      // host hint: largest block region (cells) at t = T -- sizes the 1D CTA
  int ntaps;             // host hint: nonzero weights (selects a register-tap specialisation)
  int64_t clip_lo, clip_hi;   // only outer-axis rows [clip_lo, clip_hi) are produced (pipelined run_host)
  PeerStore peer;        // multi-GPU peer transport: boundary rows also stored to the neighbours
};

// Copy a box (embedded coordinates) from src to dst0 and dst1 (either may be null).
struct BoxCopyArgs {
  const double* src;
  double* dst0;
  double* dst1;
  int64_t n[3];
  int64_t lo[3], hi[3];  // global embedded coordinates
  int oax;               // embedded index of the outer axis
  int64_t src_off, dst_off;   // global outer-axis row of buffer row 0 (src / dst0 and dst1)
};

// V: kernel variant (kernel_fft2d.cu header): 0 sync loads, 1 cp.async double buffer,
// 2 double buffer + F through L1.  Fre/Fim for the 2D kernel are column-permuted (perm8).
int fused2d_threads(int L);
size_t fused2d_smem(int L, int V);
cudaError_t fused2d_configure(int L, int V, int* max_blocks_per_sm);
cudaError_t launch_fused2d(int L, int V, const Fft2dArgs& a, int grid, cudaStream_t s);
// Unfused ablation (NEXT-3): stage 1 = forward DFT -> a.spec, stage 2 = a.spec -> inverse + store,
// launch_spec_mul in between (spectrum *= S_t in HBM).
cudaError_t launch_unfused2d(int L, int stage, const Fft2dArgs& a, int grid, cudaStream_t s);
cudaError_t launch_spec_mul(double* spec, int64_t npairs, int L, const double* Sre, const double* Sim, cudaStream_t s);

// Factored-DFT 2D kernel (kernel_fft2d_ct.cu): L = 64 = 8 x 8 Cooley-Tukey per axis.
// Fre/Fim = [F8 (8x8) | twiddles w64^(ka lb) (8x8)]; Sre/Sim = S_T in [k1][8 g + c] order with
// k0 = g + 8 c.  cfg = 10 * (warps per CTA) + (lines per warp step): 81, 82, 84, 161, 162.
size_t fused2d_ct_smem();
cudaError_t fused2d_ct_configure(int cfg, int* max_blocks_per_sm);
// tm: tensor map of the source buffer (dims {n1, gn}, box {64, 64}) or null (cp.async path).
cudaError_t launch_fused2d_ct(int cfg, const Fft2dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s);

constexpr int kFft1dWarpsPerBlock = 8;
cudaError_t fused1d_configure(int* max_blocks_per_sm);
cudaError_t launch_fused1d(const Fft1dArgs& a, int grid, cudaStream_t s);

// A whole fftstencil_run of a small non-periodic 1D PFA plan in one launch of one CTA, the grid
// resident in shared memory (kernel_small1d.cu).
constexpr int64_t kSmall1dMaxCells = 8192;   // 2 buffers = 128 KB of shared memory
constexpr int kSmall1dMaxBand = 64;          // cells of one band cone region, h + r t <= 2h < 56
constexpr int kSmall1dMaxR = 8;              // radius limit of the C ABI
struct Small1dArgs {
  const double* in;      // global grid (read once)
  double* out;           // global grid (written once; may alias in)
  int64_t n;
  int h, S, L, r, T, rem, rmax;   // rem = steps mod T (0: none); rmax = min(h + r T, n)
  int64_t ntiles, passes;
  const double* Fre;     // as Fft1dArgs
  const double* Fim;
  const int* crt;
  const double* Sre_T;   // powered spectra S_T and S_rem (Ruritanian 8 x 8)
  const double* Sim_T;
  const double* Sre_rem;
  const double* Sim_rem;
  const double* w;       // 2r + 1 weights
};
size_t small1d_smem(int64_t n, int rmax);
cudaError_t small1d_configure();
cudaError_t launch_small1d(const Small1dArgs& a, cudaStream_t s);
size_t fused1d_ct_smem();
// Butterfly ALU engine of the factored 1D tile (kernel_fft1d_bf.cu): Fre/Fim[0..63] = w64^m,
// tw = w4096^m (m < 256, interleaved); Sre/Sim = S_T at [column position][row position].
// tm: the buffer as rows of 64 cells (dims {64, gn / 64}, box {16, 64}, SWIZZLE_128B) or null.
size_t fused1d_bf_smem();
cudaError_t fused1d_bf_configure(int* max_blocks_per_sm);
cudaError_t launch_fused1d_bf(const Fft1dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s);
cudaError_t fused1d_ct_configure(int* max_blocks_per_sm);
cudaError_t launch_fused1d_ct(const Fft1dArgs& a, int grid, cudaStream_t s);

size_t fused3d_smem();
cudaError_t fused3d_configure(int* max_blocks_per_sm);
cudaError_t launch_fused3d(const Fft3dArgs& a, int grid, cudaStream_t s);

// Factored 3D kernel (kernel_fft3d_ct.cu): 16 = 8 x 2 per axis.  Fre/Fim = [F8 (8x8) | w16^k,
// k = 0..15]; Sre/Sim = S_T in [k1][k2][k0 % 8][k0 / 8] order.
size_t fused3d_ct_smem();
cudaError_t fused3d_ct_configure(int* max_blocks_per_sm);
// tm: tensor map of the source buffer (dims {n2, n1, gn}, box {16, 16, 16}) or null (cp.async).
cudaError_t launch_fused3d_ct(const Fft3dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s);

// Radix-8 ALU engine of the factored 2D tile (kernel_fft2d_bf.cu): 64 = 8 x 8 Cooley-Tukey with
// DFT-8 butterflies in registers.  Fre/Fim[0..63] = w64^m; Sre/Sim = S_T in position order
// (position 8a + b <-> frequency a + 8b per axis).  tm: dims {n1, gn}, box {16, 64}, SWIZZLE_128B.
size_t fused2d_bf_smem(bool tma);
cudaError_t fused2d_bf_configure(int* max_blocks_per_sm);
cudaError_t launch_fused2d_bf(const Fft2dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s);

// Radix-4 ALU engine of the factored 3D tile (kernel_fft3d_bf.cu): 16-point line FFTs in
// registers; Sre/Sim = S_T in natural [k0][k1][k2] order.  tm: as for fft3d_ct but encoded with
// SWIZZLE_128B.
size_t fused3d_bf_smem(bool tma);
cudaError_t fused3d_bf_configure(int* max_blocks_per_sm);
cudaError_t launch_fused3d_bf(const Fft3dArgs& a, const CUtensorMap* tm, int grid, cudaStream_t s);

constexpr int kBandThreads = 256;
cudaError_t band_configure(size_t smem);
cudaError_t launch_band(const BandArgs& a, size_t smem, cudaStream_t s);

cudaError_t launch_box_copy(const BoxCopyArgs& a, cudaStream_t s);

}  // namespace fstencil
