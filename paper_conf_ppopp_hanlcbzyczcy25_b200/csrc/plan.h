// Host plan builder of the FFT-stencil hot path (no CUDA in this translation unit).
//
// What it precomputes:
//   - tile extent L and valid extent S = L - 2h per axis (Splitting, Eq. 3 L167 /
//     Eq. 4, tile-length rule Eq. 5 L174-L179 re-derived for B200);
//   - DFT matrices F_L[j][k] = exp(-2 pi i (jk mod L)/L) (L192, Alg. 1; the inverse
//     is conj(F), L258, recomputed in the kernel rather than stored, L278);
//   - powered spectra S_t = sigma(2 pi k/L)^t / prod(L), t = 1..T (Eq. 10;
//     reading Q6: sigma evaluated directly from the weights);
//   - 1D: the prime-factor split N1 x N2 with the CRT (diagonal, L232) input map and
//     the Ruritanian spectrum order of Eq. 8 L216 (reading Q8);
//   - the overlap-save tile schedule, the fixed-ring boxes and the boundary-band blocks.
#pragma once

#include <cstdint>
#include <string>
#include <vector>

namespace fstencil {

constexpr int kMaxRadius = 8;

// Complex 8x8x8 products of the factored kernels (ct_line.cuh): the 3-multiply form by
// default (6 DMMA.8x8x4 + 256 FP64 adds per product of 64 outputs), else 4-multiply (8 DMMA).
#ifndef FFTSTENCIL_CMUL3
#define FFTSTENCIL_CMUL3 1
#endif
#ifndef FFTSTENCIL_CMUL3_3D
#define FFTSTENCIL_CMUL3_3D 0
#endif
constexpr bool kCmul3 = FFTSTENCIL_CMUL3 != 0;        // factored 1D and 2D kernels
constexpr bool kCmul3_3d = FFTSTENCIL_CMUL3_3D != 0;  // factored 3D kernel
constexpr double prod_dmma_flops(bool m3) { return m3 ? 6 * 512.0 : 8 * 512.0; }   // executed on the tensor pipe
constexpr double prod_flops(bool m3) { return m3 ? 6 * 512.0 + 256.0 : 8 * 512.0; }
constexpr double kProdDmmaFlops = prod_dmma_flops(kCmul3);
constexpr double kProdFlops = prod_flops(kCmul3);
constexpr int kPfaN1 = 8;     // 1D prime-factor split (gcd(8,7) = 1), N2 padded to 8
constexpr int kPfaN2 = 7;
constexpr int k3DTile = 16;   // 3D tile side (a 16^3 complex tile is 64 KiB of SMEM)
constexpr int kCt1dL = 4096;  // factored 1D tile (64 x 64 four-step Cooley-Tukey, 64 KiB per pair)

struct Box {                   // half-open box in embedded 3-axis coordinates
  int64_t lo[3];
  int64_t hi[3];
  int face = -1;               // embedded axis of the face a band box lies on
};

struct HostPlan {
  int ndim = 0, radius = 0, T = 0, h = 0;
  int64_t n[3] = {1, 1, 1};        // embedded extents (leading 1s for ndim < 3)
  int64_t ext[3] = {0, 0, 0};      // user extents (ndim entries)
  std::vector<double> w;           // (2r+1)^ndim weights
  int L[3] = {1, 1, 1};            // tile extent per user axis
  int S[3] = {1, 1, 1};            // valid extent per user axis
  int N1 = 0, N2 = 0;              // 1D split: prime-factor 8 x 7, or 64 x 64 (factored)
  int algo = 0;                    // 0 dense DFT GEMMs (1D: PFA 8x7), 1 factored (1D 64x64 CT, 2D CT 8x8, 3D 8x2),
                                   // 2 unfused 2D ablation
  int periodic = 0;                // 1: periodic boundary (no ring/band, wrap-around tiles)
  int engine = 0;                  // line-DFT engine of the factored 3D tile: 0 DFT-8 GEMMs on the
                                   // FP64 tensor pipe (kernel_fft3d_ct.cu), 1 radix-4 FFTs on the
                                   // FP64 ALU (kernel_fft3d_bf.cu); FFTSTENCIL_ENGINE=dmma|alu
  double alu_ops_per_pair = 0;     // FP64 ALU instructions per pair (engine 1: adds, muls, FMAs)
  int64_t nt[3] = {1, 1, 1};       // tiles per user axis
  int64_t tiles = 0, pairs = 0;
  int64_t npr = 1;                 // pairs per outer tile row (2D) / tile line (3D)
  // ---- outer-axis decomposition (a10; nranks = 1 on a single GPU) ----
  // Unit of the partition: one outer tile row (2D/3D: S rows) or one pair (1D: 2S cells).
  int nranks = 1, rank = 0;
  int64_t units = 0, unit_lo = 0, unit_hi = 0, pairs_per_unit = 1;
  int64_t row_lo = 0, row_hi = 0;    // owned global outer rows [row_lo, row_hi)
  int64_t g0 = 0, g1 = 0;            // buffer window: owned rows + ghosts, [g0, g1)
  int64_t pair_lo = 0, pair_hi = 0;  // this rank's tile pairs
  int64_t ipair_lo = 0, ipair_hi = 0;  // pairs whose inputs lie in owned rows (no ghosts)
  // Device-format auxiliary tables (planar re / im, row-major):
  //   2D/3D: F is L x L;  1D: F holds F_N1 (8x8) then F_N2 zero-padded to 8x8.
  std::vector<double> Fre, Fim;
  //   spectra: index t-1, each prod(tile) (1D: 8x8, Ruritanian, zero-padded).
  std::vector<std::vector<double>> Sre, Sim;
  //   1D: crt[l1*8 + l2] = tile position l stored at (l1, l2), or -1 for padding.
  std::vector<int> crt;
  //   factored 1D: w4096^(a c) at [a][c], interleaved (re, im), 2 x 4096 doubles.
  std::vector<double> tw;
  std::vector<Box> ring_boxes;     // the fixed ring, partitioned exactly
  std::vector<Box> band_boxes;     // output boxes of the band kernel (exactly-once cover)
  std::vector<int32_t> band_blocks; // 7 ints per block: out lo[3], hi[3], face axis
  int band_region_cells = 0;       // max SMEM region (cells) of one band block at t = T
  double flops_per_cell_step = 0;  // algorithmic (unpadded dense-DFT tile)
  double mma_flops_per_pair = 0;   // executed by the fused kernel (padded)
  size_t fused_smem = 0;
};

// Builds the plan; returns 0 or a negative FFTSTENCIL_* code with `err` set.
// nranks/rank select one slab of the outer-axis decomposition (1/0 = whole grid).
// algo: -1 = choose by the cost model, 0 = dense (1D: PFA 8 x 7), 1 = factored, 2 = unfused (2D).
int build_host_plan(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                    HostPlan& p, std::string& err, int nranks = 1, int rank = 0, int algo = -1,
                    int periodic = 0);

// Pipelined run_host schedule: ops of 4 int64 {op, x, y, z} in issue order.
//   op 0: copy input rows [x, y) host -> device (then the run stream waits for it);
//   op 1: copy the fixed ring's rows [x, y) from the input into both pass buffers;
//   op 2: pass x (1-based) on outer tile rows ("units") [y, z): fused pairs and band rows;
//   op 3: copy result rows [x, y) device -> host once everything before it is done.
// Returns 0 with the ops, or FFTSTENCIL_EINVAL when the plan is not eligible (1D, periodic,
// a slab plan, the unfused ablation, h > S, fewer than 2K units, no steps).
// Qt: skewed passes of the tail (<= 0: Q); ramp: 1 small first input / last output chunk, 2 also a
// small last input / first output chunk.
int build_e2e_schedule(const HostPlan& p, int64_t total_steps, int K, int Q, std::vector<int64_t>& ops, int Qt = 0,
                       int ramp = 1);

// Peer-transport run of one rank (capi.cu run_dist_peer executes exactly this list): ops of 4
// int64 {op, a, b, c} in stream order, epochs absolute (the rank has sent `epoch0` signals before):
//   0 WAIT e        the stream waits until both neighbours have signalled >= e times;
//   1 COPYIN        the caller's slab -> owned rows of buffer 0 (+ fixed ring into buffer 1);
//   2 PUSH f, t     own boundary rows of buffer f -> the neighbours' halo rows of their buffer t;
//   3 SIGNAL e      write e into both neighbours' flag words (this rank's e-th signal);
//   4 INTERIOR k, s      pass k's halo-free tile pairs: reads owned rows of buffer s, writes rows
//                        [row_lo + h, row_hi - h) of buffer s ^ 1;
//   5 EDGE k, s, f       pass k's edge pairs and band: reads rows [g0, g1) of s (halos included),
//                        writes the owned boundary rows of s ^ 1 and, if f, the same rows into
//                        the neighbours' buffer s ^ 1 (fused stores);
//   6 COPYOUT s     owned rows of buffer s -> the caller's slab.
int build_peer_schedule(const HostPlan& p, int64_t total_steps, bool fused, int64_t epoch0, std::vector<int64_t>& ops);

// Dense-DFT tile cost model (executed FP64 tensor flops per cell-step) used to pick L/T.
double model_flops_2d(int L, int S, int T);
// Factored (CT 8 x 8, L = 64) tile: executed FP64 flops per cell-step (DMMA + twiddles + S_T).
double model_flops_2d_ct(int S, int T);

}  // namespace fstencil
