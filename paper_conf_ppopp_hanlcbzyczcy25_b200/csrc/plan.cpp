// Host plan builder (see plan.h).  Pure C++: no CUDA here, so the builder can be
// exercised by the CPU test-suite through fftstencil_describe / fftstencil_export_aux.
#include "plan.h"

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <cmath>
#include <complex>

#include "fftstencil.h"

namespace fstencil {
namespace {

using cplx = std::complex<double>;
constexpr double kTwoPi = 6.283185307179586476925286766559;

int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
int round8(int x) { return (x + 7) / 8 * 8; }

// exp(-2 pi i m / L) with the argument reduced to [0, L) first (SURVEY §7 pitfall 6).
cplx root(int64_t m, int64_t L) {
  m %= L;
  if (m < 0) m += L;
  const double a = -kTwoPi * (double)m / (double)L;
  return cplx(std::cos(a), std::sin(a));
}

// sigma(theta_k) = sum_o w[o] exp(+i o.theta_k), theta_a = 2 pi k_a / L_a  (reading Q6/Q7).
// exp(+i o 2 pi k / L) = root(-o k, L): reduced per axis, multiplied across axes.
cplx symbol(const HostPlan& p, const int* k, const int* L) {
  const int r = p.radius, wd = 2 * r + 1, nd = p.ndim;
  cplx acc(0.0, 0.0);
  const int total = (int)p.w.size();
  for (int idx = 0; idx < total; ++idx) {
    const double wv = p.w[idx];
    if (wv == 0.0) continue;
    int rem = idx;
    int o[3] = {0, 0, 0};
    for (int a = nd - 1; a >= 0; --a) { o[a] = rem % wd - r; rem /= wd; }
    cplx ph(1.0, 0.0);
    for (int a = 0; a < nd; ++a) ph *= root(-(int64_t)o[a] * k[a], L[a]);
    acc += wv * ph;
  }
  return acc;
}

void fill_dft(int L, int ld, int row0, int col0, std::vector<double>& re, std::vector<double>& im) {
  for (int j = 0; j < L; ++j)
    for (int k = 0; k < L; ++k) {
      const cplx v = root((int64_t)j * k, L);
      re[(size_t)(row0 + j) * ld + col0 + k] = v.real();
      im[(size_t)(row0 + j) * ld + col0 + k] = v.imag();
    }
}

}  // namespace

double model_flops_2d(int L, int S, int T) {
  const double Sp = round8(S);
  const double dm = 2.0 * L * L * L + Sp * L * L + Sp * Sp * L;  // DMMA.8x8x4 count * 64
  return 8.0 * dm / (2.0 * S * (double)S * T);
}

// Factored tile (kernel_fft2d_ct.cu), per pair: complex 8x8x8 products (kProdFlops each)
// for 64 rows x 2 stages + 64 columns x 4 stages + S rows x 2 stages, twiddles (6 flops per
// element, 192 + S lines of 64) and the S_T multiply (6 flops per element).
static double products_2d_ct(int S) { return 384.0 + 2.0 * S; }
double model_flops_2d_ct(int S, int T) {
  const double f = kProdFlops * products_2d_ct(S) + 384.0 * (192.0 + S) + 6.0 * 4096.0;
  return f / (2.0 * S * (double)S * T);
}

// measured: fused-kernel algorithmic flop rate / 37.18 TF/s on B200, Heat-2D / Box-2D9P /
// Star-2D13P / Box-2D49P 0.82-0.84 (profiles/r01_configs.txt)
static constexpr double kEffCt = 0.83;

// Butterfly ALU engine (kernel_fft2d_bf.cu, 64 = 4 x 16 per axis), per pair and per thread of
// the 256 that transform it: P1 and P5 eight DFT-4 (128 adds) + 24 complex twiddle multiplies
// (96 instr., 144 flops); P2 and P4 one DFT-16 (160 instr., 168 flops); P3 two DFT-16 + 16
// spectrum multiplies (384 instr., 432 flops) -- independent of S (no crop before the stores).
// BF_TW_REG (ablation, kernel_fft2d_bf.cu): P1 and P5 also form the squares and cubes of the
// two twiddle bases (16 instr., 22 flops per pass; measured 1% slower than table loads).
// BF_TW_COMB (default 0): one combined twiddle per element, 15 instead of 24 multiplies.
#ifndef BF_TW_REG
#define BF_TW_REG 0
#endif
#ifndef BF_TW_COMB
#define BF_TW_COMB 0
#endif
static constexpr int kP15Instr2d = BF_TW_COMB ? 128 + 60 : 224 + (BF_TW_REG ? 16 : 0);
static constexpr int kP15Flops2d = BF_TW_COMB ? 128 + 90 : 272 + (BF_TW_REG ? 22 : 0);
static double flops_pair_2d_bf(int) { return 256.0 * (2 * kP15Flops2d + 2 * 168 + 432); }
static double alu_ops_2d_bf(int) { return 256.0 * (2 * kP15Instr2d + 2 * 160 + 384); }
static double model_flops_2d_bf(int S, int T) { return flops_pair_2d_bf(S) / (2.0 * S * (double)S * T); }
// measured: Heat-2D 1325 GSt/s x 8.65 flop = 11.5 TF (0.31 of 37.18), Box-2D49P 422 x 26.2 =
// 11.1 TF (0.30) (BENCH_r01.json, profiles/r01_s3_sweep.txt)
static constexpr double kEff2dBf = 0.30;

// Measured DMMA issue efficiency of the fused 2D kernel per tile side (fraction of the
// 37.18 TF/s peak, B200, profiles/r01_sweep.txt / r01_variants.txt): the plan minimises
// executed flops / efficiency, i.e. predicted time per cell-step (the role of Eq. 5's
// auto-tuning of L, L174).
static double eff_2d(int L) {
  switch (L) {
    case 16: return 0.68;
    case 24: return 0.66;
    case 32: return 0.70;
    case 40: return 0.64;
    case 48: return 0.74;
    case 56: return 0.66;
    default: return 0.70;
  }
}

// Factored 3D tile (kernel_fft3d_ct.cu): line groups of 4 per pair (64 per forward axis,
// 64 for the inverse axis 0, 4S for inverse axis 1, S ceil(S/4) for inverse axis 2), each
// one complex 8x8x8 product (kProdFlops) + twiddle (32 x 6) + DFT-2 (64 x 2); + S_T.
static double groups_3d_ct(int S) { return 256.0 + 4.0 * S + S * (double)((S + 3) / 4); }
static double model_flops_3d_ct(int S, int T) {
  return ((prod_flops(kCmul3_3d) + 320.0) * groups_3d_ct(S) + 6.0 * 4096.0) / (2.0 * S * (double)S * S * T);
}
// Radix-4 ALU engine (kernel_fft3d_bf.cu), per pair: 16-point line FFTs -- 256 per forward
// axis, 256 inverse axis 0, 16 S inverse axis 1, S^2 inverse axis 2 -- of 168 flops
// (160 FP64 instructions, fft_radix.cuh) each, + S_T (6 flops, 4 instructions per element).
static double lines_3d_bf(int S) { return 1024.0 + 16.0 * S + (double)S * S; }
static double model_flops_3d_bf(int S, int T) {
  return (168.0 * lines_3d_bf(S) + 6.0 * 4096.0) / (2.0 * S * (double)S * S * T);
}
static double alu_ops_3d_bf(int S) { return 160.0 * lines_3d_bf(S) + 4.0 * 4096.0; }
// Flop rate of the ALU engine relative to the 37.18 TF/s DMMA peak (both share the FP64 pipe,
// profiles/r01_fp64_shared.txt), measured: Heat-3D 214 GSt/s x 36.6 flop = 7.8 TF (0.21)
// (profiles/r01_s3_sweep.txt, gpurun_out r02 Heat-3D runs).
static constexpr double kEff3dBf = 0.21;
// FFTSTENCIL_ENGINE=dmma|alu pins the line engine of the factored 2D and 3D tiles (ablation);
// default alu.
static int env_engine() {
  const char* v = std::getenv("FFTSTENCIL_ENGINE");
  if (v && !std::strcmp(v, "dmma")) return 0;
  return 1;
}
static constexpr double kEff3d = 0.70;     // dense 3D: executed DMMA efficiency (profiles/r01_sweep.txt)
static constexpr double kEff3dCt = 0.62;   // factored 3D: measured 0.617 (profiles/r01_configs.txt)

static double model_flops_3d(int L, int S, int T) {
  const double Sp = round8(S), l = L;
  const double f = 24.0 * l * l * l * l + 8.0 * Sp * l * l * l + 8.0 * Sp * Sp * l * l + 8.0 * Sp * Sp * Sp * l;
  return f / (2.0 * S * (double)S * S * T);
}

static double model_flops_1d(int S, int T) {  // one 8x8 complex tile, 4 GEMMs of 8 DMMAs
  return 32.0 * 512.0 / (2.0 * S * (double)T);
}
static constexpr double kEff1d = 0.73;     // PFA 8x7: executed DMMA efficiency (profiles/r01_fft1d_ncu.txt)

// Factored 1D tile (kernel_fft1d_ct.cu), per pair: 4 x 64 lines of DFT-64 (2 complex 8x8x8
// products each) + 7 complex multiplies per element (2 w4096 twiddles, 4 w64 twiddles, S_T;
// 6 flops each).
static double flops_pair_1d_ct() { return kProdFlops * 512.0 + 6.0 * 7.0 * 4096.0; }
static double model_flops_1d_ct(int S, int T) { return flops_pair_1d_ct() / (2.0 * S * (double)T); }
static constexpr double kEff1dCt = 0.59;   // measured 0.586-0.605 on 2^29 cells (profiles/r01_configs.txt)
// Butterfly ALU engine (kernel_fft1d_bf.cu), per pair and per thread of 256: P1/P3/P5/P7 four
// DFT-4 + 12 twiddle multiplies (112 instr., 136 flops), P2/P6 a DFT-16 + 31 complex multiplies
// (w4096 powers: 284 instr., 354 flops), P4 two DFT-16 + 16 spectrum multiplies (384, 432).
static double flops_pair_1d_bf() { return 256.0 * (4 * 136 + 2 * 354 + 432); }
static double alu_ops_1d_bf() { return 256.0 * (4 * 112 + 2 * 284 + 384); }
static double model_flops_1d_bf(int S, int T) { return flops_pair_1d_bf() / (2.0 * S * (double)T); }
// measured: Heat-1D 2^29, T = 1024: 103.9 k GSt/s x 0.103 flop = 10.7 TF (0.29 of 37.18)
// (profiles/r01_s3_sweep.txt)
static constexpr double kEff1dBf = 0.29;

static int env_engine();

int build_host_plan(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                    HostPlan& p, std::string& err, int nranks, int rank, int algo, int periodic) {
  p = HostPlan();
  p.periodic = periodic != 0;
  if (p.periodic && nranks > 1) { err = "periodic boundaries are single-GPU in this build"; return FFTSTENCIL_EUNSUPPORTED; }
  if (nranks < 1 || rank < 0 || rank >= nranks) { err = "need 0 <= rank < nranks"; return FFTSTENCIL_EINVAL; }
  if (ndim < 1 || ndim > 3) { err = "ndim must be 1, 2 or 3"; return FFTSTENCIL_EINVAL; }
  if (!extents || !weights) { err = "extents and weights must be non-NULL"; return FFTSTENCIL_EINVAL; }
  if (radius < 1 || radius > kMaxRadius) { err = "radius must be in 1..8"; return FFTSTENCIL_EINVAL; }
  if (T < 0) { err = "T must be >= 0 (0 = automatic)"; return FFTSTENCIL_EINVAL; }
  for (int a = 0; a < ndim; ++a) {
    if (extents[a] <= 2 * radius) { err = "every extent must exceed 2*radius"; return FFTSTENCIL_EINVAL; }
    if (extents[a] > (int64_t(1) << 31) - 1) { err = "extent too large (>= 2^31)"; return FFTSTENCIL_EINVAL; }
  }
  const int wd = 2 * radius + 1;
  int64_t nw = 1;
  for (int a = 0; a < ndim; ++a) nw *= wd;
  p.w.assign(weights, weights + nw);
  for (double v : p.w)
    if (!std::isfinite(v)) { err = "weights must be finite"; return FFTSTENCIL_EINVAL; }
  p.ndim = ndim;
  p.radius = radius;
  for (int a = 0; a < ndim; ++a) { p.ext[a] = extents[a]; p.n[3 - ndim + a] = extents[a]; }
  int64_t nmin = extents[0];
  for (int a = 1; a < ndim; ++a) nmin = std::min(nmin, extents[a]);
  // h = rT must leave a non-empty exact region on every axis: 2h < n_a.
  const int hmax_grid = (int)std::min<int64_t>((nmin - 1) / 2, 1 << 20);

  // ---- tile and depth selection (Eq. 5's role, re-derived: DESIGN.md §Plan) ----
  if (ndim == 1) {
    // candidates: the prime-factor 8 x 7 tile (the paper's, §3.2.1) and the factored
    // 4096 = 64 x 64 tile (long tiles for deep temporal fusion, kernel_fft1d_ct.cu)
    const int engine1d = env_engine();
    double best = 1e300;
    int bT = 0, bA = 0;
    for (int al = 0; al < 2; ++al) {
      if (algo >= 0 && al != algo) continue;
      const int L = al ? kCt1dL : kPfaN1 * kPfaN2;
      // the cost model is per cell-step; it ignores parallelism, so the long tile is chosen
      // automatically only when it still yields >= 64 tiles (short grids such as BASELINE
      // configs[0], 4096 cells, keep the paper's 8 x 7 prime-factor tile)
      if (al && algo < 0 && extents[0] < 64 * (int64_t)(kCt1dL / 2)) continue;
      const int smin = al ? 64 : 8;
      const int hmax = std::min(hmax_grid, (L - smin) / 2);
      if (hmax < radius) continue;
      const int tmax = hmax / radius;
      const int tlo = T == 0 ? 1 : std::min(T, tmax), thi = T == 0 ? (al ? tmax : std::min(tmax, 64)) : tlo;
      for (int t = tlo; t <= thi; ++t) {
        const int S = L - 2 * radius * t;
        // ALU engine: 64-aligned valid lengths keep the tile origins on 64-cell rows (TMA staging)
        const double f = !al ? model_flops_1d(S, t) / kEff1d
                         : engine1d ? model_flops_1d_bf(S, t) / kEff1dBf * (S % 64 ? 1.05 : 1.0)
                                    : model_flops_1d_ct(S, t) / kEff1dCt;
        if (f < best * (1 - 1e-12)) { best = f; bT = t; bA = al; }
      }
    }
    if (bT == 0) { err = "grid or radius too small for the 1D tile"; return FFTSTENCIL_EINVAL; }
    p.algo = bA;
    p.N1 = bA ? 64 : kPfaN1;
    p.N2 = bA ? 64 : kPfaN2;
    const int L = bA ? kCt1dL : p.N1 * p.N2;
    p.T = bT;
    p.h = radius * p.T;
    p.L[0] = L;
    p.S[0] = L - 2 * p.h;
    if (bA && engine1d) {
      p.engine = 1;
      p.flops_per_cell_step = model_flops_1d_bf(p.S[0], p.T);
      p.mma_flops_per_pair = 0;
      p.alu_ops_per_pair = alu_ops_1d_bf();
      p.fused_smem = (size_t)6 * kCt1dL * sizeof(double) + (64 + 256) * 16 + 1024;
    } else if (bA) {
      p.flops_per_cell_step = model_flops_1d_ct(p.S[0], p.T);
      p.mma_flops_per_pair = kProdDmmaFlops * 512.0;
      p.fused_smem = (size_t)2 * kCt1dL * sizeof(double);
    } else {
      p.flops_per_cell_step = (16.0 * p.N1 * p.N2 * (p.N1 + p.N2) + 6.0 * p.N1 * p.N2) / (2.0 * p.S[0] * p.T);
      p.mma_flops_per_pair = 32.0 * 512.0;
    }
  } else if (ndim == 2) {
    // candidates: dense L x L DFT tiles and the factored 64 = 8 x 8 tile (NEXT-1)
    static const int cand[] = {16, 24, 32, 40, 48, 56, 64};
    const int engine = env_engine();
    auto cost = [&](int al, int L, int S, int t) {
      return al ? (engine ? model_flops_2d_bf(S, t) / kEff2dBf : model_flops_2d_ct(S, t) / kEffCt)
                : model_flops_2d(L, S, t) / eff_2d(L);
    };
    double best = 1e300;
    int bL = 0, bT = 0, bA = 0;
    const int tlo = T == 0 ? 1 : T, thi = T == 0 ? 16 : T;
    for (int pass = 0; pass < 2 && bL == 0; ++pass) {
      // pass 0: the requested T (or the auto range); pass 1: lower a too-deep T
      const int a0 = pass == 0 ? tlo : 1, a1 = pass == 0 ? thi : std::min(thi, 64);
      for (int t = a0; t <= a1; ++t) {
        const int h = radius * t;
        if (h > hmax_grid) break;
        for (int al = 0; al < 2; ++al) {
          if (algo >= 0 && al != (algo == 2 ? 0 : algo)) continue;   // 2 = unfused: dense geometry
          for (int L : cand) {
            if (al == 1 && L != 64) continue;
            const int S = L - 2 * h;
            if (S < 8) continue;
            const double f = cost(al, L, S, t);
            if (f < best * (1 - 1e-12)) { best = f; bL = L; bT = t; bA = al; }
          }
        }
      }
    }
    if (bL == 0) { err = "no 2D tile fits this radius/grid"; return FFTSTENCIL_EINVAL; }
    p.algo = algo == 2 ? 2 : bA;
    if (p.algo == 2 && nranks > 1) { err = "the unfused ablation is single-GPU"; return FFTSTENCIL_EUNSUPPORTED; }
    p.T = bT;
    p.h = radius * bT;
    p.L[0] = p.L[1] = bL;
    p.S[0] = p.S[1] = bL - 2 * p.h;
    const double L = bL, S = p.S[0];
    if (bA == 0) {   // dense (and the unfused ablation, same GEMMs)
      p.flops_per_cell_step = (16.0 * L * L * L + 6.0 * L * L + 8.0 * S * L * L + 8.0 * S * S * L) / (2.0 * S * S * bT);
      const double Sp = round8(p.S[0]);
      p.mma_flops_per_pair = 8.0 * (2.0 * L * L * L + Sp * L * L + Sp * Sp * L);
      p.fused_smem = (size_t)(bL >= 56 ? 48 : 32) * bL * (bL + 4);   // F + pair buffer(s)
    } else if (engine) {
      p.engine = 1;
      p.flops_per_cell_step = model_flops_2d_bf(p.S[0], bT);
      p.mma_flops_per_pair = 0;
      p.alu_ops_per_pair = alu_ops_2d_bf(p.S[0]);
      p.fused_smem = (size_t)6 * 64 * 64 * sizeof(double) + 64 * 16 + 1024;   // 2 pair buffers + S_T + w64
    } else {
      p.flops_per_cell_step = model_flops_2d_ct(p.S[0], bT);
      p.mma_flops_per_pair = kProdDmmaFlops * products_2d_ct(p.S[0]);
      p.fused_smem = (size_t)2 * 64 * 64 * sizeof(double);
    }
  } else {
    // candidates: the dense 16^3 tile and the factored one (16 = 8 x 2 per axis)
    const int L = k3DTile;
    const int hmax = std::min(hmax_grid, (L - 2) / 2);
    const int tmax = hmax / radius;
    if (tmax < 1) { err = "radius too large for the 16^3 3D tile"; return FFTSTENCIL_EINVAL; }
    const int engine = env_engine();
    double best = 1e300;
    int bestT = 1, bA = 0;
    for (int t = 1; t <= tmax; ++t) {
      if (T != 0 && t != std::min(T, tmax)) continue;
      for (int al = 0; al < 2; ++al) {
        if (algo >= 0 && al != algo) continue;
        const int S = L - 2 * radius * t;
        const double f = !al ? model_flops_3d(L, S, t) / kEff3d
                         : engine ? model_flops_3d_bf(S, t) / kEff3dBf : model_flops_3d_ct(S, t) / kEff3dCt;
        if (f < best) { best = f; bestT = t; bA = al; }
      }
    }
    p.algo = bA;
    p.T = bestT;
    p.h = radius * bestT;
    for (int a = 0; a < 3; ++a) { p.L[a] = L; p.S[a] = L - 2 * p.h; }
    const double l = L, S = p.S[0];
    if (bA == 0) {
      p.flops_per_cell_step =
          (24.0 * l * l * l * l + 6.0 * l * l * l + 8.0 * l * (S * l * l + S * S * l + S * S * S)) /
          (2.0 * S * S * S * bestT);
      const double Sp = round8(p.S[0]);
      // executed DMMAs per pair (kernel_fft3d.cu): phase 1 16 slices x 128, phase 2 32 row
      // blocks x (32 + 16 Sp/8), phase 3 S slices x (64 Sp/8 + 16 (Sp/8)^2)
      const double mt = Sp / 8.0;
      p.mma_flops_per_pair = 512.0 * (16 * 128 + 32 * (32 + 16 * mt) + S * (64 * mt + 16 * mt * mt));
      p.fused_smem = (size_t)(2 * 16 * 20 + 2 * 16 * (16 * 20 + 4)) * sizeof(double);
    } else if (engine) {
      p.engine = 1;
      p.mma_flops_per_pair = 0;
      p.flops_per_cell_step = model_flops_3d_bf(p.S[0], bestT);
      p.alu_ops_per_pair = alu_ops_3d_bf(p.S[0]);
      p.fused_smem = (size_t)6 * 16 * 16 * 16 * sizeof(double) + 1024;   // 2 pair buffers + S_T
    } else {
      p.flops_per_cell_step = model_flops_3d_ct(p.S[0], bestT);
      p.mma_flops_per_pair = prod_dmma_flops(kCmul3_3d) * groups_3d_ct(p.S[0]);
      p.fused_smem = (size_t)2 * 16 * 16 * 16 * sizeof(double);
    }
  }

  // ---- overlap-save schedule (Eq. 3 / Eq. 4 / Eq. 7; reading Q4: centred window) ----
  p.tiles = 1;
  for (int a = 0; a < ndim; ++a) {
    // fixed ring: the exact region [h, n-h) is tiled; periodic: every cell is (NEXT-2)
    p.nt[a] = ceil_div(p.periodic ? p.ext[a] : p.ext[a] - 2 * p.h, p.S[a]);
    p.tiles *= p.nt[a];
  }
  // Double-layer Filling pairs (Eq. 9): along the innermost tile axis within one outer
  // tile row/line (kernels.cuh), so a decomposition by whole tile rows keeps every pair.
  const int inner = ndim - 1;
  p.npr = (p.nt[inner] + 1) / 2;
  p.pairs = p.tiles / p.nt[inner] * p.npr;

  // ---- outer-axis decomposition: whole units per rank (DESIGN.md a10) ----
  {
    const int64_t n0 = p.ext[0];
    int64_t US;                        // outer rows per unit
    if (ndim == 1) {
      p.units = p.pairs;
      p.pairs_per_unit = 1;
      US = 2 * (int64_t)p.S[0];
    } else {
      p.units = p.nt[0];
      p.pairs_per_unit = p.pairs / p.nt[0];
      US = p.S[0];
    }
    p.nranks = nranks;
    p.rank = rank;
    if (p.units < nranks) { err = "fewer outer tile rows than ranks"; return FFTSTENCIL_EINVAL; }
    p.unit_lo = p.units * rank / nranks;
    p.unit_hi = p.units * (rank + 1) / nranks;
    p.row_lo = rank == 0 ? 0 : p.unit_lo * US + p.h;
    p.row_hi = rank == nranks - 1 ? n0 : p.unit_hi * US + p.h;
    if (nranks > 1) {
      for (int k = 0; k < nranks; ++k) {   // every slab must cover one halo (ghosts = neighbours only)
        const int64_t ul = p.units * k / nranks, uh = p.units * (k + 1) / nranks;
        const int64_t s = k == 0 ? 0 : ul * US + p.h, e = k == nranks - 1 ? n0 : uh * US + p.h;
        if (e - s < p.h) { err = "a rank's slab is thinner than the halo r*T"; return FFTSTENCIL_EINVAL; }
      }
    }
    p.g0 = std::max<int64_t>(0, p.row_lo - p.h);
    p.g1 = std::min<int64_t>(n0, p.row_hi + p.h);
    p.pair_lo = p.unit_lo * p.pairs_per_unit;
    p.pair_hi = p.unit_hi * p.pairs_per_unit;
    // interior units: every input row of the unit's tiles lies in the owned rows
    const int64_t span = ndim == 1 ? (int64_t)p.S[0] + p.L[0] : p.L[0];   // input rows of a unit
    int64_t ilo = p.unit_hi, ihi = p.unit_hi;
    for (int64_t u = p.unit_lo; u < p.unit_hi; ++u) {
      const int64_t in_lo = u * US, in_hi = std::min<int64_t>(n0, u * US + span);
      if (in_lo >= p.row_lo && in_hi <= p.row_hi) {
        if (ilo == p.unit_hi) ilo = u;
        ihi = u + 1;
      }
    }
    if (ilo == p.unit_hi) ilo = ihi = p.unit_lo;
    p.ipair_lo = ilo * p.pairs_per_unit;
    p.ipair_hi = ihi * p.pairs_per_unit;
  }

  // ---- DFT matrices (forward; the kernel conjugates for the inverse, L258/L278) ----
  if (ndim == 1 && p.algo == 1 && p.engine == 1) {
    // butterfly ALU engine: w64^m (m < 64) and w4096^m (m < 256, interleaved re, im)
    p.Fre.assign(128, 0.0);
    p.Fim.assign(128, 0.0);
    for (int m = 0; m < 64; ++m) {
      const cplx v = root(m, 64);
      p.Fre[m] = v.real();
      p.Fim[m] = v.imag();
    }
    p.tw.assign(2 * 256, 0.0);
    for (int m = 0; m < 256; ++m) {
      const cplx v = root(m, kCt1dL);
      p.tw[2 * m] = v.real();
      p.tw[2 * m + 1] = v.imag();
    }
  } else if (ndim == 1 && p.algo == 1) {
    // [F8 | twiddles w64^(ka lb)] as in 2D, and the four-step twiddles w4096^(a c)
    p.Fre.assign(128, 0.0);
    p.Fim.assign(128, 0.0);
    fill_dft(8, 8, 0, 0, p.Fre, p.Fim);
    for (int ka = 0; ka < 8; ++ka)
      for (int lb = 0; lb < 8; ++lb) {
        const cplx v = root((int64_t)ka * lb, 64);
        p.Fre[64 + ka * 8 + lb] = v.real();
        p.Fim[64 + ka * 8 + lb] = v.imag();
      }
    p.tw.assign(2 * kCt1dL, 0.0);
    for (int a = 0; a < 64; ++a)
      for (int c = 0; c < 64; ++c) {
        const cplx v = root((int64_t)a * c, kCt1dL);
        p.tw[2 * (a * 64 + c)] = v.real();
        p.tw[2 * (a * 64 + c) + 1] = v.imag();
      }
  } else if (ndim == 1) {
    p.Fre.assign(2 * 64, 0.0);
    p.Fim.assign(2 * 64, 0.0);
    fill_dft(p.N1, 8, 0, 0, p.Fre, p.Fim);          // rows 0..7   : F_N1
    fill_dft(p.N2, 8, 8, 0, p.Fre, p.Fim);          // rows 8..14  : F_N2 (row 15, col 7 zero)
    p.crt.assign(64, -1);
    const int L = p.N1 * p.N2;
    for (int l = 0; l < L; ++l) p.crt[(l % p.N1) * 8 + (l % p.N2)] = l;   // diagonal / CRT map
  } else if (ndim == 3 && p.algo == 1) {
    // [F8 | w16^k, k = 0..15] (kernel_fft3d_ct.cu)
    p.Fre.assign(128, 0.0);
    p.Fim.assign(128, 0.0);
    fill_dft(8, 8, 0, 0, p.Fre, p.Fim);
    for (int k = 0; k < 16; ++k) {
      const cplx v = root(k, 16);
      p.Fre[64 + k] = v.real();
      p.Fim[64 + k] = v.imag();
    }
  } else if (ndim == 2 && p.algo == 1 && p.engine == 1) {
    // w64^m, m = 0..63 (kernel_fft2d_bf.cu twiddle table)
    p.Fre.assign(128, 0.0);
    p.Fim.assign(128, 0.0);
    for (int m = 0; m < 64; ++m) {
      const cplx v = root(m, 64);
      p.Fre[m] = v.real();
      p.Fim[m] = v.imag();
    }
  } else if (ndim == 2 && p.algo == 1) {
    // [F8 | twiddles w64^(ka lb)], 8 x 8 each (kernel_fft2d_ct.cu)
    p.Fre.assign(128, 0.0);
    p.Fim.assign(128, 0.0);
    fill_dft(8, 8, 0, 0, p.Fre, p.Fim);
    for (int ka = 0; ka < 8; ++ka)
      for (int lb = 0; lb < 8; ++lb) {
        const cplx v = root((int64_t)ka * lb, 64);
        p.Fre[64 + ka * 8 + lb] = v.real();
        p.Fim[64 + ka * 8 + lb] = v.imag();
      }
  } else {
    const int L = p.L[0];
    p.Fre.assign((size_t)L * L, 0.0);
    p.Fim.assign((size_t)L * L, 0.0);
    fill_dft(L, L, 0, 0, p.Fre, p.Fim);
  }

  // ---- powered spectra S_t, t = 1..T (Eq. 10) with 1/prod(L) folded in (Q7) ----
  // Powers by repeated multiplication, v_t = v_{t-1} * sigma (reading Q6), kept running
  // across t so the build is O(T vol), not O(T^2 vol).
  p.Sre.assign(p.T, {});
  p.Sim.assign(p.T, {});
  if (ndim == 1 && p.algo == 0) {
    const int L = p.N1 * p.N2;
    std::vector<cplx> sig(L), pw(L, cplx(1.0, 0.0));
    for (int k = 0; k < L; ++k) { int kk[1] = {k}; int LL[1] = {L}; sig[k] = symbol(p, kk, LL); }
    for (int t = 1; t <= p.T; ++t) {
      auto& re = p.Sre[t - 1];
      auto& im = p.Sim[t - 1];
      re.assign(64, 0.0);
      im.assign(64, 0.0);
      for (int k = 0; k < L; ++k) pw[k] *= sig[k];
      for (int k1 = 0; k1 < p.N1; ++k1)
        for (int k2 = 0; k2 < p.N2; ++k2) {
          const int k = (k1 * p.N2 + k2 * p.N1) % L;   // Ruritanian order (Eq. 8, reading Q8)
          const cplx v = pw[k] / (double)L;
          re[k1 * 8 + k2] = v.real();
          im[k1 * 8 + k2] = v.imag();
        }
    }
  } else {
    int64_t vol = 1;
    for (int a = 0; a < ndim; ++a) vol *= p.L[a];
    std::vector<cplx> sig(vol), pw(vol, cplx(1.0, 0.0));
    for (int64_t i = 0; i < vol; ++i) {
      int k[3], rem = (int)i;
      for (int a = ndim - 1; a >= 0; --a) { k[a] = rem % p.L[a]; rem /= p.L[a]; }
      sig[i] = symbol(p, k, p.L);
    }
    for (int t = 1; t <= p.T; ++t) {
      auto& re = p.Sre[t - 1];
      auto& im = p.Sim[t - 1];
      re.resize(vol);
      im.resize(vol);
      for (int64_t i = 0; i < vol; ++i) {
        pw[i] *= sig[i];
        const cplx v = pw[i] / (double)vol;
        // 2D: natural [k0][k1].  3D: [k1][k2][k0] -- the 3D kernel multiplies in C fragments
        // whose two adjacent columns are consecutive k0 (kernel_fft3d.cu phase 2).
        int64_t dst = i;
        if (ndim == 1 && p.engine == 1) {
          // ALU engine: k = c + 64 d at [column position q(d)][row position p(c)], position
          // 16 a + b <-> frequency a + 4 b (kernel_fft1d_bf.cu)
          const int64_t c = i % 64, d = i / 64;
          dst = (16 * (d % 4) + d / 4) * 64 + 16 * (c % 4) + c / 4;
        } else if (ndim == 1) {
          // factored 1D: k = c + 64 d at [c][8 (d % 8) + d / 8] (row c, CT digit order of d)
          const int64_t c = i % 64, d = i / 64;
          dst = c * 64 + 8 * (d % 8) + d / 8;
        } else if (ndim == 3 && p.algo == 1 && p.engine == 1) {
          // radix-4 ALU engine: natural [k0][k1][k2]
        } else if (ndim == 3 && p.algo == 1) {
          // factored 3D: [k1][k2][k0 % 8][k0 / 8] (the thread-local DFT-2 output pair)
          const int64_t L = p.L[0], k0 = i / (L * L), k12 = i % (L * L);
          dst = (k12 * 8 + k0 % 8) * 2 + k0 / 8;
        } else if (ndim == 3) {
          const int64_t L = p.L[0], k0 = i / (L * L), k12 = i % (L * L);
          dst = k12 * L + k0;
        } else if (p.algo == 1 && p.engine == 1) {
          // butterfly ALU engine: position order on both axes, position 16 a + b <-> frequency a + 4 b
          const int64_t k0 = i / 64, k1 = i % 64;
          dst = (16 * (k0 % 4) + k0 / 4) * 64 + 16 * (k1 % 4) + k1 / 4;
        } else if (p.algo == 1) {
          // factored 2D: [k1][8 g + c] holds k0 = g + 8 c (digit order of the CT output)
          const int64_t k0 = i / 64, k1 = i % 64;
          dst = k1 * 64 + 8 * (k0 % 8) + k0 / 8;
        }
        re[dst] = v.real();
        im[dst] = v.imag();
      }
    }
  }

  // ---- fixed ring: exact partition into boxes (axis a faces, lower axes interior) ----
  const int r = radius, h = p.h;
  const int off = 3 - ndim;
  for (int a = 0; a < ndim && !p.periodic; ++a) {
    for (int side = 0; side < 2; ++side) {
      Box b;
      for (int e = 0; e < 3; ++e) { b.lo[e] = 0; b.hi[e] = p.n[e]; }
      const int e = off + a;
      b.lo[e] = side == 0 ? 0 : p.n[e] - r;
      b.hi[e] = side == 0 ? r : p.n[e];
      for (int c = 0; c < a; ++c) { b.lo[off + c] = r; b.hi[off + c] = p.n[off + c] - r; }
      b.lo[off] = std::max<int64_t>(b.lo[off], p.row_lo);   // this rank's rows only
      b.hi[off] = std::min<int64_t>(b.hi[off], p.row_hi);
      if (b.hi[off] > b.lo[off]) p.ring_boxes.push_back(b);
    }
  }
  // ---- boundary band: interior cells outside the exact region [h, n-h) (reading Q5) ----
  // Face of axis a: c_a in [r, h) or [n_a-h, n_a-r); axes before a exact ([h, n-h)),
  // axes after a interior ([r, n-r)).  The boxes partition the band exactly.
  if (h > r && !p.periodic) {
    for (int a = 0; a < ndim; ++a)
      for (int side = 0; side < 2; ++side) {
        Box b;
        for (int e = 0; e < 3; ++e) { b.lo[e] = 0; b.hi[e] = p.n[e]; }
        const int e = off + a;
        b.lo[e] = side == 0 ? r : p.n[e] - h;
        b.hi[e] = side == 0 ? h : p.n[e] - r;
        for (int c = 0; c < ndim; ++c) {
          if (c == a) continue;
          const int ec = off + c;
          b.lo[ec] = c < a ? h : r;
          b.hi[ec] = c < a ? p.n[ec] - h : p.n[ec] - r;
        }
        b.face = e;
        b.lo[off] = std::max<int64_t>(b.lo[off], p.row_lo);   // this rank's rows only
        b.hi[off] = std::min<int64_t>(b.hi[off], p.row_hi);
        bool empty = false;
        for (int q = 0; q < 3; ++q) empty |= b.hi[q] <= b.lo[q];
        if (!empty) p.band_boxes.push_back(b);
      }
  }
  // Split each band box into CTA blocks whose input region (block + r*T on every
  // active side) fits the band kernel's shared-memory budget (2 buffers of FP64).
  // 24 KB of FP64 pairs: small enough to co-reside with three 64 KB fused CTAs per SM (the
  // band runs concurrently on its own stream, capi.cu).  The 2D ALU engine fills the register
  // file, so its band never co-resides and runs between fused launches: blocks of 2240 cells
  // per buffer (still 6 CTAs per SM, bound by registers) recompute less halo per band cell and
  // fit the 10240^2 band into about one wave (Heat-2D +1.5%; 3D measured best at 1536,
  // profiles/r01_s3_ab_band_budget.txt).  FFTSTENCIL_BAND_BUDGET overrides (cells per buffer).
  // cells per band block buffer: 2240 for 2D ALU plans (profiles/r01_s3_ab_band_budget.txt), 4608
  // for 3D ALU plans (fewer, larger blocks once the block setup is cheap: band alone 0.40 ->
  // 0.26 ms per Heat-3D pass, profiles/r02_band3d.txt), 1536 otherwise
  int budget_cells = p.engine == 1 && p.ndim == 2 ? 2240 : p.engine == 1 && p.ndim == 3 ? 4608 : 1536;
  if (const char* v = std::getenv("FFTSTENCIL_BAND_BUDGET")) budget_cells = std::max(256, std::atoi(v));
  const int grow = 2 * r * p.T;
  for (const Box& b : p.band_boxes) {
    int64_t len[3], blk[3];
    for (int q = 0; q < 3; ++q) len[q] = b.hi[q] - b.lo[q];
    const int face = b.face;   // the face axis keeps its whole band width
    int ntan = 0;
    for (int q = 0; q < 3; ++q) {
      blk[q] = len[q];
      if (q >= off && q != face) ++ntan;
    }
    const int64_t fw = face >= 0 ? len[face] + grow : 1;
    int64_t tb = 1024;
    if (ntan == 1) tb = std::max<int64_t>(8, std::min<int64_t>(256, budget_cells / fw - grow));
    if (ntan == 2) {
      int64_t s = (int64_t)std::sqrt((double)budget_cells / (double)fw) - grow;
      tb = std::max<int64_t>(8, std::min<int64_t>(64, s));
    }
    for (int q = off; q < 3; ++q)
      if (q != face) blk[q] = std::min<int64_t>(len[q], tb);
    for (int64_t i0 = b.lo[0]; i0 < b.hi[0]; i0 += blk[0])
      for (int64_t i1 = b.lo[1]; i1 < b.hi[1]; i1 += blk[1])
        for (int64_t i2 = b.lo[2]; i2 < b.hi[2]; i2 += blk[2]) {
          const int64_t lo[3] = {i0, i1, i2};
          int64_t hi[3] = {std::min(i0 + blk[0], b.hi[0]), std::min(i1 + blk[1], b.hi[1]),
                           std::min(i2 + blk[2], b.hi[2])};
          int64_t cells = 1;
          for (int q = 0; q < 3; ++q) {
            const int64_t g = (q >= off) ? r * (int64_t)p.T : 0;
            const int64_t rl = std::max<int64_t>(0, lo[q] - g), rh = std::min<int64_t>(p.n[q], hi[q] + g);
            cells *= rh - rl;
          }
          p.band_region_cells = std::max<int>(p.band_region_cells, (int)cells);
          for (int q = 0; q < 3; ++q) p.band_blocks.push_back((int32_t)lo[q]);
          for (int q = 0; q < 3; ++q) p.band_blocks.push_back((int32_t)hi[q]);
          p.band_blocks.push_back(face);
          p.band_blocks.push_back(0);
        }
  }
  return FFTSTENCIL_OK;
}


// ---- pipelined run_host schedule ----
// Unit u (outer tile row) of pass k reads pass k-1's rows [uS, uS+L) = its output rows +- h,
// i.e. units u-1..u+1 when h <= S.  Band and ring cells belong to the unit whose row range
// R(u) = [row(u), row(u+1)) holds them (row(0) = 0, row(U) = n0), and their dependency cone
// (+- h rows) stays within units u-1..u+1 too.  Frontiers f[k] (units [0, f[k]) of pass k
// issued) with f[k] <= f[k-1] - 1 (or f[k-1] = U) satisfy the read dependency and the
// ping-pong anti-dependency at once, so the ops run in issue order on one stream.
int build_e2e_schedule(const HostPlan& p, int64_t total_steps, int K, int Q, std::vector<int64_t>& ops, int Qt,
                       int ramp) {
  ops.clear();
  if (Qt <= 0) Qt = Q;
  if (K < 2 || Q < 1 || p.ndim < 2 || p.periodic || p.algo == 2 || p.nranks != 1 || total_steps <= 0)
    return FFTSTENCIL_EINVAL;
  const int64_t U = p.nt[0], n0 = p.ext[0], S = p.S[0], h = p.h;
  if (h > S || U < 2 * (int64_t)K || p.pair_lo != 0 || p.pair_hi != p.pairs) return FFTSTENCIL_EINVAL;
  const int64_t P = total_steps / p.T + (total_steps % p.T ? 1 : 0);
  auto row_of = [&](int64_t u) -> int64_t { return u <= 0 ? 0 : u >= U ? n0 : u * S + h; };
  auto push = [&](int64_t op, int64_t x, int64_t y, int64_t z) {
    ops.push_back(op); ops.push_back(x); ops.push_back(y); ops.push_back(z);
  };
  std::vector<int64_t> f((size_t)P + 1, 0);
  auto propagate = [&](auto cap) {
    for (int64_t k = 1; k <= P; ++k) {
      int64_t want = f[k - 1] >= U ? U : std::max<int64_t>(0, f[k - 1] - 1);
      want = std::min<int64_t>(want, cap(k));
      if (want > f[k]) {
        push(2, k, f[k], want);
        f[k] = want;
      }
    }
  };
  // Chunk boundaries (outer tile rows): K regular chunks, with the FIRST input chunk and the LAST
  // output chunk split 1/4 + 3/4 -- nothing overlaps the first H2D chunk or the last D2H chunk,
  // so those two are the small ones (Heat-2D: 2 x 2.4 ms exposed copies at K = 6 -> 2 x 0.6 ms).
  // ramp = 2 also splits the LAST input chunk 3/4 + 1/4 and the FIRST output chunk 1/4 + 3/4: the
  // head's drain after the last H2D (every head pass catching up on that chunk) and the tail's
  // fill before the first D2H (the tail passes advancing to it) scale with those chunks' size.
  const int64_t q4 = std::max<int64_t>(1, U / (4 * (int64_t)K));
  std::vector<int64_t> ib{0, q4}, ob{0};
  if (ramp >= 2) ob.push_back(q4);
  for (int c = 1; c <= K; ++c) {
    if (ramp >= 2 && c == K && U - q4 > ib.back()) ib.push_back(U - q4);
    ib.push_back(U * c / K);
  }
  for (int j = 1; j < K; ++j)
    if (U * j / K > ob.back()) ob.push_back(U * j / K);
  if (U - q4 > ob.back()) ob.push_back(U - q4);
  ob.push_back(U);
  // head: input chunk c, its ring rows, then the first Q passes advance behind it
  for (size_t c = 1; c < ib.size(); ++c) {
    const int64_t y0 = row_of(ib[c - 1]), y1 = row_of(ib[c]);
    push(0, y0, y1, 0);
    push(1, y0, y1, 0);
    f[0] = ib[c];
    propagate([&](int64_t k) { return k <= Q ? U : (int64_t)0; });
  }
  // tail: the last Q passes advance until pass P holds chunk j, which is then copied out
  for (size_t j = 1; j < ob.size(); ++j) {
    const int64_t bj = ob[j];
    propagate([&](int64_t k) { return k <= P - Qt ? U : std::min<int64_t>(U, bj + (P - k)); });
    if (f[(size_t)P] < bj) { ops.clear(); return FFTSTENCIL_EINVAL; }
    push(3, row_of(ob[j - 1]), row_of(bj), 0);
  }
  return FFTSTENCIL_OK;
}

int build_peer_schedule(const HostPlan& p, int64_t total_steps, bool fused, int64_t epoch0, std::vector<int64_t>& ops) {
  ops.clear();
  if (p.nranks < 2 || total_steps < 0) return FFTSTENCIL_EINVAL;
  auto push = [&](int64_t op, int64_t a, int64_t b, int64_t c) {
    ops.push_back(op); ops.push_back(a); ops.push_back(b); ops.push_back(c);
  };
  if (total_steps == 0) return FFTSTENCIL_OK;   // a copy, no exchange and no signal (all ranks alike)
  int64_t e = epoch0;
  push(0, e, 0, 0);                 // neighbours done with the previous run: their pushes may land
  push(1, 0, 0, 0);
  push(2, 0, 0, 0);
  if (fused) push(2, 0, 1, 0);      // fused stores cover computed cells only: ring cells into both
  push(3, ++e, 0, 0);
  const int64_t P = total_steps / p.T + (total_steps % p.T ? 1 : 0);
  int cur = 0;
  for (int64_t k = 1; k <= P; ++k) {
    push(4, k, cur, 0);
    push(0, e, 0, 0);
    push(5, k, cur, fused ? 1 : 0);
    cur ^= 1;
    if (k < P) {
      if (!fused) push(2, cur, cur, 0);
      push(3, ++e, 0, 0);
    }
  }
  push(6, cur, 0, 0);
  push(3, ++e, 0, 0);
  return FFTSTENCIL_OK;
}

}  // namespace fstencil
