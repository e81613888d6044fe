// C ABI (include/fftstencil.h): plan lifetime, device upload and the run driver.
//
// The run driver is the temporal loop of PAPER.md §4 (Eq. 10): floor(steps/T) fused
// passes with S_T, then one pass with S_T' (T' = steps mod T; reading Q15).  Each pass is
// fused FFT-tile launch(es) over the exact region plus one boundary-band launch, reading
// `src` and writing disjoint cells of `dst`.
//   single GPU: buffers ping-pong between the caller's `out` and the plan's scratch grid so
//               the last pass lands in `out`; the fixed ring is copied once per run.
//   multi-GPU:  each rank keeps two slab buffers with r*T halo rows above and below
//               (DESIGN.md a10); before every pass the halo rows of `src` are exchanged
//               with the neighbouring ranks (NCCL send/recv on a comm stream, or device
//               copies for loopback groups) while the pairs that need no halo run.
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "fftstencil.h"
#include "kernels.cuh"
#include "plan.h"
#include "tma.cuh"

using namespace fstencil;

namespace {

thread_local std::string g_last_error;

// FFTSTENCIL_ALGO=dense|factored|unfused pins the tile algorithm (ablations); default: cost model.
int env_algo() {
  const char* v = std::getenv("FFTSTENCIL_ALGO");
  if (!v) return -1;
  if (!std::strcmp(v, "dense")) return 0;
  if (!std::strcmp(v, "factored")) return 1;
  if (!std::strcmp(v, "unfused")) return 2;   // NEXT-3 ablation (2D): three kernels per pass
  return -1;
}

void set_error(const std::string& s) { g_last_error = s; }

int env_int(const char* name, int dflt) {
  const char* v = std::getenv(name);
  return v && *v ? std::atoi(v) : dflt;
}
void clear_error() { g_last_error.clear(); }

// Pipelined run_host schedule knobs (plan.h build_e2e_schedule), read by run_host and by the
// exported fftstencil_e2e_schedule alike so the CPU replay tests see the schedule that runs:
// FFTSTENCIL_E2E_DEPTH_TAIL (tail skew depth, default = the head's), FFTSTENCIL_E2E_RAMP (1).
// Measured (profiles/r02_e2e_ramp2.txt): ramp 2 and a deeper tail are within noise or slower
// (Heat-3D 507 vs 509-511 ms, Heat-2D 88.3-89.4 vs 88.9-89.7 ms per e2e step), so the defaults stay.
int pipe_tail_depth() { return env_int("FFTSTENCIL_E2E_DEPTH_TAIL", 0); }
int pipe_ramp() { return env_int("FFTSTENCIL_E2E_RAMP", 1); }

}  // namespace

struct fftstencil_plan {
  HostPlan hp;
  int device = 0;
  int sm_count = 0;
  double* dF = nullptr;       // Fre | Fim (2D: columns permuted)
  double* dS = nullptr;       // for t = 1..T: Sre | Sim, each spec_vol
  int* dCrt = nullptr;
  double* dW = nullptr;
  int* dBlocks = nullptr;
  double* dScratch = nullptr; // single GPU: ping-pong partner of `out`
  double* dSpec = nullptr;    // unfused ablation: per-pair spectra in HBM
  double* dHostIn = nullptr;  // run_host staging grids (lazy)
  double* dHostOut = nullptr;
  size_t spec_vol = 0;
  size_t grid_cells = 0;      // cells of the caller's in/out (the slab for a dist plan)
  size_t row_cells = 0;       // cells per outer-axis row
  size_t device_bytes = 0;
  int fused_grid = 0;
  int variant = 0;            // fused-kernel variant (2D dense)
  int ct_cfg = 81;            // factored 2D kernel: 10 * warps per CTA + lines per warp step (TMA: 3 CTAs/SM)
  bool use_tma = true;        // TMA tile loads where the grid allows (FFTSTENCIL_TMA=0 disables)
  int band_reference = 0;     // FFTSTENCIL_BAND=reference selects the first band kernel
  size_t band_smem = 0;
  int64_t last_launches = 0;
  bool last_pipelined = false;   // the last run_host took the pipelined schedule
  int last_chunks = 0, last_depth = 0;   // and its K / Q
  bool last_peer_fused = false;          // the last peer-transport run pushed with the kernels' stores
  // ---- decomposition (dist) ----
  bool dist = false;          // slab plan with halo buffers
  bool loopback = false;      // no communicator: run by fftstencil_run_group
  ncclComm_t comm = nullptr;
  cudaStream_t comm_stream = nullptr;
  cudaEvent_t ev_ready = nullptr, ev_xchg = nullptr;
  // ---- the band kernel runs on a side stream, concurrent with the fused kernel (it reads
  // the same source and writes disjoint cells); FFTSTENCIL_BAND_STREAM=0 serialises it ----
  bool band_concurrent = true;
  bool band_e2e_concurrent = true;   // the pipelined run_host's items run the band on the side stream
  bool small1d = false;       // whole run in one on-chip launch (small 1D PFA plans, kernel_small1d.cu)
  cudaStream_t band_stream = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_band = nullptr;
  bool band_pending = false;

  int64_t band_clip_lo = 0, band_clip_hi = INT64_MAX;   // outer rows the band pass produces
  // ---- pipelined run_host: chunked H2D / D2H on their own stream (FFTSTENCIL_E2E_PIPE) ----
  cudaStream_t copy_stream = nullptr;
  cudaStream_t pipe_stream = nullptr;   // greatest priority: fused CTAs dispatch before the band's
  std::vector<cudaEvent_t> ev_copy;
  std::vector<int64_t> blk_lo;   // outer-axis start of each band block (blocks sorted by it)
  int64_t blk_hmax = 0;          // tallest band block along the outer axis
  int grid_cap = 0;              // > 0: fused launches use at most this many CTAs
  bool st256 = true;             // 3D ALU kernel: 32-byte output stores (FFTSTENCIL_ST256=0: 16-byte only)
  int trav_blk = 0;              // 3D ALU kernel traversal blocks (FFTSTENCIL_3D_TRAV=6: 6 x 6 tile lines; measured slower)
  int max_ctas = 0;              // FFTSTENCIL_MAX_CTAS (tests): cap on every fused launch's grid, so each
                                 // persistent CTA walks many pairs through its refill / mbarrier loop
  double* dE[2] = {nullptr, nullptr};   // slab + halo buffers, rows [g0, g1)
  // ---- peer-memory transport (no NCCL; fftstencil_plan_create_dist_peer) ----
  bool peer = false;            // halo rows pushed into the neighbours' buffers through CUDA IPC
  bool peer_connected = false;
  uint32_t* dFlags = nullptr;   // [0]: epoch signalled by the lower neighbour, [1]: by the upper one
  double* pE[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};   // [lower, upper][buffer] (IPC-mapped)
  uint32_t* pFlags[2] = {nullptr, nullptr};                       // the neighbours' dFlags
  int64_t pG0[2] = {0, 0};      // the neighbours' window starts g0
  uint32_t epoch = 0;           // signals sent so far (both neighbours send the same count)
  bool peer_fused = true;       // boundary rows stored into the neighbours by the pass's own kernels
                                // (FFTSTENCIL_PEER_FUSED=0: copy-engine push after the pass)
  PeerStore peer_store = {nullptr, nullptr, 0, 0, 0, 0};   // set around a pass's edge launches + band
  int ecur = 0;               // index of the buffer holding the current state
  // ---- profiling: event pairs (start, end, kind 0 = fused, 1 = band) recorded by run() ----
  bool profiling = false;
  std::vector<cudaEvent_t> ev_pool;
  std::vector<int> ev_kind;
  size_t ev_used = 0;
};

namespace {

using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// Stream memory operations (driver API through the runtime's entry-point query, like the
// tensor-map encoder): the peer transport's cross-process signal and wait.
using StreamValue32Fn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
StreamValue32Fn stream_fn(const char* name) {
  void* f = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &f, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
    return nullptr;
  return (StreamValue32Fn)f;
}
StreamValue32Fn write_value_fn() {
  static StreamValue32Fn fn = stream_fn("cuStreamWriteValue32");
  return fn;
}
StreamValue32Fn wait_value_fn() {
  static StreamValue32Fn fn = stream_fn("cuStreamWaitValue32");
  return fn;
}

EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return (EncodeTiledFn) nullptr;
    return (EncodeTiledFn)f;
  }();
  return fn;
}

int cuda_fail(cudaError_t e, const char* what) {
  char buf[256];
  std::snprintf(buf, sizeof buf, "%s: %s", what, cudaGetErrorString(e));
  set_error(buf);
  return FFTSTENCIL_ECUDA;
}

int nccl_fail(ncclResult_t r, const char* what) {
  char buf[256];
  std::snprintf(buf, sizeof buf, "%s: %s", what, ncclGetErrorString(r));
  set_error(buf);
  return FFTSTENCIL_ENCCL;
}

template <typename T>
cudaError_t upload(T** dptr, const T* src, size_t n, size_t& acc) {
  if (n == 0) { *dptr = nullptr; return cudaSuccess; }
  cudaError_t e = cudaMalloc((void**)dptr, n * sizeof(T));
  if (e != cudaSuccess) return e;
  acc += n * sizeof(T);
  return cudaMemcpy(*dptr, src, n * sizeof(T), cudaMemcpyHostToDevice);
}

void free_plan(fftstencil_plan* p) {
  if (!p) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(p->device);
  if (p->comm) ncclCommDestroy(p->comm);
  for (int side = 0; side < 2; ++side) {
    for (int b = 0; b < 2; ++b)
      if (p->pE[side][b]) cudaIpcCloseMemHandle(p->pE[side][b]);
    if (p->pFlags[side]) cudaIpcCloseMemHandle(p->pFlags[side]);
  }
  cudaFree(p->dFlags);
  if (p->comm_stream) cudaStreamDestroy(p->comm_stream);
  if (p->ev_ready) cudaEventDestroy(p->ev_ready);
  if (p->ev_xchg) cudaEventDestroy(p->ev_xchg);
  if (p->band_stream) cudaStreamDestroy(p->band_stream);
  if (p->copy_stream) cudaStreamDestroy(p->copy_stream);
  if (p->pipe_stream) cudaStreamDestroy(p->pipe_stream);
  for (cudaEvent_t ev : p->ev_copy) cudaEventDestroy(ev);
  if (p->ev_fork) cudaEventDestroy(p->ev_fork);
  if (p->ev_band) cudaEventDestroy(p->ev_band);
  for (cudaEvent_t ev : p->ev_pool) cudaEventDestroy(ev);
  cudaFree(p->dF);
  cudaFree(p->dS);
  cudaFree(p->dCrt);
  cudaFree(p->dW);
  cudaFree(p->dBlocks);
  cudaFree(p->dScratch);
  cudaFree(p->dSpec);
  cudaFree(p->dHostIn);
  cudaFree(p->dHostOut);
  cudaFree(p->dE[0]);
  cudaFree(p->dE[1]);
  cudaSetDevice(cur);
  delete p;
}

void fill_info(const HostPlan& hp, fftstencil_info* info) {
  std::memset(info, 0, sizeof *info);
  info->ndim = hp.ndim;
  info->T = hp.T;
  info->radius = hp.radius;
  info->halo = hp.h;
  for (int a = 0; a < 3; ++a) { info->tile[a] = a < hp.ndim ? hp.L[a] : 1; info->valid[a] = a < hp.ndim ? hp.S[a] : 1; }
  info->pfa[0] = hp.N1;
  info->pfa[1] = hp.N2;
  for (int a = 0; a < hp.ndim; ++a) info->extents[a] = hp.ext[a];
  info->tiles = hp.tiles;
  info->pairs = hp.pairs;
  info->band_blocks = (int64_t)(hp.band_blocks.size() / 8);
  info->flops_per_cell_step = hp.flops_per_cell_step;
  info->mma_flops_per_pass = hp.mma_flops_per_pair * (double)(hp.pair_hi - hp.pair_lo);
  info->smem_bytes = hp.fused_smem;
  info->nranks = hp.nranks;
  info->rank = hp.rank;
  info->row_begin = hp.row_lo;
  info->row_end = hp.row_hi;
  info->pair_begin = hp.pair_lo;
  info->pair_end = hp.pair_hi;
  info->interior_begin = hp.ipair_lo;
  info->interior_end = hp.ipair_hi;
  info->ghost_lo = hp.row_lo - hp.g0;
  info->ghost_hi = hp.g1 - hp.row_hi;
  info->algo = hp.algo;
  info->periodic = hp.periodic;
  info->engine = hp.engine;
  info->alu_ops_per_pass = hp.alu_ops_per_pair * (double)(hp.pair_hi - hp.pair_lo);
}

// Profiling: a (start, end) event pair around one launch; returns the pair index or -1.
long prof_begin(fftstencil_plan* p, int kind, cudaStream_t s) {
  if (!p->profiling) return -1;
  if (p->ev_used + 2 > p->ev_pool.size()) {
    for (int i = 0; i < 64; ++i) {
      cudaEvent_t ev;
      if (cudaEventCreate(&ev) != cudaSuccess) return -1;
      p->ev_pool.push_back(ev);
    }
    p->ev_kind.resize(p->ev_pool.size() / 2, 0);
  }
  const size_t i = p->ev_used;
  p->ev_used += 2;
  p->ev_kind[i / 2] = kind;
  cudaEventRecord(p->ev_pool[i], s);
  return (long)i;
}

void prof_end(fftstencil_plan* p, long i, cudaStream_t s) {
  if (i >= 0) cudaEventRecord(p->ev_pool[(size_t)i + 1], s);
}

int band_args(const fftstencil_plan* p, const double* src, double* dst, int t, BandArgs& b);

// One fused launch over pairs [pb, pe): src -> dst with t steps (t <= T), tile geometry of
// T.  The buffers hold global outer rows [g0, g1); only rows [row_lo, row_hi) are written.
int launch_fused(fftstencil_plan* p, const double* src, double* dst, int t, int64_t pb, int64_t pe,
                 cudaStream_t s) {
  if (pe <= pb) return FFTSTENCIL_OK;
  const HostPlan& hp = p->hp;
  const double* Sre = p->dS + (size_t)(t - 1) * 2 * p->spec_vol;
  const double* Sim = Sre + p->spec_vol;
  Window win;
  win.g0 = hp.g0;
  win.gn = hp.g1 - hp.g0;
  win.w_lo = hp.row_lo;
  win.w_hi = hp.row_hi;
  win.p_begin = pb;
  win.p_end = pe;
  const int64_t np = pe - pb;
  int64_t fg = p->grid_cap > 0 ? std::min(p->grid_cap, p->fused_grid) : p->fused_grid;
  if (p->max_ctas > 0) fg = std::min<int64_t>(fg, p->max_ctas);
  Bound bd;
  bd.wrap = hp.periodic;
  bd.shift = hp.periodic ? -hp.h : 0;
  const int64_t lim[3] = {hp.periodic ? hp.ext[0] : hp.ext[0] - hp.h,
                          hp.ndim > 1 ? (hp.periodic ? hp.ext[1] : hp.ext[1] - hp.h) : 0,
                          hp.ndim > 2 ? (hp.periodic ? hp.ext[2] : hp.ext[2] - hp.h) : 0};
  bd.lim0 = lim[0];
  bd.lim1 = lim[1];
  bd.lim2 = lim[2];
  cudaError_t e = cudaSuccess;
  const long pe_ = prof_begin(p, 0, s);
  if (hp.ndim == 2) {
    Fft2dArgs a;
    a.peer = p->peer_store;
    a.src = src;
    a.dst = dst;
    a.n0 = hp.ext[0];
    a.n1 = hp.ext[1];
    a.h = hp.h;
    a.S = hp.S[0];
    a.nt1 = hp.nt[1];
    a.npr = hp.npr;
    a.win = win;
    a.bd = bd;
    a.Sre = Sre;
    a.Sim = Sim;
    a.Fre = p->dF;
    a.spec = p->dSpec;
    if (hp.algo == 2) {
      // unfused ablation: forward -> HBM spectrum, multiply in HBM, inverse (3 launches)
      a.Fim = p->dF + (size_t)hp.L[0] * hp.L[0];
      const int grid = (int)std::min<int64_t>(fg, np);
      e = launch_unfused2d(hp.L[0], 1, a, grid, s);
      if (e == cudaSuccess) e = launch_spec_mul(p->dSpec, hp.pairs, hp.L[0], Sre, Sim, s);
      if (e == cudaSuccess) e = launch_unfused2d(hp.L[0], 2, a, grid, s);
      p->last_launches += 2;
    } else if (hp.algo == 1) {
      a.Fim = p->dF + 128;
      CUtensorMap tm;
      const uint64_t dims[2] = {(uint64_t)hp.ext[1], (uint64_t)(hp.g1 - hp.g0)};
      const uint32_t box[2] = {64, 64}, box_bf[2] = {16, 64};
      const bool bf = hp.engine == 1;
      const bool use_tma = p->use_tma && !hp.periodic && encode_tensor_map(&tm, src, 2, dims, bf ? box_bf : box, bf);
      if (bf)
        e = launch_fused2d_bf(a, use_tma ? &tm : nullptr, (int)std::min<int64_t>(fg, np), s);
      else
        e = launch_fused2d_ct(p->ct_cfg, a, use_tma ? &tm : nullptr, (int)std::min<int64_t>(fg, np), s);
    } else {
      a.Fim = p->dF + (size_t)hp.L[0] * hp.L[0];
      e = launch_fused2d(hp.L[0], p->variant, a, (int)std::min<int64_t>(fg, np), s);
    }
  } else if (hp.ndim == 1) {
    Fft1dArgs a;
    a.peer = p->peer_store;
    a.src = src;
    a.dst = dst;
    a.n = hp.ext[0];
    a.h = hp.h;
    a.S = hp.S[0];
    a.L = hp.L[0];
    a.ntiles = hp.tiles;
    a.win = win;
    a.bd = bd;
    a.Fre = p->dF;
    a.Fim = p->dF + 128;
    a.Sre = Sre;
    a.Sim = Sim;
    a.crt = p->dCrt;
    a.tw = p->dF + 256;
    if (hp.algo == 1 && hp.engine == 1) {
      // TMA staging when every tile starts on a 64-cell row of the (window) buffer
      CUtensorMap tm;
      const int64_t gn = hp.g1 - hp.g0;
      const bool aligned = !hp.periodic && hp.ext[0] % 64 == 0 && hp.S[0] % 64 == 0 && hp.g0 % 64 == 0 &&
                           gn % 64 == 0;
      const uint64_t dims[2] = {64, (uint64_t)(gn / 64)};
      const uint32_t box[2] = {16, 64};
      const bool use_tma = p->use_tma && aligned && encode_tensor_map(&tm, src, 2, dims, box, true);
      e = launch_fused1d_bf(a, use_tma ? &tm : nullptr, (int)std::min<int64_t>(fg, np), s);
    } else if (hp.algo == 1) {
      e = launch_fused1d_ct(a, (int)std::min<int64_t>(fg, np), s);
    } else {
      const int64_t blocks = (np + kFft1dWarpsPerBlock - 1) / kFft1dWarpsPerBlock;
      e = launch_fused1d(a, (int)std::max<int64_t>(1, std::min<int64_t>(fg, blocks)), s);
    }
  } else {
    Fft3dArgs a;
    a.peer = p->peer_store;
    a.src = src;
    a.dst = dst;
    a.n0 = hp.ext[0];
    a.n1 = hp.ext[1];
    a.n2 = hp.ext[2];
    a.h = hp.h;
    a.S = hp.S[0];
    a.nt1 = hp.nt[1];
    a.nt2 = hp.nt[2];
    a.npr = hp.npr;
    a.win = win;
    a.bd = bd;
    a.Fre = p->dF;
    a.Sre = Sre;
    a.Sim = Sim;
    a.blk0 = a.blk1 = 0;
    a.st32 = a.st16 = 0;
    {
      const bool al32 = (hp.S[0] % 4) == 0 && (hp.ext[2] % 4) == 0 && bd.shift % 4 == 0 &&
                        (reinterpret_cast<uintptr_t>(dst) & 31) == 0 && p->st256;
      for (int l2 = hp.h; l2 < hp.h + hp.S[0]; l2 += 2) {
        if (al32 && (l2 & 3) == 0 && l2 + 4 <= hp.h + hp.S[0]) {
          a.st32 |= 1 << l2;
          l2 += 2;
        } else {
          a.st16 |= 1 << l2;
        }
      }
    }
    if (hp.algo == 1 && hp.engine == 1 && !hp.periodic) {   // blocked traversal (kernel_fft3d_bf.cu)
      a.blk0 = a.blk1 = p->trav_blk;
      const int64_t ppu = hp.nt[1] * hp.npr;
      if (a.blk0 > 0 && (pb % ppu || pe % ppu)) a.blk0 = a.blk1 = 0;   // ranges of whole tile rows only
    }
    if (hp.algo == 1) {
      a.Fim = p->dF + 128;
      CUtensorMap tm;
      const uint64_t dims[3] = {(uint64_t)hp.ext[2], (uint64_t)hp.ext[1], (uint64_t)(hp.g1 - hp.g0)};
      const uint32_t box[3] = {16, 16, 16};
      const bool use_tma = p->use_tma && !hp.periodic && encode_tensor_map(&tm, src, 3, dims, box, hp.engine == 1);
      if (hp.engine == 1)
        e = launch_fused3d_bf(a, use_tma ? &tm : nullptr, (int)std::min<int64_t>(fg, np), s);
      else
        e = launch_fused3d_ct(a, use_tma ? &tm : nullptr, (int)std::min<int64_t>(fg, np), s);
    } else {
      a.Fim = p->dF + (size_t)hp.L[0] * hp.L[0];
      e = launch_fused3d(a, (int)std::min<int64_t>(fg, np), s);
    }
  }
  prof_end(p, pe_, s);
  if (e != cudaSuccess) return cuda_fail(e, "fused FFT-tile launch");
  ++p->last_launches;
  return FFTSTENCIL_OK;
}

// The band pass of one fused pass.  Concurrent mode: forked from `s` (after everything
// already enqueued there, i.e. after the pass that produced `src`) onto the band stream;
// band_join() makes `s` wait for it before the next pass touches either buffer.
// The band blocks of one pass (rows [band_clip_lo, band_clip_hi) when clipped: the pipelined
// run_host) as kernel arguments; returns the number of blocks.
int band_args(const fftstencil_plan* p, const double* src, double* dst, int t, BandArgs& b) {
  const HostPlan& hp = p->hp;
  int64_t i0 = 0, i1 = (int64_t)(hp.band_blocks.size() / 8);
  if (p->band_clip_lo > 0 || p->band_clip_hi < INT64_MAX) {   // blocks meeting the clip rows
    i0 = std::upper_bound(p->blk_lo.begin(), p->blk_lo.end(), p->band_clip_lo - p->blk_hmax) - p->blk_lo.begin();
    i1 = std::lower_bound(p->blk_lo.begin(), p->blk_lo.end(), p->band_clip_hi) - p->blk_lo.begin();
  }
  const int nb = (int)std::max<int64_t>(0, i1 - i0);
  b.src = src;
  b.dst = dst;
  for (int q = 0; q < 3; ++q) { b.n[q] = hp.n[q]; b.active[q] = q >= 3 - hp.ndim; }
  b.r = hp.radius;
  b.t = t;
  b.w = p->dW;
  b.blocks = p->dBlocks + 8 * i0;
  b.nblocks = nb;
  b.oax = 3 - hp.ndim;
  b.g0 = hp.g0;
  b.gn = hp.g1 - hp.g0;
  b.reference = p->band_reference;
  b.region_cells = hp.band_region_cells;
  b.ntaps = 0;
  for (double wv : hp.w) b.ntaps += wv != 0.0;
  b.clip_lo = p->band_clip_lo;
  b.clip_hi = p->band_clip_hi;
  b.peer = p->peer_store;
  return nb;
}

int launch_band_pass(fftstencil_plan* p, const double* src, double* dst, int t, cudaStream_t s,
                     bool forked = false) {
  BandArgs b;
  if (band_args(p, src, dst, t, b) == 0) return FFTSTENCIL_OK;
  cudaStream_t bs = s;
  if (p->band_concurrent && !forked) {
    cudaError_t e = cudaEventRecord(p->ev_fork, s);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(p->band_stream, p->ev_fork, 0);
    if (e != cudaSuccess) return cuda_fail(e, "band fork");
  }
  if (p->band_concurrent) bs = p->band_stream;
  const long pb = prof_begin(p, 1, bs);
  cudaError_t e = launch_band(b, p->band_smem, bs);
  prof_end(p, pb, bs);
  if (e != cudaSuccess) return cuda_fail(e, "band launch");
  if (p->band_concurrent) {
    if ((e = cudaEventRecord(p->ev_band, bs)) != cudaSuccess) return cuda_fail(e, "band event");
    p->band_pending = true;
  }
  ++p->last_launches;
  return FFTSTENCIL_OK;
}

int band_join(fftstencil_plan* p, cudaStream_t s) {
  if (!p->band_pending) return FFTSTENCIL_OK;
  p->band_pending = false;
  cudaError_t e = cudaStreamWaitEvent(s, p->ev_band, 0);
  return e == cudaSuccess ? FFTSTENCIL_OK : cuda_fail(e, "band join");
}

// Copy the (rank's) fixed ring from src (buffer rows start at global row src_off) into
// d0/d1 (buffer rows start at dst_off).
int copy_ring(fftstencil_plan* p, const double* src, int64_t src_off, double* d0, double* d1, int64_t dst_off,
              cudaStream_t s) {
  for (const Box& b : p->hp.ring_boxes) {
    BoxCopyArgs a;
    a.src = src;
    a.dst0 = d0;
    a.dst1 = d1;
    for (int q = 0; q < 3; ++q) { a.n[q] = p->hp.n[q]; a.lo[q] = b.lo[q]; a.hi[q] = b.hi[q]; }
    a.oax = 3 - p->hp.ndim;
    a.src_off = src_off;
    a.dst_off = dst_off;
    cudaError_t e = launch_box_copy(a, s);
    if (e != cudaSuccess) return cuda_fail(e, "ring copy launch");
    ++p->last_launches;
  }
  return FFTSTENCIL_OK;
}

// ---------------------------------------------------------------- single-GPU driver
int run_single(fftstencil_plan* p, const double* in, double* out, int64_t total_steps, cudaStream_t s) {
  const size_t bytes = p->grid_cells * sizeof(double);
  if (total_steps == 0) {
    if (in != out) {
      cudaError_t e = cudaMemcpyAsync(out, in, bytes, cudaMemcpyDeviceToDevice, s);
      if (e != cudaSuccess) return cuda_fail(e, "copy");
    }
    return FFTSTENCIL_OK;
  }
  const int T = p->hp.T;
  const int64_t nfull = total_steps / T;
  const int rem = (int)(total_steps % T);
  const int64_t passes = nfull + (rem ? 1 : 0);
  if (p->small1d) {
    const HostPlan& hp = p->hp;
    Small1dArgs a;
    a.in = in;
    a.out = out;
    a.n = hp.ext[0];
    a.h = hp.h;
    a.S = hp.S[0];
    a.L = hp.L[0];
    a.r = hp.radius;
    a.T = T;
    a.rem = rem;
    a.rmax = (int)std::min<int64_t>(hp.h + (int64_t)hp.radius * T, hp.ext[0]);
    a.ntiles = hp.tiles;
    a.passes = passes;
    a.Fre = p->dF;
    a.Fim = p->dF + 128;
    a.crt = p->dCrt;
    a.Sre_T = p->dS + (size_t)(T - 1) * 2 * p->spec_vol;
    a.Sim_T = a.Sre_T + p->spec_vol;
    a.Sre_rem = p->dS + (size_t)((rem ? rem : T) - 1) * 2 * p->spec_vol;
    a.Sim_rem = a.Sre_rem + p->spec_vol;
    a.w = p->dW;
    const long pb = prof_begin(p, 0, s);
    cudaError_t e = launch_small1d(a, s);
    prof_end(p, pb, s);
    if (e != cudaSuccess) return cuda_fail(e, "small 1D launch");
    ++p->last_launches;
    return FFTSTENCIL_OK;
  }
  // destination sequence: alternate out / scratch so the last pass writes `out`;
  // with in == out the first destination must be scratch (a final copy if needed).
  const bool alias = in == out;
  double* dsts[2];
  bool final_copy = false;
  if (!alias) {
    dsts[0] = (passes % 2) ? out : p->dScratch;
    dsts[1] = (passes % 2) ? p->dScratch : out;
  } else {
    dsts[0] = p->dScratch;
    dsts[1] = out;
    final_copy = (passes % 2) == 1;
  }
  int rc = copy_ring(p, in, 0, alias ? nullptr : out, passes > 1 || alias ? p->dScratch : nullptr, 0, s);
  if (rc) return rc;
  const double* src = in;
  for (int64_t i = 0; i < passes; ++i) {
    const int t = i < nfull ? T : rem;
    double* dst = dsts[i % 2];
    if ((rc = launch_band_pass(p, src, dst, t, s))) return rc;   // forked: overlaps the fused kernel
    if ((rc = launch_fused(p, src, dst, t, p->hp.pair_lo, p->hp.pair_hi, s))) return rc;
    if ((rc = band_join(p, s))) return rc;
    src = dst;
  }
  if (final_copy) {
    cudaError_t e = cudaMemcpyAsync(out, p->dScratch, bytes, cudaMemcpyDeviceToDevice, s);
    if (e != cudaSuccess) return cuda_fail(e, "final copy");
  }
  return FFTSTENCIL_OK;
}

// ---------------------------------------------------------------- multi-GPU driver pieces
double* owned_ptr(fftstencil_plan* p, int which) {
  return p->dE[which] + (size_t)(p->hp.row_lo - p->hp.g0) * p->row_cells;
}

int dist_begin(fftstencil_plan* p, const double* in, cudaStream_t s) {
  const size_t bytes = p->grid_cells * sizeof(double);
  p->ecur = 0;
  cudaError_t e = cudaMemcpyAsync(owned_ptr(p, 0), in, bytes, cudaMemcpyDeviceToDevice, s);
  if (e != cudaSuccess) return cuda_fail(e, "slab copy-in");
  return copy_ring(p, in, p->hp.row_lo, p->dE[1], nullptr, p->hp.g0, s);
}

int dist_end(fftstencil_plan* p, double* out, cudaStream_t s) {
  cudaError_t e = cudaMemcpyAsync(out, owned_ptr(p, p->ecur), p->grid_cells * sizeof(double),
                                  cudaMemcpyDeviceToDevice, s);
  if (e != cudaSuccess) return cuda_fail(e, "slab copy-out");
  return FFTSTENCIL_OK;
}

// NCCL halo exchange of the current buffer on the comm stream (after `s`'s prior work).
int nccl_exchange(fftstencil_plan* p, cudaStream_t s) {
  const HostPlan& hp = p->hp;
  double* buf = p->dE[p->ecur];
  const size_t rc_ = p->row_cells;
  const int64_t glo = hp.row_lo - hp.g0, ghi = hp.g1 - hp.row_hi, own = hp.row_hi - hp.row_lo;
  cudaError_t e = cudaEventRecord(p->ev_ready, s);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(p->comm_stream, p->ev_ready, 0);
  if (e != cudaSuccess) return cuda_fail(e, "exchange ordering");
  ncclResult_t r = ncclGroupStart();
  if (r == ncclSuccess && hp.rank > 0) {
    r = ncclSend(buf + (size_t)glo * rc_, (size_t)hp.h * rc_, ncclDouble, hp.rank - 1, p->comm, p->comm_stream);
    if (r == ncclSuccess) r = ncclRecv(buf, (size_t)glo * rc_, ncclDouble, hp.rank - 1, p->comm, p->comm_stream);
  }
  if (r == ncclSuccess && hp.rank < hp.nranks - 1) {
    r = ncclSend(buf + (size_t)(glo + own - hp.h) * rc_, (size_t)hp.h * rc_, ncclDouble, hp.rank + 1, p->comm,
                 p->comm_stream);
    if (r == ncclSuccess)
      r = ncclRecv(buf + (size_t)(glo + own) * rc_, (size_t)ghi * rc_, ncclDouble, hp.rank + 1, p->comm,
                   p->comm_stream);
  }
  const ncclResult_t r2 = ncclGroupEnd();
  if (r != ncclSuccess) return nccl_fail(r, "halo send/recv");
  if (r2 != ncclSuccess) return nccl_fail(r2, "halo group");
  e = cudaEventRecord(p->ev_xchg, p->comm_stream);
  if (e != cudaSuccess) return cuda_fail(e, "exchange event");
  return FFTSTENCIL_OK;
}

// ---- peer transport: push own boundary rows into the neighbours' halo rows, signal, wait ----
// Rows [row_lo, row_lo + h) of buffer `b` go to the lower neighbour's halo (its rows from
// row_lo on, at its local row row_lo - g0_lower); rows [row_hi - h, row_hi) to the upper
// neighbour's (its local rows from 0).  Copy engine over NVLink (same-device copy when the
// "neighbour" is another process on this GPU), ordered on `s` after the pass that wrote them.
// Here from this rank's buffer `from` into the neighbours' buffer `to`.
int peer_push_from(fftstencil_plan* p, int from, int to, cudaStream_t s) {
  const HostPlan& hp = p->hp;
  const size_t rc_ = p->row_cells, bytes = (size_t)hp.h * rc_ * sizeof(double);
  cudaError_t e = cudaSuccess;
  if (hp.rank > 0)
    e = cudaMemcpyAsync(p->pE[0][to] + (size_t)(hp.row_lo - p->pG0[0]) * rc_,
                        p->dE[from] + (size_t)(hp.row_lo - hp.g0) * rc_, bytes, cudaMemcpyDeviceToDevice, s);
  if (e == cudaSuccess && hp.rank < hp.nranks - 1)
    e = cudaMemcpyAsync(p->pE[1][to] + (size_t)(hp.row_hi - hp.h - p->pG0[1]) * rc_,
                        p->dE[from] + (size_t)(hp.row_hi - hp.h - hp.g0) * rc_, bytes, cudaMemcpyDeviceToDevice, s);
  return e == cudaSuccess ? FFTSTENCIL_OK : cuda_fail(e, "peer halo push");
}

// Epoch ++ written into both neighbours' flag words (stream-ordered after the push; the write
// carries a memory barrier, so the neighbour sees the rows before the flag).
int peer_signal(fftstencil_plan* p, uint32_t e, cudaStream_t s) {
  const HostPlan& hp = p->hp;
  p->epoch = e;
  CUresult r = CUDA_SUCCESS;
  if (hp.rank > 0) r = write_value_fn()((CUstream)s, (CUdeviceptr)(p->pFlags[0] + 1), p->epoch, 0);
  if (r == CUDA_SUCCESS && hp.rank < hp.nranks - 1)
    r = write_value_fn()((CUstream)s, (CUdeviceptr)(p->pFlags[1] + 0), p->epoch, 0);
  if (r != CUDA_SUCCESS) {
    set_error("cuStreamWriteValue32 failed (" + std::to_string((int)r) + ")");
    return FFTSTENCIL_ECUDA;
  }
  return FFTSTENCIL_OK;
}

// `s` waits until both neighbours have signalled as often as this rank.
int peer_wait(fftstencil_plan* p, uint32_t target, cudaStream_t s) {
  const HostPlan& hp = p->hp;
  // peer copies land in this device's memory before the writer's flag (the write-value carries a
  // memory barrier); no remote-write flush is needed (that flag is for third-party RDMA writers)
  const unsigned flags = CU_STREAM_WAIT_VALUE_GEQ;
  CUresult r = CUDA_SUCCESS;
  if (hp.rank > 0) r = wait_value_fn()((CUstream)s, (CUdeviceptr)(p->dFlags + 0), target, flags);
  if (r == CUDA_SUCCESS && hp.rank < hp.nranks - 1)
    r = wait_value_fn()((CUstream)s, (CUdeviceptr)(p->dFlags + 1), target, flags);
  if (r != CUDA_SUCCESS) {
    set_error("cuStreamWaitValue32 failed (" + std::to_string((int)r) + ")");
    return FFTSTENCIL_ECUDA;
  }
  return FFTSTENCIL_OK;
}

// One run over the peer transport.  Per run every rank signals P + 1 times (after the copy-in,
// after every pass but the last, at the end), so the ranks stay in lockstep:
//   wait (neighbours done with the previous run: its halo rows are free) -> copy-in, push
//   buffer 0, signal -> per pass: halo-free pairs, wait, edge pairs + band, push dst, signal.
// A neighbour writes this rank's buffer b only after the pass that last read it (it waited
// for that pass's signal first), and never the owned rows the passes write.
int run_dist_peer(fftstencil_plan* p, const double* in, double* out, int64_t total_steps, cudaStream_t s) {
  const HostPlan& hp = p->hp;
  // fused pushes need the ALU kernels' PEER instantiations and the cone band kernel
  int taps = 1;
  for (int q = 0; q < hp.ndim; ++q) taps *= 2 * hp.radius + 1;
  const bool fused = p->peer_fused && hp.algo == 1 && hp.engine == 1 && !p->band_reference && taps <= 512;
  p->last_peer_fused = fused;
  // the schedule (plan.cpp build_peer_schedule; replayed on the CPU by tests/test_dist.py) and
  // its execution, op by op
  std::vector<int64_t> ops;
  int rc = build_peer_schedule(hp, total_steps, fused, p->epoch, ops);
  if (rc) { set_error("peer schedule"); return rc; }
  const int T = hp.T;
  const int64_t nfull = total_steps / T;
  for (size_t i = 0; i < ops.size() && !rc; i += 4) {
    const int64_t op = ops[i], a = ops[i + 1], b = ops[i + 2], c = ops[i + 3];
    const int t = a <= nfull ? T : (int)(total_steps % T);
    switch (op) {
      case 0: rc = peer_wait(p, (uint32_t)a, s); break;
      case 1: rc = dist_begin(p, in, s); break;
      case 2: rc = peer_push_from(p, (int)a, (int)b, s); break;
      case 3: rc = peer_signal(p, (uint32_t)a, s); break;
      case 4: rc = launch_fused(p, p->dE[b], p->dE[b ^ 1], t, hp.ipair_lo, hp.ipair_hi, s); break;
      case 5: {
        const double* src = p->dE[b];
        double* dst = p->dE[b ^ 1];
        if (c) {   // the boundary rows' producers store them into the neighbours' buffer b ^ 1 too
          p->peer_store.lo = hp.rank > 0 ? p->pE[0][b ^ 1] : nullptr;
          p->peer_store.lo_end = hp.row_lo + hp.h;
          p->peer_store.lo_g0 = p->pG0[0];
          p->peer_store.hi = hp.rank < hp.nranks - 1 ? p->pE[1][b ^ 1] : nullptr;
          p->peer_store.hi_begin = hp.row_hi - hp.h;
          p->peer_store.hi_g0 = p->pG0[1];
        }
        rc = launch_fused(p, src, dst, t, hp.pair_lo, hp.ipair_lo, s);
        if (!rc) rc = launch_fused(p, src, dst, t, hp.ipair_hi, hp.pair_hi, s);
        if (!rc) rc = launch_band_pass(p, src, dst, t, s);
        p->peer_store = PeerStore{nullptr, nullptr, 0, 0, 0, 0};
        if (!rc) rc = band_join(p, s);
        break;
      }
      default:
        p->ecur = (int)a;
        rc = dist_end(p, out, s);
    }
  }
  return rc;
}

// One pass of a dist rank: interior pairs overlap the exchange (if `xchg`), then the
// halo-dependent pairs and the band.
int dist_pass(fftstencil_plan* p, int t, bool xchg, cudaStream_t s) {
  const HostPlan& hp = p->hp;
  const double* src = p->dE[p->ecur];
  double* dst = p->dE[p->ecur ^ 1];
  int rc;
  if (xchg && (rc = nccl_exchange(p, s))) return rc;
  if ((rc = launch_fused(p, src, dst, t, hp.ipair_lo, hp.ipair_hi, s))) return rc;
  if (xchg) {
    cudaError_t e = cudaStreamWaitEvent(s, p->ev_xchg, 0);
    if (e != cudaSuccess) return cuda_fail(e, "wait for halo exchange");
  }
  if ((rc = launch_fused(p, src, dst, t, hp.pair_lo, hp.ipair_lo, s))) return rc;
  if ((rc = launch_fused(p, src, dst, t, hp.ipair_hi, hp.pair_hi, s))) return rc;
  if ((rc = launch_band_pass(p, src, dst, t, s))) return rc;
  if ((rc = band_join(p, s))) return rc;
  p->ecur ^= 1;
  return FFTSTENCIL_OK;
}

int run_dist(fftstencil_plan* p, const double* in, double* out, int64_t total_steps, cudaStream_t s) {
  if (p->loopback) {
    set_error("a loopback rank runs only through fftstencil_run_group");
    return FFTSTENCIL_EINVAL;
  }
  if (total_steps == 0) {
    if (in != out) {
      cudaError_t e = cudaMemcpyAsync(out, in, p->grid_cells * sizeof(double), cudaMemcpyDeviceToDevice, s);
      if (e != cudaSuccess) return cuda_fail(e, "copy");
    }
    return FFTSTENCIL_OK;
  }
  if (p->peer) {
    if (!p->peer_connected) {
      set_error("a peer-transport rank must be connected (fftstencil_peer_connect) before it runs");
      return FFTSTENCIL_EINVAL;
    }
    return run_dist_peer(p, in, out, total_steps, s);
  }
  int rc = dist_begin(p, in, s);
  if (rc) return rc;
  const int T = p->hp.T;
  const int64_t nfull = total_steps / T;
  const int rem = (int)(total_steps % T);
  for (int64_t i = 0; i < nfull + (rem ? 1 : 0); ++i)
    if ((rc = dist_pass(p, i < nfull ? T : rem, true, s))) return rc;
  return dist_end(p, out, s);
}

// Allocates and uploads everything a plan needs after its host plan is built.
int setup_device(fftstencil_plan* p) {
  HostPlan& hp = p->hp;
  cudaError_t e = cudaGetDevice(&p->device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
  e = cudaDeviceGetAttribute(&p->sm_count, cudaDevAttrMultiProcessorCount, p->device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceGetAttribute");

  size_t acc = 0;
  std::vector<double> F(hp.Fre);
  F.insert(F.end(), hp.Fim.begin(), hp.Fim.end());
  F.insert(F.end(), hp.tw.begin(), hp.tw.end());   // factored 1D: [Fre 128 | Fim 128 | w4096]
  if (hp.ndim == 2 && (hp.algo == 0 || hp.algo == 2)) {
    // the dense 2D kernel reads F with columns permuted within groups of 8 (device_common.cuh)
    const int L = hp.L[0];
    for (int plane = 0; plane < 2; ++plane)
      for (int r = 0; r < L; ++r)
        for (int c = 0; c < L; ++c)
          F[(size_t)plane * L * L + (size_t)r * L + ((c & ~7) | ((c & 1) << 2) | ((c & 7) >> 1))] =
              (plane ? hp.Fim : hp.Fre)[(size_t)r * L + c];
  }
  p->spec_vol = hp.Sre[0].size();
  std::vector<double> Sv;
  Sv.reserve((size_t)hp.T * 2 * p->spec_vol);
  for (int t = 0; t < hp.T; ++t) {
    Sv.insert(Sv.end(), hp.Sre[t].begin(), hp.Sre[t].end());
    Sv.insert(Sv.end(), hp.Sim[t].begin(), hp.Sim[t].end());
  }
  p->row_cells = 1;
  for (int a = 1; a < hp.ndim; ++a) p->row_cells *= (size_t)hp.ext[a];
  p->grid_cells = p->row_cells * (size_t)(hp.row_hi - hp.row_lo);
  // band blocks sorted by their outer-axis start (blocks are independent), so a row range of
  // the pipelined run_host maps to one contiguous index range
  std::vector<int32_t> blocks(hp.band_blocks);
  {
    const int oax = 3 - hp.ndim;
    const size_t nb = blocks.size() / 8;
    std::vector<size_t> order(nb);
    for (size_t i = 0; i < nb; ++i) order[i] = i;
    std::stable_sort(order.begin(), order.end(), [&](size_t x, size_t y) {
      return hp.band_blocks[8 * x + oax] < hp.band_blocks[8 * y + oax];
    });
    p->blk_lo.resize(nb);
    for (size_t i = 0; i < nb; ++i) {
      for (int q = 0; q < 8; ++q) blocks[8 * i + q] = hp.band_blocks[8 * order[i] + q];
      p->blk_lo[i] = blocks[8 * i + oax];
      p->blk_hmax = std::max<int64_t>(p->blk_hmax, blocks[8 * i + 3 + oax] - blocks[8 * i + oax]);
    }
  }
  if ((e = upload(&p->dF, F.data(), F.size(), acc)) != cudaSuccess ||
      (e = upload(&p->dS, Sv.data(), Sv.size(), acc)) != cudaSuccess ||
      (e = upload(&p->dW, hp.w.data(), hp.w.size(), acc)) != cudaSuccess ||
      (e = upload(&p->dBlocks, blocks.data(), blocks.size(), acc)) != cudaSuccess ||
      (hp.ndim == 1 && (e = upload(&p->dCrt, hp.crt.data(), hp.crt.size(), acc)) != cudaSuccess))
    return cuda_fail(e, "device upload");
  if (!p->dist) {
    e = cudaMalloc((void**)&p->dScratch, p->grid_cells * sizeof(double));
    if (e != cudaSuccess) return cuda_fail(e, "scratch grid allocation");
    acc += p->grid_cells * sizeof(double);
  } else {
    const size_t ecells = p->row_cells * (size_t)(hp.g1 - hp.g0);
    for (int k = 0; k < 2; ++k) {
      e = cudaMalloc((void**)&p->dE[k], ecells * sizeof(double));
      if (e != cudaSuccess) return cuda_fail(e, "slab buffer allocation");
      acc += ecells * sizeof(double);
    }
  }
  p->device_bytes = acc;

  int occ = 0;
  if (hp.ndim == 2 && hp.algo == 1) {
    if (const char* v = std::getenv("FFTSTENCIL_CT_CFG")) p->ct_cfg = std::atoi(v);
    if (const char* v = std::getenv("FFTSTENCIL_TMA")) p->use_tma = std::atoi(v) != 0;
    e = hp.engine == 1 ? fused2d_bf_configure(&occ) : fused2d_ct_configure(p->ct_cfg, &occ);
    if (e == cudaErrorInvalidValue) {
      set_error("FFTSTENCIL_CT_CFG must be one of 81, 82, 84, 161, 162");
      return FFTSTENCIL_EINVAL;
    }
    if (e != cudaSuccess) return cuda_fail(e, "factored 2D kernel configuration");
  } else if (hp.ndim == 2) {
    // double-buffered prefetch pays only where it does not cost occupancy (profiles/r01_variants.txt)
    p->variant = hp.L[0] >= 56 ? 1 : 0;
    if (hp.algo == 2) {
      const size_t sb = (size_t)hp.pairs * 2 * hp.L[0] * hp.L[0] * sizeof(double);
      e = cudaMalloc((void**)&p->dSpec, sb);
      if (e != cudaSuccess) return cuda_fail(e, "unfused spectrum buffer");
      p->device_bytes += sb;
    }
    if (const char* v = std::getenv("FFTSTENCIL_VARIANT")) p->variant = std::atoi(v);
    if (p->variant < 0 || p->variant > 2) {
      set_error("FFTSTENCIL_VARIANT must be 0, 1 or 2");
      return FFTSTENCIL_EINVAL;
    }
    if (hp.algo == 2) p->variant = 0;   // the unfused stages use the V = 0 layout
    e = fused2d_configure(hp.L[0], p->variant, &occ);
    if (e != cudaSuccess) return cuda_fail(e, "fused 2D kernel configuration");
  } else if (hp.ndim == 3 && hp.algo == 1) {
    if (const char* v = std::getenv("FFTSTENCIL_TMA")) p->use_tma = std::atoi(v) != 0;
    e = hp.engine == 1 ? fused3d_bf_configure(&occ) : fused3d_ct_configure(&occ);
    if (e != cudaSuccess) return cuda_fail(e, "factored 3D kernel configuration");
  } else if (hp.ndim == 3) {
    e = fused3d_configure(&occ);
    if (e != cudaSuccess) return cuda_fail(e, "fused 3D kernel configuration");
  } else if (hp.algo == 1 && hp.engine == 1) {
    if (const char* v = std::getenv("FFTSTENCIL_TMA")) p->use_tma = std::atoi(v) != 0;
    e = fused1d_bf_configure(&occ);
    if (e != cudaSuccess) return cuda_fail(e, "factored 1D kernel configuration");
  } else if (hp.algo == 1) {
    e = fused1d_ct_configure(&occ);
    if (e != cudaSuccess) return cuda_fail(e, "factored 1D kernel configuration");
  } else {
    e = fused1d_configure(&occ);
    if (e != cudaSuccess) return cuda_fail(e, "fused 1D kernel configuration");
  }
  if (occ < 1) {
    set_error("fused kernel cannot be resident on this device");
    return FFTSTENCIL_EUNSUPPORTED;
  }
  p->fused_grid = (int)std::max<int64_t>(1, (int64_t)p->sm_count * occ);
  // 1D: the band is two blocks of t (~1000) sequential direct steps, as long as the fused pass;
  // the register-full ALU kernel (one CTA per SM) would serialise it, so leave it its SMs
  if (hp.ndim == 1 && hp.algo == 1 && hp.engine == 1 && !hp.band_blocks.empty())
    p->fused_grid = (int)std::max<int64_t>(1, p->fused_grid - (int64_t)(hp.band_blocks.size() / 8));
  if (const char* v = std::getenv("FFTSTENCIL_MAX_CTAS")) p->max_ctas = std::max(0, std::atoi(v));
  if (const char* v = std::getenv("FFTSTENCIL_3D_TRAV")) p->trav_blk = std::max(0, std::atoi(v));
  if (const char* v = std::getenv("FFTSTENCIL_ST256")) p->st256 = std::atoi(v) != 0;
  if (const char* v = std::getenv("FFTSTENCIL_PEER_FUSED")) p->peer_fused = std::atoi(v) != 0;
  if (const char* v = std::getenv("FFTSTENCIL_BAND")) p->band_reference = !std::strcmp(v, "reference");
  // 2D plans run the band on its side stream, concurrent with the fused kernel.  3D plans run it
  // before the fused kernel on the run stream in fftstencil_run: concurrent, its CTAs hold SMs the
  // register-full fused CTAs then wait for (Heat-3D 224.1 vs 228.1 serialised with the round-1
  // band, profiles/r02_band3d.txt); with the faster cp.async / fdiv band the comparison depends on
  // the box: +0.55 % concurrent on one, -1.5 % on a power-capped one where the overlap lowers the
  // SM clock (1935 vs 1950 MHz) (profiles/r02_bandstream2.txt, r02_bandstream3.txt) -- so the device
  // path stays serialised, while the pipelined run_host, whose many small band launches gain from
  // overlapping the fused items on both boxes (e2e +0.6 / +0.9 %), runs them concurrently
  // (band_e2e_concurrent).  FFTSTENCIL_BAND_STREAM=0|1 and FFTSTENCIL_E2E_BAND_STREAM=0|1 override.
  if (hp.ndim == 3) p->band_concurrent = false;
  if (const char* v = std::getenv("FFTSTENCIL_BAND_STREAM")) p->band_concurrent = std::atoi(v) != 0;
  if (const char* v = std::getenv("FFTSTENCIL_E2E_BAND_STREAM")) p->band_e2e_concurrent = std::atoi(v) != 0;
  if (hp.band_blocks.empty()) p->band_concurrent = p->band_e2e_concurrent = false;
  if (p->band_concurrent || p->band_e2e_concurrent) {
    e = cudaStreamCreateWithFlags(&p->band_stream, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->ev_band, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_fail(e, "band stream/events");
  }
  // small non-periodic 1D grids: the whole run in one launch, the grid in shared memory
  // (FFTSTENCIL_SMALL1D=0 keeps the per-pass driver)
  p->small1d = hp.ndim == 1 && hp.algo == 0 && !hp.periodic && !p->dist && hp.ext[0] <= kSmall1dMaxCells &&
               hp.ext[0] >= 4 * (int64_t)hp.h + 2 * hp.radius && std::min<int64_t>(2 * hp.h, hp.ext[0]) <= kSmall1dMaxBand;
  if (const char* v = std::getenv("FFTSTENCIL_SMALL1D")) p->small1d = p->small1d && std::atoi(v) != 0;
  if (p->small1d && (e = small1d_configure()) != cudaSuccess) return cuda_fail(e, "small 1D kernel configuration");
  p->band_smem = (size_t)2 * hp.band_region_cells * sizeof(double);
  if (p->band_smem > 0) {
    e = band_configure(p->band_smem);
    if (e != cudaSuccess) return cuda_fail(e, "band kernel configuration");
  }
  return FFTSTENCIL_OK;
}

}  // namespace

namespace fstencil {
bool encode_tensor_map(CUtensorMap* map, const void* base, int rank, const uint64_t* dims, const uint32_t* box,
                       bool swizzle128) {
  EncodeTiledFn fn = encode_fn();
  if (!fn || rank < 1 || rank > 3 || (reinterpret_cast<uintptr_t>(base) & 15)) return false;
  cuuint64_t gdim[3], gstride[2];
  cuuint32_t bdim[3], es[3] = {1, 1, 1};
  uint64_t stride = sizeof(double);
  for (int i = 0; i < rank; ++i) {
    gdim[i] = dims[i];
    bdim[i] = box[i];
    if (i > 0) {
      gstride[i - 1] = stride;
      if (stride % 16) return false;
    }
    stride *= dims[i];
  }
  return fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, (cuuint32_t)rank, const_cast<void*>(base), gdim, gstride, bdim, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE,
            swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
}  // namespace fstencil

extern "C" {

const char* fftstencil_last_error(void) { return g_last_error.c_str(); }

int fftstencil_describe(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                        fftstencil_info* info) {
  return fftstencil_describe_dist(ndim, extents, weights, radius, T, 1, 0, info);
}

int fftstencil_describe_ex(int ndim, const int64_t* extents, const double* weights, int radius, int T, int flags,
                           fftstencil_info* info) {
  if (!info) { set_error("info must be non-NULL"); return FFTSTENCIL_EINVAL; }
  if (flags & ~FFTSTENCIL_PERIODIC) { set_error("unknown flags"); return FFTSTENCIL_EINVAL; }
  HostPlan hp;
  std::string err;
  const int rc = build_host_plan(ndim, extents, weights, radius, T, hp, err, 1, 0, env_algo(),
                                 (flags & FFTSTENCIL_PERIODIC) ? 1 : 0);
  if (rc != FFTSTENCIL_OK) { set_error(err); return rc; }
  fill_info(hp, info);
  clear_error();
  return FFTSTENCIL_OK;
}

int fftstencil_describe_dist(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                             int nranks, int rank, fftstencil_info* info) {
  if (!info) { set_error("info must be non-NULL"); return FFTSTENCIL_EINVAL; }
  HostPlan hp;
  std::string err;
  const int rc = build_host_plan(ndim, extents, weights, radius, T, hp, err, nranks, rank, env_algo());
  if (rc != FFTSTENCIL_OK) { set_error(err); return rc; }
  fill_info(hp, info);
  clear_error();
  return FFTSTENCIL_OK;
}

int64_t fftstencil_peer_schedule(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                                 int nranks, int rank, int64_t total_steps, int fused, int64_t epoch0, int64_t* out,
                                 int64_t cap) {
  HostPlan hp;
  std::string err;
  int rc = build_host_plan(ndim, extents, weights, radius, T, hp, err, nranks, rank, env_algo());
  if (rc != FFTSTENCIL_OK) { set_error(err); return rc; }
  std::vector<int64_t> ops;
  if ((rc = build_peer_schedule(hp, total_steps, fused != 0, epoch0, ops)) != FFTSTENCIL_OK) {
    set_error("nranks must be >= 2 and total_steps >= 0");
    return rc;
  }
  const int64_t n = (int64_t)ops.size() / 4;
  if (out) {
    if (cap < n) { set_error("cap smaller than the number of ops"); return FFTSTENCIL_EINVAL; }
    std::memcpy(out, ops.data(), ops.size() * sizeof(int64_t));
  }
  clear_error();
  return n;
}

int64_t fftstencil_e2e_schedule(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                                int64_t total_steps, int chunks, int depth, int64_t* out, int64_t cap) {
  HostPlan hp;
  std::string err;
  int rc = build_host_plan(ndim, extents, weights, radius, T, hp, err, 1, 0, env_algo());
  if (rc != FFTSTENCIL_OK) { set_error(err); return rc; }
  std::vector<int64_t> ops;
  if ((rc = build_e2e_schedule(hp, total_steps, chunks, depth, ops, pipe_tail_depth(), pipe_ramp())) != FFTSTENCIL_OK) {
    set_error("plan not eligible for the pipelined run_host schedule");
    return rc;
  }
  const int64_t n = (int64_t)ops.size() / 4;
  if (out) {
    if (cap < n) { set_error("cap smaller than the number of ops"); return FFTSTENCIL_EINVAL; }
    std::memcpy(out, ops.data(), ops.size() * sizeof(int64_t));
  }
  clear_error();
  return n;
}

int64_t fftstencil_export_aux(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                              int which, int axis, int t, double* out, int64_t cap) {
  HostPlan hp;
  std::string err;
  const int rc = build_host_plan(ndim, extents, weights, radius, T, hp, err, 1, 0, env_algo());
  if (rc != FFTSTENCIL_OK) { set_error(err); return rc; }
  std::vector<double> v;
  if (which == 0) {
    int L, row0 = 0, ld;
    if (hp.ndim == 1 && hp.algo == 1 && hp.engine == 1) {
      // ALU engine: axis 0 = w64^m (m < 64), axis 2 = w4096^m (m < 256)
      if (axis != 0 && axis != 2) { set_error("axis must be 0 (w64^m) or 2 (w4096^m) for the ALU engine"); return FFTSTENCIL_EINVAL; }
      if (axis == 0)
        for (int m = 0; m < 64; ++m) { v.push_back(hp.Fre[m]); v.push_back(hp.Fim[m]); }
      else
        v.assign(hp.tw.begin(), hp.tw.end());
      L = 0;
    } else if (hp.ndim == 1 && hp.algo == 1) {
      // factored 1D: axis 0 = F_8, 1 = twiddles w64^(ka lb) (8 x 8), 2 = w4096^(a c) (64 x 64)
      if (axis < 0 || axis > 2) { set_error("axis must be 0 (F_8), 1 (w64) or 2 (w4096)"); return FFTSTENCIL_EINVAL; }
      if (axis == 2) {
        v.assign(hp.tw.begin(), hp.tw.end());
        L = 0;
      } else {
        L = 8;
      }
      row0 = 8 * (axis & 1);
      ld = 8;
    } else if (hp.ndim == 1) {
      if (axis < 0 || axis > 1) { set_error("axis must be 0 (N1) or 1 (N2) for 1D"); return FFTSTENCIL_EINVAL; }
      L = axis == 0 ? hp.N1 : hp.N2;
      row0 = axis == 0 ? 0 : 8;
      ld = 8;
    } else if (hp.ndim == 2 && hp.algo == 1 && hp.engine == 1) {
      // radix-8 ALU engine: axis 0 = the w64^m table, m = 0..63
      if (axis != 0) { set_error("axis must be 0 (w64^m) for the ALU engine"); return FFTSTENCIL_EINVAL; }
      for (int m = 0; m < 64; ++m) { v.push_back(hp.Fre[m]); v.push_back(hp.Fim[m]); }
      L = 0;
    } else if (hp.ndim == 2 && hp.algo == 1) {
      if (axis < 0 || axis > 1) { set_error("axis must be 0 (F_8) or 1 (twiddles)"); return FFTSTENCIL_EINVAL; }
      L = 8;
      row0 = 8 * axis;
      ld = 8;
    } else if (hp.ndim == 3 && hp.algo == 1) {
      if (axis < 0 || axis > 1) { set_error("axis must be 0 (F_8) or 1 (w16^k)"); return FFTSTENCIL_EINVAL; }
      if (axis == 1) {
        for (int k = 0; k < 16; ++k) { v.push_back(hp.Fre[64 + k]); v.push_back(hp.Fim[64 + k]); }
        L = 0;
      } else {
        L = 8;
      }
      row0 = 0;
      ld = 8;
    } else {
      if (axis < 0 || axis >= hp.ndim) { set_error("axis out of range"); return FFTSTENCIL_EINVAL; }
      L = hp.L[axis];
      ld = hp.L[0];
    }
    for (int j = 0; j < L; ++j)
      for (int k = 0; k < L; ++k) {
        v.push_back(hp.Fre[(size_t)(row0 + j) * ld + k]);
        v.push_back(hp.Fim[(size_t)(row0 + j) * ld + k]);
      }
  } else if (which == 1) {
    if (t < 1 || t > hp.T) { set_error("t must be in 1..T"); return FFTSTENCIL_EINVAL; }
    const auto& re = hp.Sre[t - 1];
    const auto& im = hp.Sim[t - 1];
    for (size_t i = 0; i < re.size(); ++i) { v.push_back(re[i]); v.push_back(im[i]); }
  } else if (which == 2) {
    for (int64_t ti = 0; ti < hp.tiles; ++ti) {
      int64_t rem = ti, idx[3] = {0, 0, 0};
      for (int a = hp.ndim - 1; a >= 0; --a) { idx[a] = rem % hp.nt[a]; rem /= hp.nt[a]; }
      for (int a = 0; a < hp.ndim; ++a) {
        const int64_t o = idx[a] * hp.S[a] - (hp.periodic ? hp.h : 0);
        const int64_t first = o + hp.h;
        const int64_t last = std::min<int64_t>(o + hp.h + hp.S[a], hp.periodic ? hp.ext[a] : hp.ext[a] - hp.h);
        v.push_back((double)o);
        v.push_back((double)first);
        v.push_back((double)(last - first));
      }
    }
  } else if (which == 3) {
    if (hp.ndim != 1 || hp.crt.empty()) { set_error("the PFA map exists for 1D prime-factor plans only"); return FFTSTENCIL_EINVAL; }
    for (int l1 = 0; l1 < hp.N1; ++l1)
      for (int l2 = 0; l2 < hp.N2; ++l2) v.push_back((double)hp.crt[l1 * 8 + l2]);
  } else if (which == 4) {
    // band blocks: 7 values per block (lo[3], hi[3], face) in embedded coordinates
    for (size_t b = 0; b + 8 <= hp.band_blocks.size(); b += 8)
      for (int q = 0; q < 7; ++q) v.push_back((double)hp.band_blocks[b + q]);
  } else if (which == 5) {
    for (const Box& b : hp.ring_boxes) {
      for (int q = 0; q < 3; ++q) v.push_back((double)b.lo[q]);
      for (int q = 0; q < 3; ++q) v.push_back((double)b.hi[q]);
    }
  } else {
    set_error("unknown table");
    return FFTSTENCIL_EINVAL;
  }
  if (out) {
    if (cap < (int64_t)v.size()) { set_error("output buffer too small"); return FFTSTENCIL_EINVAL; }
    std::memcpy(out, v.data(), v.size() * sizeof(double));
  }
  clear_error();
  return (int64_t)v.size();
}

fftstencil_plan* fftstencil_plan_create(int ndim, const int64_t* extents, const double* weights, int radius,
                                        int T) {
  return fftstencil_plan_create_ex(ndim, extents, weights, radius, T, 0);
}

fftstencil_plan* fftstencil_plan_create_ex(int ndim, const int64_t* extents, const double* weights, int radius,
                                           int T, int flags) {
  if (flags & ~FFTSTENCIL_PERIODIC) { set_error("unknown flags"); return nullptr; }
  fftstencil_plan* p = new (std::nothrow) fftstencil_plan();
  if (!p) { set_error("host allocation failed"); return nullptr; }
  std::string err;
  int rc = build_host_plan(ndim, extents, weights, radius, T, p->hp, err, 1, 0, env_algo(),
                           (flags & FFTSTENCIL_PERIODIC) ? 1 : 0);
  if (rc != FFTSTENCIL_OK) { set_error(err); delete p; return nullptr; }
  if (setup_device(p) != FFTSTENCIL_OK) { free_plan(p); return nullptr; }
  clear_error();
  return p;
}

fftstencil_plan* fftstencil_plan_create_dist(int ndim, const int64_t* extents, const double* weights, int radius,
                                             int T, int nranks, int rank, const void* nccl_unique_id) {
  if (nranks == 1 && rank == 0) return fftstencil_plan_create(ndim, extents, weights, radius, T);
  fftstencil_plan* p = new (std::nothrow) fftstencil_plan();
  if (!p) { set_error("host allocation failed"); return nullptr; }
  std::string err;
  int rc = build_host_plan(ndim, extents, weights, radius, T, p->hp, err, nranks, rank, env_algo());
  if (rc != FFTSTENCIL_OK) { set_error(err); delete p; return nullptr; }
  p->dist = true;
  p->loopback = nccl_unique_id == nullptr;
  if (setup_device(p) != FFTSTENCIL_OK) { free_plan(p); return nullptr; }
  if (!p->loopback) {
    ncclUniqueId id;
    std::memcpy(&id, nccl_unique_id, sizeof id);
    ncclResult_t r = ncclCommInitRank(&p->comm, nranks, id, rank);
    if (r != ncclSuccess) { nccl_fail(r, "ncclCommInitRank"); p->comm = nullptr; free_plan(p); return nullptr; }
    cudaError_t e = cudaStreamCreateWithFlags(&p->comm_stream, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->ev_ready, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->ev_xchg, cudaEventDisableTiming);
    if (e != cudaSuccess) { cuda_fail(e, "comm stream/events"); free_plan(p); return nullptr; }
  }
  clear_error();
  return p;
}

int fftstencil_nccl_unique_id(void* out) {
  if (!out) { set_error("out must be non-NULL"); return FFTSTENCIL_EINVAL; }
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(out, &id, sizeof id);
  clear_error();
  return FFTSTENCIL_OK;
}

fftstencil_plan* fftstencil_plan_create_dist_peer(int ndim, const int64_t* extents, const double* weights, int radius,
                                                  int T, int nranks, int rank) {
  if (nranks < 2 || rank < 0 || rank >= nranks) { set_error("the peer transport needs nranks >= 2, 0 <= rank < nranks"); return nullptr; }
  if (!write_value_fn() || !wait_value_fn()) { set_error("stream memory operations unavailable"); return nullptr; }
  fftstencil_plan* p = new (std::nothrow) fftstencil_plan();
  if (!p) { set_error("host allocation failed"); return nullptr; }
  std::string err;
  int rc = build_host_plan(ndim, extents, weights, radius, T, p->hp, err, nranks, rank, env_algo());
  if (rc != FFTSTENCIL_OK) { set_error(err); delete p; return nullptr; }
  p->dist = true;
  p->peer = true;
  if (setup_device(p) != FFTSTENCIL_OK) { free_plan(p); return nullptr; }
  cudaError_t e = cudaMalloc((void**)&p->dFlags, 2 * sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaMemset(p->dFlags, 0, 2 * sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { cuda_fail(e, "peer flags"); free_plan(p); return nullptr; }
  clear_error();
  return p;
}

// Handle blob: IPC handles of dE[0], dE[1], dFlags (3 x 64 bytes), then int64 g0, row_lo, row_hi, rank.
int fftstencil_peer_handle(const fftstencil_plan* p, void* out, int64_t cap) {
  if (!p || !out || !p->peer) { set_error("a peer-transport plan and an output buffer are required"); return FFTSTENCIL_EINVAL; }
  if (cap < FFTSTENCIL_PEER_HANDLE_BYTES) { set_error("cap < FFTSTENCIL_PEER_HANDLE_BYTES"); return FFTSTENCIL_EINVAL; }
  unsigned char* o = static_cast<unsigned char*>(out);
  std::memset(o, 0, FFTSTENCIL_PEER_HANDLE_BYTES);
  cudaIpcMemHandle_t hd;
  void* ptrs[3] = {p->dE[0], p->dE[1], p->dFlags};
  for (int k = 0; k < 3; ++k) {
    cudaError_t e = cudaIpcGetMemHandle(&hd, ptrs[k]);
    if (e != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle");
    std::memcpy(o + 64 * k, &hd, sizeof hd);
  }
  const int64_t geo[4] = {p->hp.g0, p->hp.row_lo, p->hp.row_hi, p->hp.rank};
  std::memcpy(o + 192, geo, sizeof geo);
  clear_error();
  return FFTSTENCIL_OK;
}

int fftstencil_peer_connect(fftstencil_plan* p, const void* lower, const void* upper) {
  if (!p || !p->peer) { set_error("a peer-transport plan is required"); return FFTSTENCIL_EINVAL; }
  const HostPlan& hp = p->hp;
  if ((hp.rank > 0) != (lower != nullptr) || (hp.rank < hp.nranks - 1) != (upper != nullptr)) {
    set_error("pass exactly the existing neighbours' handles (lower for rank > 0, upper for rank < nranks - 1)");
    return FFTSTENCIL_EINVAL;
  }
  if (p->peer_connected) { set_error("already connected"); return FFTSTENCIL_EINVAL; }
  int cur = -1;
  cudaGetDevice(&cur);
  if (cur != p->device) cudaSetDevice(p->device);
  const void* hs[2] = {lower, upper};
  int rc = FFTSTENCIL_OK;
  for (int side = 0; side < 2 && rc == FFTSTENCIL_OK; ++side) {
    if (!hs[side]) continue;
    const unsigned char* h = static_cast<const unsigned char*>(hs[side]);
    int64_t geo[4];
    std::memcpy(geo, h + 192, sizeof geo);
    const int64_t want = side == 0 ? hp.rank - 1 : hp.rank + 1;
    // the lower neighbour's rows end where ours begin, the upper one's begin where ours end
    if (geo[3] != want || (side == 0 ? geo[2] != hp.row_lo : geo[1] != hp.row_hi)) {
      set_error("peer handle of the wrong rank or geometry");
      rc = FFTSTENCIL_EINVAL;
      break;
    }
    p->pG0[side] = geo[0];
    void* ptrs[3] = {nullptr, nullptr, nullptr};
    for (int k = 0; k < 3 && rc == FFTSTENCIL_OK; ++k) {
      cudaIpcMemHandle_t hd;
      std::memcpy(&hd, h + 64 * k, sizeof hd);
      cudaError_t e = cudaIpcOpenMemHandle(&ptrs[k], hd, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess) rc = cuda_fail(e, "cudaIpcOpenMemHandle");
    }
    p->pE[side][0] = static_cast<double*>(ptrs[0]);
    p->pE[side][1] = static_cast<double*>(ptrs[1]);
    p->pFlags[side] = static_cast<uint32_t*>(ptrs[2]);
  }
  if (rc == FFTSTENCIL_OK) {
    // probe both mechanisms now, so a missing peer path fails here (where callers can still agree
    // on another transport) and not in the middle of a run: an 8-byte copy into each neighbour's
    // first halo row (overwritten by the first push before any pass reads it) and a write of this
    // rank's current epoch into the flag word only this rank writes
    cudaStream_t ps = nullptr;
    cudaError_t e = cudaStreamCreateWithFlags(&ps, cudaStreamNonBlocking);
    for (int side = 0; side < 2 && e == cudaSuccess; ++side) {
      if (!hs[side]) continue;
      const int64_t row = side == 0 ? hp.row_lo : hp.row_hi - hp.h;   // its halo row this rank pushes first
      e = cudaMemcpyAsync(p->pE[side][0] + (size_t)(row - p->pG0[side]) * p->row_cells,
                          p->dE[0] + (size_t)(row - hp.g0) * p->row_cells, sizeof(double), cudaMemcpyDeviceToDevice, ps);
      if (e == cudaSuccess &&
          write_value_fn()((CUstream)ps, (CUdeviceptr)(p->pFlags[side] + (side == 0 ? 1 : 0)), p->epoch, 0) != CUDA_SUCCESS)
        e = cudaErrorNotSupported;
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(ps);
    if (ps) cudaStreamDestroy(ps);
    if (e != cudaSuccess) rc = cuda_fail(e, "peer transport probe (copy / stream write into a neighbour's memory)");
  }
  if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
  if (rc == FFTSTENCIL_OK) {
    p->peer_connected = true;
    clear_error();
  }
  return rc;
}

int fftstencil_run(fftstencil_plan* p, const double* in, double* out, int64_t total_steps, void* stream) {
  if (!p || !in || !out) { set_error("plan, in and out must be non-NULL"); return FFTSTENCIL_EINVAL; }
  if (total_steps < 0) { set_error("total_steps must be >= 0"); return FFTSTENCIL_EINVAL; }
  cudaStream_t s = (cudaStream_t)stream;
  p->last_launches = 0;
  int cur = -1;
  cudaGetDevice(&cur);
  if (cur != p->device) cudaSetDevice(p->device);
  const int rc = p->dist ? run_dist(p, in, out, total_steps, s) : run_single(p, in, out, total_steps, s);
  if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
  if (rc == FFTSTENCIL_OK) clear_error();
  return rc;
}

int fftstencil_run_group(fftstencil_plan* const* plans, const double* const* in, double* const* out, int nranks,
                         int64_t total_steps, void* stream) {
  if (!plans || !in || !out || nranks < 1) { set_error("invalid group arguments"); return FFTSTENCIL_EINVAL; }
  if (total_steps < 0) { set_error("total_steps must be >= 0"); return FFTSTENCIL_EINVAL; }
  for (int k = 0; k < nranks; ++k) {
    const fftstencil_plan* p = plans[k];
    if (!p || !in[k] || !out[k] || !p->dist || !p->loopback || p->hp.nranks != nranks || p->hp.rank != k ||
        p->hp.T != plans[0]->hp.T || p->device != plans[0]->device) {
      set_error("plans must be loopback ranks 0..nranks-1 of one decomposition on one device");
      return FFTSTENCIL_EINVAL;
    }
  }
  cudaStream_t s = (cudaStream_t)stream;
  int rc = FFTSTENCIL_OK;
  for (int k = 0; k < nranks; ++k) plans[k]->last_launches = 0;
  if (total_steps == 0) {
    for (int k = 0; k < nranks && !rc; ++k)
      if (in[k] != out[k]) {
        cudaError_t e = cudaMemcpyAsync(out[k], in[k], plans[k]->grid_cells * sizeof(double),
                                        cudaMemcpyDeviceToDevice, s);
        if (e != cudaSuccess) rc = cuda_fail(e, "copy");
      }
    return rc;
  }
  for (int k = 0; k < nranks && !rc; ++k) rc = dist_begin(plans[k], in[k], s);
  const int T = plans[0]->hp.T;
  const int64_t nfull = total_steps / T;
  const int rem = (int)(total_steps % T);
  for (int64_t i = 0; i < nfull + (rem ? 1 : 0) && !rc; ++i) {
    // loopback halo exchange: neighbours' owned boundary rows -> this rank's halo rows
    for (int k = 0; k < nranks && !rc; ++k) {
      fftstencil_plan* p = plans[k];
      const HostPlan& hp = p->hp;
      double* buf = p->dE[p->ecur];
      const size_t rcs = p->row_cells * sizeof(double);
      cudaError_t e = cudaSuccess;
      if (k > 0) {
        const fftstencil_plan* q = plans[k - 1];
        const double* src = q->dE[q->ecur] + (size_t)(q->hp.row_hi - hp.h - q->hp.g0) * q->row_cells;
        e = cudaMemcpyAsync(buf, src, (size_t)(hp.row_lo - hp.g0) * rcs, cudaMemcpyDeviceToDevice, s);
      }
      if (e == cudaSuccess && k < nranks - 1) {
        const fftstencil_plan* q = plans[k + 1];
        const double* src = q->dE[q->ecur] + (size_t)(q->hp.row_lo - q->hp.g0) * q->row_cells;
        e = cudaMemcpyAsync(buf + (size_t)(hp.row_hi - hp.g0) * p->row_cells, src, (size_t)(hp.g1 - hp.row_hi) * rcs,
                            cudaMemcpyDeviceToDevice, s);
      }
      if (e != cudaSuccess) rc = cuda_fail(e, "loopback halo copy");
    }
    for (int k = 0; k < nranks && !rc; ++k) rc = dist_pass(plans[k], i < nfull ? T : rem, false, s);
  }
  for (int k = 0; k < nranks && !rc; ++k) rc = dist_end(plans[k], out[k], s);
  if (rc == FFTSTENCIL_OK) clear_error();
  return rc;
}

int fftstencil_run_emit(fftstencil_plan* p, const double* in, const int64_t* emit_steps, int n_emit,
                        double* const* outs, void* stream) {
  if (!p || !in || !emit_steps || !outs || n_emit < 1) { set_error("invalid emit arguments"); return FFTSTENCIL_EINVAL; }
  int64_t prev = 0;
  for (int k = 0; k < n_emit; ++k) {
    if (emit_steps[k] < prev || !outs[k]) { set_error("emit steps must be non-decreasing, outs non-NULL"); return FFTSTENCIL_EINVAL; }
    prev = emit_steps[k];
  }
  // each segment is an ordinary run from the previous output (the semigroup property)
  const double* src = in;
  int64_t done = 0, launches = 0;
  for (int k = 0; k < n_emit; ++k) {
    const int rc = fftstencil_run(p, src, outs[k], emit_steps[k] - done, stream);
    if (rc != FFTSTENCIL_OK) return rc;
    launches += p->last_launches;
    src = outs[k];
    done = emit_steps[k];
  }
  p->last_launches = launches;
  return FFTSTENCIL_OK;
}

// ---------------------------------------------------------------- pipelined run_host
// The host->device copy of the input and the device->host copy of the result take ~30% of a
// Heat-2D run_host call (2 x 839 MB over PCIe).  They overlap the passes here by
// skewing the passes over outer tile rows ("units", the Eq. 3 tiles of one outer index):
// pass k may produce unit u once pass k-1 holds units u-1..u+1 (a unit reads rows
// [uS, uS+L) = its own output rows +- h, and h <= S), which is also the ping-pong
// anti-dependency (pass k+1 overwrites pass k-1's buffer only where pass k is done with it).
// Keeping f[k] (units of pass k produced, from the top) <= f[k-1] - 1 therefore makes any issue
// order on one stream correct.  Head: the input arrives in K row chunks; after each chunk the
// first Q passes advance.  Tail: the last Q passes advance in K steps whose pass-P frontier
// reaches chunk j's last unit, and chunk j of the result is copied out while the next advances.
// Band (boundary-strip) cells go with the unit whose row range R(u) holds them, the fixed
// ring with the input chunk.  Same kernels, same per-cell arithmetic: bitwise equal to
// fftstencil_run (tests/test_gpu_e2e_pipe.py).
static int copy_ring_rows(fftstencil_plan* p, const double* src, double* d0, double* d1, int64_t y0, int64_t y1,
                          cudaStream_t s) {
  const int oax = 3 - p->hp.ndim;
  for (const Box& b : p->hp.ring_boxes) {
    BoxCopyArgs a;
    a.src = src;
    a.dst0 = d0;
    a.dst1 = d1;
    for (int q = 0; q < 3; ++q) { a.n[q] = p->hp.n[q]; a.lo[q] = b.lo[q]; a.hi[q] = b.hi[q]; }
    a.lo[oax] = std::max<int64_t>(a.lo[oax], y0);
    a.hi[oax] = std::min<int64_t>(a.hi[oax], y1);
    if (a.hi[oax] <= a.lo[oax]) continue;
    a.oax = oax;
    a.src_off = 0;
    a.dst_off = 0;
    cudaError_t e = launch_box_copy(a, s);
    if (e != cudaSuccess) return cuda_fail(e, "ring copy launch");
    ++p->last_launches;
  }
  return FFTSTENCIL_OK;
}


// K, Q of the pipelined schedule; K = 0: disabled (the caller runs H2D, fftstencil_run, D2H).
// Default K: one input chunk per ~700 MB, 6..12 chunks -- the first H2D chunk and the last D2H
// chunk cannot overlap anything, so big grids want more chunks, but every chunk adds partial
// launches (measured: Heat-2D 839 MB K = 6 / 12 -> 90.4 / 93.5 ms per e2e step; Heat-3D 8.6 GB
// K = 6 / 12 / 24 -> 586 / 569 / 575 ms, profiles/r02_e2e_chunks.txt).
static int pipe_chunks(const fftstencil_plan* p) {
  const double gb = (double)p->grid_cells * sizeof(double) / 7e8;
  const int dflt = (int)std::min(12.0, std::max(6.0, std::floor(gb + 0.5)));
  const int K = env_int("FFTSTENCIL_E2E_PIPE", dflt);   // 0 disables; else the number of row chunks
  return p->dist || p->small1d ? 0 : K;
}

// Default Q: enough skewed passes at each end to cover one direction's copies (~49 GB/s each way
// concurrently, measured): Heat-2D 10240^2 Q = 16 (sweep: 16 best, 20 -1 %, 12 -5 %), 3D 1024^3
// Q = 20 (8.6 GB = 176 ms per direction vs 8.9 ms per pass: Q = 16 / 20 / 24 -> 530 / 514 / 516 ms
// per e2e step, profiles/r02_e2e3d.txt).
static int pipe_depth(const fftstencil_plan* p) {
  return std::max(1, env_int("FFTSTENCIL_E2E_DEPTH", p->hp.ndim == 3 ? 20 : 16));
}

static int run_host_pipelined_ops(fftstencil_plan* p, const double* h_in, double* h_out,
                                  const std::vector<int64_t>& ops, int64_t total_steps, cudaStream_t caller,
                                  cudaStream_t& s);

// On every exit, error or not, the copy stream and the pipeline stream are joined back into
// the caller's stream, so the caller's synchronize covers every queued chunk copy: a caller
// that frees its host buffers after an error cannot race a pending H2D / D2H.
static int run_host_pipelined(fftstencil_plan* p, const double* h_in, double* h_out,
                              const std::vector<int64_t>& ops, int64_t total_steps, cudaStream_t caller) {
  cudaStream_t s = caller;
  const bool conc = p->band_concurrent;
  p->band_concurrent = conc || p->band_e2e_concurrent;
  const int rc = run_host_pipelined_ops(p, h_in, h_out, ops, total_steps, caller, s);
  p->band_concurrent = conc;
  if (rc != FFTSTENCIL_OK) {
    const std::string err = g_last_error;
    cudaEvent_t ev;
    if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) == cudaSuccess) {
      for (cudaStream_t x : {p->copy_stream, s, p->band_stream}) {
        if (!x || x == caller) continue;
        if (cudaEventRecord(ev, x) == cudaSuccess) cudaStreamWaitEvent(caller, ev, 0);
      }
      cudaEventDestroy(ev);
    }
    p->band_pending = false;
    p->grid_cap = 0;
    p->band_clip_lo = 0;
    p->band_clip_hi = INT64_MAX;
    cudaGetLastError();
    set_error(err);
  }
  return rc;
}

static int run_host_pipelined_ops(fftstencil_plan* p, const double* h_in, double* h_out,
                                  const std::vector<int64_t>& ops, int64_t total_steps, cudaStream_t caller,
                                  cudaStream_t& s) {
  const HostPlan& hp = p->hp;
  const int64_t U = hp.nt[0], n0 = hp.ext[0], S = hp.S[0], h = hp.h, ppu = hp.pairs_per_unit;
  const size_t rcells = p->row_cells;
  const int T = hp.T;
  const int64_t nfull = total_steps / T;
  const int rem = (int)(total_steps % T);
  const int64_t P = nfull + (rem ? 1 : 0);
  double* in = p->dHostIn;
  double* out = p->dHostOut;
  double* dsts[2] = {(P % 2) ? out : p->dScratch, (P % 2) ? p->dScratch : out};
  auto row_of = [&](int64_t u) -> int64_t { return u <= 0 ? 0 : u >= U ? n0 : u * S + h; };
  cudaError_t e = cudaSuccess;
  if (!p->copy_stream && (e = cudaStreamCreateWithFlags(&p->copy_stream, cudaStreamNonBlocking)) != cudaSuccess)
    return cuda_fail(e, "copy stream");
  // The schedule runs on an internal greatest-priority stream: when an item's fused kernel and
  // its band kernel (band stream, default priority) are both pending, the block scheduler places
  // the fused CTAs first, so they take all but the reserved SMs and the band lands on those
  // (placed first, the band's CTAs spread one per SM and hold back as many fused CTAs for their
  // whole ~45 us latency: measured ~40 us per item).  FFTSTENCIL_E2E_PRIO=0 uses the caller's.
  s = caller;
  if (env_int("FFTSTENCIL_E2E_PRIO", 1)) {
    if (!p->pipe_stream) {
      int least = 0, greatest = 0;
      cudaDeviceGetStreamPriorityRange(&least, &greatest);
      if ((e = cudaStreamCreateWithPriority(&p->pipe_stream, cudaStreamNonBlocking, greatest)) != cudaSuccess)
        return cuda_fail(e, "pipeline stream");
    }
    s = p->pipe_stream;
  }
  size_t nev = 4;
  for (size_t i = 0; i < ops.size(); i += 4) nev += ops[i] == 0 || ops[i] == 3;
  while (p->ev_copy.size() < nev) {
    cudaEvent_t ev;
    if ((e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) != cudaSuccess) return cuda_fail(e, "copy event");
    p->ev_copy.push_back(ev);
  }
  size_t evi = 0;
  auto hand = [&](cudaStream_t from, cudaStream_t to) -> cudaError_t {
    cudaEvent_t ev = p->ev_copy[evi++];
    cudaError_t r = cudaEventRecord(ev, from);
    return r == cudaSuccess ? cudaStreamWaitEvent(to, ev, 0) : r;
  };
  const int occ = std::max(1, p->fused_grid / std::max(1, p->sm_count));
  const int reserve = std::max(0, env_int("FFTSTENCIL_E2E_BAND_SMS", 4));
  const int grid_cap = std::max(1, p->fused_grid - reserve * occ);
  auto item = [&](int64_t k, int64_t a, int64_t b) -> int {
    const int t = k <= nfull ? T : rem;
    const double* src = k == 1 ? in : dsts[(k - 2) % 2];
    double* dst = dsts[(k - 1) % 2];

    // fork the band first (it needs only what `s` holds so far), launch the fused tiles on all
    // but `reserve` SMs, then the band: its latency-bound CTAs (t sequential steps) run beside
    // the fused CTAs on the reserved SMs instead of after them
    if (p->band_concurrent) {
      cudaError_t e2 = cudaEventRecord(p->ev_fork, s);
      if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(p->band_stream, p->ev_fork, 0);
      if (e2 != cudaSuccess) return cuda_fail(e2, "band fork");
    }
    p->grid_cap = p->band_concurrent && b - a < U ? grid_cap : 0;   // whole passes: every SM
    int rc = launch_fused(p, src, dst, t, a * ppu, b * ppu, s);
    p->grid_cap = 0;
    if (rc) return rc;
    p->band_clip_lo = row_of(a);
    p->band_clip_hi = row_of(b);
    rc = launch_band_pass(p, src, dst, t, s, p->band_concurrent);
    p->band_clip_lo = 0;
    p->band_clip_hi = INT64_MAX;
    if (rc) return rc;
    return band_join(p, s);
  };
  if (s != caller && (e = hand(caller, s)) != cudaSuccess) return cuda_fail(e, "pipeline fork");
  if ((e = hand(s, p->copy_stream)) != cudaSuccess) return cuda_fail(e, "copy fork");
  int rc = FFTSTENCIL_OK;
  for (size_t i = 0; i < ops.size(); i += 4) {
    const int64_t op = ops[i], x = ops[i + 1], y = ops[i + 2], z = ops[i + 3];
    const size_t off = (size_t)x * rcells, bytes = (size_t)(y - x) * rcells * sizeof(double);
    if (op == 0) {          // input rows [x, y) -> device; the run stream waits for them
      if ((e = cudaMemcpyAsync(in + off, h_in + off, bytes, cudaMemcpyHostToDevice, p->copy_stream)) != cudaSuccess)
        return cuda_fail(e, "H2D chunk");
      if ((e = hand(p->copy_stream, s)) != cudaSuccess) return cuda_fail(e, "H2D join");
    } else if (op == 1) {   // fixed ring rows [x, y) into both pass buffers
      if ((rc = copy_ring_rows(p, in, out, P > 1 ? p->dScratch : nullptr, x, y, s))) return rc;
    } else if (op == 2) {   // pass x on units [y, z)
      if ((rc = item(x, y, z))) return rc;
    } else {                // result rows [x, y) -> host after everything issued so far
      if ((e = hand(s, p->copy_stream)) != cudaSuccess) return cuda_fail(e, "D2H fork");
      if ((e = cudaMemcpyAsync(h_out + off, out + off, bytes, cudaMemcpyDeviceToHost, p->copy_stream)) != cudaSuccess)
        return cuda_fail(e, "D2H chunk");
    }
  }
  if ((e = hand(p->copy_stream, s)) != cudaSuccess) return cuda_fail(e, "D2H join");
  if (s != caller && (e = hand(s, caller)) != cudaSuccess) return cuda_fail(e, "pipeline join");
  return FFTSTENCIL_OK;
}

int fftstencil_run_host(fftstencil_plan* p, const double* h_in, double* h_out, int64_t total_steps, void* stream) {
  if (!p || !h_in || !h_out) { set_error("plan, h_in and h_out must be non-NULL"); return FFTSTENCIL_EINVAL; }
  cudaStream_t s = (cudaStream_t)stream;
  const size_t bytes = p->grid_cells * sizeof(double);
  int cur = -1;
  cudaGetDevice(&cur);
  if (cur != p->device) cudaSetDevice(p->device);
  cudaError_t e = cudaSuccess;
  if (!p->dHostIn) {
    if ((e = cudaMalloc((void**)&p->dHostIn, bytes)) != cudaSuccess ||
        (e = cudaMalloc((void**)&p->dHostOut, bytes)) != cudaSuccess) {
      if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
      return cuda_fail(e, "run_host staging allocation");
    }
    p->device_bytes += 2 * bytes;
  }
  int rc = FFTSTENCIL_OK;
  const int K = pipe_chunks(p);
  std::vector<int64_t> ops;
  p->last_pipelined = false;
  if (K && build_e2e_schedule(p->hp, total_steps, K, pipe_depth(p), ops, pipe_tail_depth(), pipe_ramp()) == FFTSTENCIL_OK) {
    p->last_launches = 0;
    p->last_pipelined = true;
    p->last_chunks = K;
    p->last_depth = pipe_depth(p);
    rc = run_host_pipelined(p, h_in, h_out, ops, total_steps, (cudaStream_t)stream);
    // synchronise on success and on error (queued chunk copies still read / write the host buffers)
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess && rc == FFTSTENCIL_OK) rc = cuda_fail(e, "stream synchronize");
  } else if ((e = cudaMemcpyAsync(p->dHostIn, h_in, bytes, cudaMemcpyHostToDevice, s)) != cudaSuccess) {
    rc = cuda_fail(e, "H2D copy");
  } else {
    if ((rc = fftstencil_run(p, p->dHostIn, p->dHostOut, total_steps, stream)) == FFTSTENCIL_OK &&
        (e = cudaMemcpyAsync(h_out, p->dHostOut, bytes, cudaMemcpyDeviceToHost, s)) != cudaSuccess)
      rc = cuda_fail(e, "D2H copy");
    // the H2D read of h_in may still be queued when the run fails: synchronise either way
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess && rc == FFTSTENCIL_OK) rc = cuda_fail(e, "stream synchronize");
  }
  if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
  if (rc == FFTSTENCIL_OK) clear_error();
  return rc;
}

void fftstencil_destroy(fftstencil_plan* p) { free_plan(p); }

int fftstencil_plan_info(const fftstencil_plan* p, fftstencil_info* info) {
  if (!p || !info) { set_error("plan and info must be non-NULL"); return FFTSTENCIL_EINVAL; }
  fill_info(p->hp, info);
  info->device_bytes = p->device_bytes;
  info->fused_grid = p->fused_grid;
  info->last_run_launches = p->last_launches;
  info->last_run_pipelined = p->last_pipelined ? 1 : 0;
  info->last_run_chunks = p->last_pipelined ? p->last_chunks : 0;
  info->last_run_depth = p->last_pipelined ? p->last_depth : 0;
  info->last_run_peer_fused = p->last_peer_fused ? 1 : 0;
  clear_error();
  return FFTSTENCIL_OK;
}

int fftstencil_set_profiling(fftstencil_plan* p, int enable) {
  if (!p) { set_error("plan must be non-NULL"); return FFTSTENCIL_EINVAL; }
  p->profiling = enable != 0;
  p->ev_used = 0;
  clear_error();
  return FFTSTENCIL_OK;
}

int fftstencil_profile_read(fftstencil_plan* p, double* fused_ms, int64_t* fused_launches, double* band_ms,
                            int64_t* band_launches) {
  if (!p) { set_error("plan must be non-NULL"); return FFTSTENCIL_EINVAL; }
  double ms[2] = {0.0, 0.0};
  int64_t cnt[2] = {0, 0};
  for (size_t i = 0; i < p->ev_used; i += 2) {
    cudaError_t e = cudaEventSynchronize(p->ev_pool[i + 1]);
    if (e != cudaSuccess) return cuda_fail(e, "profiling event");
    float v = 0.f;
    e = cudaEventElapsedTime(&v, p->ev_pool[i], p->ev_pool[i + 1]);
    if (e != cudaSuccess) return cuda_fail(e, "profiling elapsed time");
    const int k = p->ev_kind[i / 2];
    ms[k] += v;
    cnt[k] += 1;
  }
  p->ev_used = 0;
  if (fused_ms) *fused_ms = ms[0];
  if (fused_launches) *fused_launches = cnt[0];
  if (band_ms) *band_ms = ms[1];
  if (band_launches) *band_launches = cnt[1];
  clear_error();
  return FFTSTENCIL_OK;
}

}  // extern "C"
