// C ABI (include/fftstencil.h): plan lifetime, device upload and the run driver.
//
// The run driver is the temporal loop of PAPER.md §4 (Eq. 10): floor(steps/T) fused
// passes with S_T, then one pass with S_T' (T' = steps mod T; reading Q15).  Each pass is
// one fused FFT-tile launch over the exact region plus one boundary-band launch, both
// reading `src` and writing disjoint cells of `dst`; buffers ping-pong between `out` and
// the plan's scratch grid so that the last pass lands in `out`.  The fixed ring is copied
// once per run into every buffer that is written.
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "fftstencil.h"
#include "kernels.cuh"
#include "plan.h"

using namespace fstencil;

namespace {

thread_local std::string g_last_error;

void set_error(const std::string& s) { g_last_error = s; }
void clear_error() { g_last_error.clear(); }

}  // namespace

struct fftstencil_plan {
  HostPlan hp;
  int device = 0;
  int sm_count = 0;
  double* dF = nullptr;       // Fre | Fim
  double* dS = nullptr;       // for t = 1..T: Sre | Sim, each vol
  int* dCrt = nullptr;
  double* dW = nullptr;
  int* dBlocks = nullptr;
  double* dScratch = nullptr;
  double* dHostIn = nullptr;  // run_host staging grids (lazy)
  double* dHostOut = nullptr;
  size_t spec_vol = 0;
  size_t grid_cells = 0;
  size_t device_bytes = 0;
  int fused_grid = 0;
  int variant = 0;            // fused-kernel variant (2D)
  size_t band_smem = 0;
  int64_t last_launches = 0;
  // profiling: event pairs (start, end, kind 0 = fused, 1 = band) recorded by run()
  bool profiling = false;
  std::vector<cudaEvent_t> ev_pool;
  std::vector<int> ev_kind;
  size_t ev_used = 0;
};

namespace {

int cuda_fail(cudaError_t e, const char* what) {
  char buf[256];
  std::snprintf(buf, sizeof buf, "%s: %s", what, cudaGetErrorString(e));
  set_error(buf);
  return FFTSTENCIL_ECUDA;
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
  for (cudaEvent_t ev : p->ev_pool) cudaEventDestroy(ev);
  cudaFree(p->dF);
  cudaFree(p->dS);
  cudaFree(p->dCrt);
  cudaFree(p->dW);
  cudaFree(p->dBlocks);
  cudaFree(p->dScratch);
  cudaFree(p->dHostIn);
  cudaFree(p->dHostOut);
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
  info->mma_flops_per_pass = hp.mma_flops_per_pair * (double)hp.pairs;
  info->smem_bytes = hp.fused_smem;
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

// One fused pass: src -> dst with t steps (t <= T), tile geometry of T.
int enqueue_pass(fftstencil_plan* p, const double* src, double* dst, int t, cudaStream_t s) {
  const HostPlan& hp = p->hp;
  const double* Sre = p->dS + (size_t)(t - 1) * 2 * p->spec_vol;
  const double* Sim = Sre + p->spec_vol;
  cudaError_t e = cudaSuccess;
  if (hp.ndim == 2) {
    Fft2dArgs a;
    a.src = src;
    a.dst = dst;
    a.n0 = hp.ext[0];
    a.n1 = hp.ext[1];
    a.h = hp.h;
    a.S = hp.S[0];
    a.nt1 = hp.nt[1];
    a.ntiles = hp.tiles;
    a.npairs = hp.pairs;
    a.Fre = p->dF;
    a.Fim = p->dF + (size_t)hp.L[0] * hp.L[0];
    a.Sre = Sre;
    a.Sim = Sim;
    const long pe = prof_begin(p, 0, s);
    e = launch_fused2d(hp.L[0], p->variant, a, p->fused_grid, s);
    prof_end(p, pe, s);
  } else if (hp.ndim == 1) {
    Fft1dArgs a;
    a.src = src;
    a.dst = dst;
    a.n = hp.ext[0];
    a.h = hp.h;
    a.S = hp.S[0];
    a.L = hp.L[0];
    a.ntiles = hp.tiles;
    a.npairs = hp.pairs;
    a.Fre = p->dF;
    a.Fim = p->dF + 128;
    a.Sre = Sre;
    a.Sim = Sim;
    a.crt = p->dCrt;
    const long pe = prof_begin(p, 0, s);
    e = launch_fused1d(a, p->fused_grid, s);
    prof_end(p, pe, s);
  } else {
    Fft3dArgs a;
    a.src = src;
    a.dst = dst;
    a.n0 = hp.ext[0];
    a.n1 = hp.ext[1];
    a.n2 = hp.ext[2];
    a.h = hp.h;
    a.S = hp.S[0];
    a.nt1 = hp.nt[1];
    a.nt2 = hp.nt[2];
    a.ntiles = hp.tiles;
    a.npairs = hp.pairs;
    a.Fre = p->dF;
    a.Fim = p->dF + (size_t)hp.L[0] * hp.L[0];
    a.Sre = Sre;
    a.Sim = Sim;
    const long pe = prof_begin(p, 0, s);
    e = launch_fused3d(a, p->fused_grid, s);
    prof_end(p, pe, s);
  }
  if (e != cudaSuccess) return cuda_fail(e, "fused FFT-tile launch");
  ++p->last_launches;
  const int nb = (int)(hp.band_blocks.size() / 8);
  if (nb > 0) {
    BandArgs b;
    b.src = src;
    b.dst = dst;
    for (int q = 0; q < 3; ++q) { b.n[q] = hp.n[q]; b.active[q] = q >= 3 - hp.ndim; }
    b.r = hp.radius;
    b.t = t;
    b.w = p->dW;
    b.blocks = p->dBlocks;
    b.nblocks = nb;
    const long pb = prof_begin(p, 1, s);
    e = launch_band(b, p->band_smem, s);
    prof_end(p, pb, s);
    if (e != cudaSuccess) return cuda_fail(e, "band launch");
    ++p->last_launches;
  }
  return FFTSTENCIL_OK;
}

int copy_ring(fftstencil_plan* p, const double* src, double* d0, double* d1, cudaStream_t s) {
  for (const Box& b : p->hp.ring_boxes) {
    BoxCopyArgs a;
    a.src = src;
    a.dst0 = d0;
    a.dst1 = d1;
    for (int q = 0; q < 3; ++q) { a.n[q] = p->hp.n[q]; a.lo[q] = b.lo[q]; a.hi[q] = b.hi[q]; }
    cudaError_t e = launch_box_copy(a, s);
    if (e != cudaSuccess) return cuda_fail(e, "ring copy launch");
    ++p->last_launches;
  }
  return FFTSTENCIL_OK;
}

}  // namespace

extern "C" {

const char* fftstencil_last_error(void) { return g_last_error.c_str(); }

int fftstencil_describe(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                        fftstencil_info* info) {
  if (!info) { set_error("info must be non-NULL"); return FFTSTENCIL_EINVAL; }
  HostPlan hp;
  std::string err;
  const int rc = build_host_plan(ndim, extents, weights, radius, T, hp, err);
  if (rc != FFTSTENCIL_OK) { set_error(err); return rc; }
  fill_info(hp, info);
  clear_error();
  return FFTSTENCIL_OK;
}

int64_t fftstencil_export_aux(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                              int which, int axis, int t, double* out, int64_t cap) {
  HostPlan hp;
  std::string err;
  const int rc = build_host_plan(ndim, extents, weights, radius, T, hp, err);
  if (rc != FFTSTENCIL_OK) { set_error(err); return rc; }
  std::vector<double> v;
  if (which == 0) {
    int L, row0 = 0, ld;
    if (hp.ndim == 1) {
      if (axis < 0 || axis > 1) { set_error("axis must be 0 (N1) or 1 (N2) for 1D"); return FFTSTENCIL_EINVAL; }
      L = axis == 0 ? hp.N1 : hp.N2;
      row0 = axis == 0 ? 0 : 8;
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
        const int64_t o = idx[a] * hp.S[a];
        const int64_t first = o + hp.h;
        const int64_t last = std::min<int64_t>(o + hp.h + hp.S[a], hp.ext[a] - hp.h);
        v.push_back((double)o);
        v.push_back((double)first);
        v.push_back((double)(last - first));
      }
    }
  } else if (which == 3) {
    if (hp.ndim != 1) { set_error("the PFA map exists for 1D plans only"); return FFTSTENCIL_EINVAL; }
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
  fftstencil_plan* p = new (std::nothrow) fftstencil_plan();
  if (!p) { set_error("host allocation failed"); return nullptr; }
  std::string err;
  int rc = build_host_plan(ndim, extents, weights, radius, T, p->hp, err);
  if (rc != FFTSTENCIL_OK) { set_error(err); delete p; return nullptr; }
  HostPlan& hp = p->hp;
  cudaError_t e = cudaGetDevice(&p->device);
  if (e != cudaSuccess) { cuda_fail(e, "cudaGetDevice"); delete p; return nullptr; }
  e = cudaDeviceGetAttribute(&p->sm_count, cudaDevAttrMultiProcessorCount, p->device);
  if (e != cudaSuccess) { cuda_fail(e, "cudaDeviceGetAttribute"); delete p; return nullptr; }

  size_t acc = 0;
  std::vector<double> F(hp.Fre);
  F.insert(F.end(), hp.Fim.begin(), hp.Fim.end());
  if (hp.ndim == 2) {
    // the 2D kernel reads F with columns permuted within groups of 8 (device_common.cuh)
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
  p->grid_cells = 1;
  for (int a = 0; a < hp.ndim; ++a) p->grid_cells *= (size_t)hp.ext[a];
  if ((e = upload(&p->dF, F.data(), F.size(), acc)) != cudaSuccess ||
      (e = upload(&p->dS, Sv.data(), Sv.size(), acc)) != cudaSuccess ||
      (e = upload(&p->dW, hp.w.data(), hp.w.size(), acc)) != cudaSuccess ||
      (e = upload(&p->dBlocks, hp.band_blocks.data(), hp.band_blocks.size(), acc)) != cudaSuccess ||
      (hp.ndim == 1 && (e = upload(&p->dCrt, hp.crt.data(), hp.crt.size(), acc)) != cudaSuccess)) {
    cuda_fail(e, "device upload");
    free_plan(p);
    return nullptr;
  }
  e = cudaMalloc((void**)&p->dScratch, p->grid_cells * sizeof(double));
  if (e != cudaSuccess) {
    set_error(std::string("scratch grid allocation: ") + cudaGetErrorString(e));
    free_plan(p);
    return nullptr;
  }
  acc += p->grid_cells * sizeof(double);
  p->device_bytes = acc;

  int occ = 0;
  if (hp.ndim == 2) {
    // double-buffered prefetch pays only where it does not cost occupancy (profiles/r01_variants.txt)
    p->variant = hp.L[0] >= 56 ? 1 : 0;
    if (const char* v = std::getenv("FFTSTENCIL_VARIANT")) p->variant = std::atoi(v);
    if (p->variant < 0 || p->variant > 2) { set_error("FFTSTENCIL_VARIANT must be 0, 1 or 2"); free_plan(p); return nullptr; }
    e = fused2d_configure(hp.L[0], p->variant, &occ);
    if (e != cudaSuccess) { cuda_fail(e, "fused 2D kernel configuration"); free_plan(p); return nullptr; }
    if (occ < 1) { set_error("fused 2D kernel cannot be resident"); free_plan(p); return nullptr; }
    const int64_t want = (int64_t)p->sm_count * occ;
    p->fused_grid = (int)std::max<int64_t>(1, std::min<int64_t>(want, hp.pairs));
  } else if (hp.ndim == 3) {
    e = fused3d_configure(&occ);
    if (e != cudaSuccess) { cuda_fail(e, "fused 3D kernel configuration"); free_plan(p); return nullptr; }
    if (occ < 1) { set_error("fused 3D kernel cannot be resident"); free_plan(p); return nullptr; }
    const int64_t want = (int64_t)p->sm_count * occ;
    p->fused_grid = (int)std::max<int64_t>(1, std::min<int64_t>(want, hp.pairs));
  } else {
    e = fused1d_configure(&occ);
    if (e != cudaSuccess || occ < 1) { cuda_fail(e, "fused 1D kernel configuration"); free_plan(p); return nullptr; }
    const int64_t blocks = (hp.pairs + kFft1dWarpsPerBlock - 1) / kFft1dWarpsPerBlock;
    p->fused_grid = (int)std::max<int64_t>(1, std::min<int64_t>(blocks, (int64_t)p->sm_count * occ));
  }
  p->band_smem = (size_t)2 * hp.band_region_cells * sizeof(double);
  if (p->band_smem > 0) {
    e = band_configure(p->band_smem);
    if (e != cudaSuccess) { cuda_fail(e, "band kernel configuration"); free_plan(p); return nullptr; }
  }
  clear_error();
  return p;
}

int fftstencil_run(fftstencil_plan* p, const double* in, double* out, int64_t total_steps, void* stream) {
  if (!p || !in || !out) { set_error("plan, in and out must be non-NULL"); return FFTSTENCIL_EINVAL; }
  if (total_steps < 0) { set_error("total_steps must be >= 0"); return FFTSTENCIL_EINVAL; }
  cudaStream_t s = (cudaStream_t)stream;
  const size_t bytes = p->grid_cells * sizeof(double);
  p->last_launches = 0;
  int cur = -1;
  cudaGetDevice(&cur);
  if (cur != p->device) cudaSetDevice(p->device);
  int rc = FFTSTENCIL_OK;
  do {
    if (total_steps == 0) {
      if (in != out) {
        cudaError_t e = cudaMemcpyAsync(out, in, bytes, cudaMemcpyDeviceToDevice, s);
        if (e != cudaSuccess) { rc = cuda_fail(e, "copy"); break; }
      }
      break;
    }
    const int T = p->hp.T;
    const int64_t nfull = total_steps / T;
    const int rem = (int)(total_steps % T);
    const int64_t passes = nfull + (rem ? 1 : 0);
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
    // fixed ring: copied once into every buffer that receives a pass
    rc = copy_ring(p, in, alias ? nullptr : out, passes > 1 || alias ? p->dScratch : nullptr, s);
    if (rc) break;
    const double* src = in;
    for (int64_t i = 0; i < passes; ++i) {
      const int t = i < nfull ? T : rem;
      double* dst = dsts[i % 2];
      rc = enqueue_pass(p, src, dst, t, s);
      if (rc) break;
      src = dst;
    }
    if (rc) break;
    if (final_copy) {
      cudaError_t e = cudaMemcpyAsync(out, p->dScratch, bytes, cudaMemcpyDeviceToDevice, s);
      if (e != cudaSuccess) { rc = cuda_fail(e, "final copy"); break; }
    }
  } while (0);
  if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
  if (rc == FFTSTENCIL_OK) clear_error();
  return rc;
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
  if ((e = cudaMemcpyAsync(p->dHostIn, h_in, bytes, cudaMemcpyHostToDevice, s)) != cudaSuccess) {
    rc = cuda_fail(e, "H2D copy");
  } else if ((rc = fftstencil_run(p, p->dHostIn, p->dHostOut, total_steps, stream)) == FFTSTENCIL_OK) {
    if ((e = cudaMemcpyAsync(h_out, p->dHostOut, bytes, cudaMemcpyDeviceToHost, s)) != cudaSuccess)
      rc = cuda_fail(e, "D2H copy");
    else if ((e = cudaStreamSynchronize(s)) != cudaSuccess)
      rc = cuda_fail(e, "stream synchronize");
  }
  if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
  if (rc == FFTSTENCIL_OK) clear_error();
  return rc;
}

void fftstencil_destroy(fftstencil_plan* p) { free_plan(p); }

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

int fftstencil_plan_info(const fftstencil_plan* p, fftstencil_info* info) {
  if (!p || !info) { set_error("plan and info must be non-NULL"); return FFTSTENCIL_EINVAL; }
  fill_info(p->hp, info);
  info->device_bytes = p->device_bytes;
  info->fused_grid = p->fused_grid;
  info->last_run_launches = p->last_launches;
  clear_error();
  return FFTSTENCIL_OK;
}

}  // extern "C"
