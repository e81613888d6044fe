// NEXT-4 microbenchmark: one length-16 DFT stage over many
// lines, evaluated (a) as the radix-4 butterfly FFT-16 on the FP64 ALU that the default 3D
// kernel uses (fft_radix.cuh), and (b) as an Ozaki-scheme emulated-FP64 GEMM on the INT8
// tensor cores (tcgen05.mma kind::i8, int32 accumulators in tensor memory), split and
// recombination included, on the same data, each checked against an FP64 direct DFT.
//
// Ozaki scheme (error-free slicing): per line, x = 2^(e+1) sum_i a_i 2^(-7(i+1)) with int8
// slices a_i (|a_i| <= 64, e = the line's exponent); the DFT matrix in real form
// G = [[Fr, -Fi], [Fi, Fr]] / 2 likewise (b_j, exponent 0).  Then y = G' x is
// 2^(e+2) sum_d 2^(-7(d+2)) Q_d with Q_d = sum_{i+j=d} A_i B_j^T (int8 x int8 -> int32, exact),
// d = 0..S-1 (terms i + j >= S dropped: relative error ~2^(-7S)).  One 128-line tile is one
// M = 128, N = 32, K = 32 MMA per slice pair: S(S+1)/2 = 15 MMAs for S = 5.
//
// The point: the slicing and the recombination are FP64 ALU work --
// per line 32 values x S slices x (scale, round, subtract) and 32 outputs x S diagonals x
// (convert, FMA) -- several times the 160 FP64 instructions of the butterfly FFT-16, on the
// very pipe the butterfly is bound by.  The tensor-core part is cheap; the emulation is not.
//
// Build / run (tools/r02_ozaki.sh):
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo \
//        -I paper_conf_ppopp_hanlcbzyczcy25_b200/csrc tools/ozaki_dft16.cu -o /tmp/ozaki_dft16
#include <cuda_runtime.h>

#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "fft_radix.cuh"

#define CK(x)                                                                         \
  do {                                                                                \
    cudaError_t e_ = (x);                                                             \
    if (e_ != cudaSuccess) {                                                          \
      std::fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
      std::exit(1);                                                                   \
    }                                                                                 \
  } while (0)

constexpr int NS = 5;       // slices per operand
constexpr int TM = 128;     // lines per tile (MMA M)
constexpr int KW = 32;      // real width of a complex 16-point line (MMA K and N)

// ---------------------------------------------------------------- (a) butterfly FFT-16
// Structure-of-arrays data: value k (re 0..15, im 16..31) of line l at x[k * n + l].
// R stages per load, alternating forward and (1/16-scaled) inverse DFT-16: R = 1 is one
// HBM-bound transform, large even R makes the data round trip negligible (the fused kernels
// keep tiles on chip) and y returns to x.
__global__ void __launch_bounds__(256) bf_kernel(const double* __restrict__ x, double* __restrict__ y, int n, int R) {
  for (int l = blockIdx.x * blockDim.x + threadIdx.x; l < n; l += gridDim.x * blockDim.x) {
    double xr[16], xi[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      xr[k] = x[(size_t)k * n + l];
      xi[k] = x[(size_t)(16 + k) * n + l];
    }
#pragma unroll 1
    for (int r = 0; r < R; ++r) {
      if (r & 1) {
        fstencil::radix::fft16<true>(xr, xi);
#pragma unroll
        for (int k = 0; k < 16; ++k) {
          xr[k] *= 0.0625;
          xi[k] *= 0.0625;
        }
      } else {
        fstencil::radix::fft16<false>(xr, xi);
      }
    }
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      y[(size_t)k * n + l] = xr[k];
      y[(size_t)(16 + k) * n + l] = xi[k];
    }
  }
}

// ---------------------------------------------------------------- (b) Ozaki on tcgen05 kind::i8
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// K-major, no-swizzle canonical layout (cute UMMA INTERLEAVE): element (row, k) of a slice at
// byte (row / 8) * 256 + (k / 16) * 128 + (row % 8) * 16 + (k % 16): core matrices of 8 rows x
// 16 bytes, LBO = 128 B between the two K halves, SBO = 256 B between 8-row groups.
__device__ __forceinline__ uint64_t smem_desc(uint32_t addr) {
  uint64_t d = 0;
  d |= (uint64_t)((addr >> 4) & 0x3FFF);          // start address
  d |= (uint64_t)(128 >> 4) << 16;                // leading (K) byte offset
  d |= (uint64_t)(256 >> 4) << 32;                // stride (M/N) byte offset
  d |= (uint64_t)1 << 46;                         // version (sm_100)
  return d;                                       // base offset 0, layout SWIZZLE_NONE (0)
}
// kind::i8 instruction descriptor: D s32, A / B signed int8, K-major both, N = 32, M = 128.
constexpr uint32_t kIdesc = (2u << 4) | (1u << 7) | (1u << 10) | ((32u >> 3) << 17) | ((128u >> 4) << 24);

__device__ __forceinline__ void mma_i8(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, {%5, %6, %7, %8}, p;\n\t}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(kIdesc), "r"(acc), "r"(0u), "r"(0u), "r"(0u), "r"(0u));
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, int32_t (&v)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
        "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]),
        "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]),
        "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
          smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// mode bits: 1 = slice the data (else reuse the slices in shared memory), 2 = tensor-core MMAs,
// 4 = recombine and store.  mode 7 is the full emulated DFT; the others time its parts.
__global__ void __launch_bounds__(TM, 1)
    ozaki_kernel(const double* __restrict__ x, double* __restrict__ y, int n, const int8_t* __restrict__ gsl, int mode,
                 int R) {
  __shared__ __align__(1024) int8_t sA[NS][TM * KW];      // data slices, canonical layout
  __shared__ __align__(1024) int8_t sB[2][NS][KW * KW];   // DFT-matrix slices: forward, inverse
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t tmem_base;
  const int tid = threadIdx.x, warp = tid >> 5;
  // DFT-matrix slices (row n, column k) into the canonical layout
  for (int e = tid; e < 2 * NS * KW * KW; e += TM) {
    const int d = e / (NS * KW * KW), s = (e / (KW * KW)) % NS, r = (e / KW) % KW, k = e % KW;
    sB[d][s][(r / 8) * 256 + (k / 16) * 128 + (r % 8) * 16 + (k % 16)] = gsl[e];
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;\n" ::"r"(smem_u32(&tmem_base)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;\n");
  const uint32_t tmem = tmem_base;
  uint32_t phase = 0;
  const int ntiles = n / TM;
  for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const int l = t * TM + tid;
    double v[KW];
#pragma unroll
    for (int k = 0; k < KW; ++k) v[k] = x[(size_t)k * n + l];
#pragma unroll 1
    for (int rs = 0; rs < R; ++rs) {
      // ---- split: 32 FP64 values -> NS int8 slices (exact remainders) ----
      double m = 0.0;
#pragma unroll
      for (int k = 0; k < KW; ++k) m = fmax(m, fabs(v[k]));
      int e = 0;
      if (m > 0.0) frexp(m, &e);          // m < 2^e
      const double scale = ldexp(1.0, e + 1) * ((rs & 1) ? 0.0625 : 1.0);   // inverse stages: 1/16
      const double inv = ldexp(1.0, -(e + 1));
      if (mode & 1) {
        double w8[KW];
#pragma unroll
        for (int k = 0; k < KW; ++k) w8[k] = v[k] * inv;
#pragma unroll
        for (int s = 0; s < NS; ++s) {
          uint32_t w[8];
#pragma unroll
          for (int q = 0; q < 8; ++q) {
            uint32_t packed = 0;
#pragma unroll
            for (int b = 0; b < 4; ++b) {
              // round to nearest with the 1.5 * 2^52 magic number (two adds, no conversion
              // instruction); the low byte of the biased sum is the two's-complement int8
              const int k = 4 * q + b;
              const double tt = w8[k] * 128.0;         // exact
              const double big = tt + 6755399441055744.0;
              const double r = big - 6755399441055744.0;   // rint(tt), |r| <= 64
              w8[k] = tt - r;                          // exact, |w8| <= 1/2
              packed |= ((uint32_t)__double2loint(big) & 0xFFu) << (8 * b);
            }
            w[q] = packed;
          }
          int8_t* row = &sA[s][(tid / 8) * 256 + (tid % 8) * 16];
          *reinterpret_cast<uint4*>(row) = make_uint4(w[0], w[1], w[2], w[3]);
          *reinterpret_cast<uint4*>(row + 128) = make_uint4(w[4], w[5], w[6], w[7]);
        }
      }
      asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");   // generic writes -> MMA (async proxy)
      __syncthreads();
      // ---- tensor cores: Q_d = sum_{i+j=d} A_i B_j^T into TMEM columns 32 d ----
      if (mode & 2) {
        if (tid == 0) {
          asm volatile("tcgen05.fence::after_thread_sync;\n");
          const int dir = rs & 1;
#pragma unroll
          for (int d = 0; d < NS; ++d)
#pragma unroll
            for (int i = 0; i <= d; ++i)
              mma_i8(tmem + 32 * d, smem_desc(smem_u32(sA[i])), smem_desc(smem_u32(sB[dir][d - i])), i > 0);
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                           smem_u32(&bar))
                       : "memory");
        }
        mbar_wait(&bar, phase);
        phase ^= 1;
        asm volatile("tcgen05.fence::after_thread_sync;\n");
      }
      // ---- recombine: v = 2^(e+2) sum_d 2^(-7(d+2)) Q_d ----
      if (mode & 4) {
        double acc[KW];
#pragma unroll
        for (int k = 0; k < KW; ++k) acc[k] = 0.0;
#pragma unroll
        for (int d = NS - 1; d >= 0; --d) {
          int32_t q[32];
          tmem_ld32(tmem + ((uint32_t)(32 * warp) << 16) + 32 * d, q);
          const double f = ldexp(1.0, -7 * (d + 2));
          // int32 -> double by the magic number (bias 2^31 into the low word of 1.5 * 2^52)
#pragma unroll
          for (int k = 0; k < KW; ++k)
            acc[k] = fma(__hiloint2double(0x43380000, q[k] ^ (int)0x80000000) - 6755401588539392.0, f, acc[k]);
        }
        const double sc = 2.0 * scale;
#pragma unroll
        for (int k = 0; k < KW; ++k) v[k] = acc[k] * sc;
      }
      asm volatile("tcgen05.fence::before_thread_sync;\n");
      __syncthreads();   // TMEM reads and slice reads done before the next stage's MMAs / splits
      asm volatile("tcgen05.fence::after_thread_sync;\n");
    }
#pragma unroll
    for (int k = 0; k < KW; ++k) y[(size_t)k * n + l] = v[k];
  }
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;\n" ::"r"(tmem));
}

// ---------------------------------------------------------------- host
static void slice_host(double v, int8_t* out) {   // |v| <= 1/2 -> NS slices
  for (int s = 0; s < NS; ++s) {
    const double t = v * 128.0, r = std::rint(t);
    out[s] = (int8_t)(int)r;
    v = t - r;
  }
}

int main(int argc, char** argv) {
  const int n = argc > 1 ? std::atoi(argv[1]) : 148 * 128 * 64;   // lines (multiple of 128)
  const int reps = 20;
  std::printf("lines %d (x 16 complex FP64), %d slices\n", n, NS);
  // DFT-16 in real form G[r][k] / 2: rows 0..15 real parts of the outputs, 16..31 imaginary
  // [direction][slice][row][k]; direction 1 = inverse (conjugate matrix, unscaled)
  std::vector<int8_t> gsl((size_t)2 * NS * KW * KW);
  for (int dir = 0; dir < 2; ++dir) {
    std::vector<double> G((size_t)KW * KW);
    for (int r = 0; r < 16; ++r)
      for (int k = 0; k < 16; ++k) {
        const double ang = (dir ? 2.0 : -2.0) * M_PI * ((r * k) % 16) / 16.0, c = std::cos(ang), s = std::sin(ang);
        G[r * KW + k] = c;            // Re y = Fr xr - Fi xi
        G[r * KW + 16 + k] = -s;
        G[(16 + r) * KW + k] = s;     // Im y = Fi xr + Fr xi
        G[(16 + r) * KW + 16 + k] = c;
      }
    for (int r = 0; r < KW; ++r)
      for (int k = 0; k < KW; ++k) {
        int8_t sl[NS];
        slice_host(G[r * KW + k] / 2.0, sl);
        for (int s = 0; s < NS; ++s) gsl[(((size_t)dir * NS + s) * KW + r) * KW + k] = sl[s];
      }
  }
  std::vector<double> hx((size_t)KW * n);
  uint64_t st = 0x9E3779B97F4A7C15ull;
  for (auto& v : hx) {   // U(-1, 1), seeded
    st = st * 6364136223846793005ull + 1442695040888963407ull;
    v = 2.0 * ((st >> 11) * (1.0 / 9007199254740992.0)) - 1.0;
  }
  double *dx, *dy;
  int8_t* dg;
  CK(cudaMalloc(&dx, hx.size() * 8));
  CK(cudaMalloc(&dy, hx.size() * 8));
  CK(cudaMalloc(&dg, gsl.size()));
  CK(cudaMemcpy(dx, hx.data(), hx.size() * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dg, gsl.data(), gsl.size(), cudaMemcpyHostToDevice));
  // reference: R = 1 -> the direct DFT (long double) on a sample of lines; R even -> x itself
  // (R / 2 forward + 1/16-scaled inverse round trips)
  auto check = [&](const char* name, int R) {
    std::vector<double> hy(hx.size());
    CK(cudaMemcpy(hy.data(), dy, hy.size() * 8, cudaMemcpyDeviceToHost));
    double err = 0, mx = 0;
    for (int l = 0; l < n; l += 97) {
      for (int r = 0; r < 16; ++r) {
        long double re = 0, im = 0;
        if (R == 1) {
          for (int k = 0; k < 16; ++k) {
            const long double ang = -2.0L * 3.14159265358979323846264338327950288L * ((r * k) % 16) / 16.0L;
            const long double c = cosl(ang), s = sinl(ang), a = hx[(size_t)k * n + l], b = hx[(size_t)(16 + k) * n + l];
            re += a * c - b * s;
            im += a * s + b * c;
          }
        } else {
          re = hx[(size_t)r * n + l];
          im = hx[(size_t)(16 + r) * n + l];
        }
        err = std::fmax(err, std::fabs((double)(hy[(size_t)r * n + l] - re)));
        err = std::fmax(err, std::fabs((double)(hy[(size_t)(16 + r) * n + l] - im)));
        mx = std::fmax(mx, (double)std::fabs(re));
      }
    }
    std::printf("  %-40s R=%-3d max abs err %.3e  (rel to max |y| %.3e)\n", name, R, err, err / mx);
    return err / mx;
  };
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  auto timeit = [&](auto&& launch) {
    launch();
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(e0));
    for (int i = 0; i < reps; ++i) launch();
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    CK(cudaGetLastError());
    return ms / reps;
  };
  const double bytes = 2.0 * KW * 8.0 * n;   // read + write every value once
  const char* names[8] = {"", "split only", "MMA only (slices reused)", "split + MMA", "recombine only",
                          "split + recombine (no MMA)", "MMA + recombine", "Ozaki full (split+MMA+recombine)"};
  for (int R : {1, 16}) {
    std::printf("-- %d DFT-16 stage(s) per line per load (%s)\n", R,
                R == 1 ? "one transform: HBM-bound" : "alternating forward / inverse: on-chip, compute-bound");
    const float t_bf = timeit([&] { bf_kernel<<<sms * 8, 256>>>(dx, dy, n, R); });
    const double e_bf = check("butterfly FFT-16 (FP64 ALU)", R);
    std::printf("  butterfly: %.3f ms  %.2f G line-stages/s  %.0f GB/s  %.2f T FP64-instr/s (160 per stage)\n", t_bf,
                (double)n * R / t_bf / 1e6, bytes / t_bf / 1e6, 160.0 * n * R / t_bf / 1e9);
    double e_oz = -1;
    for (int mode : {7, 2, 1, 5, 6}) {
      const float t = timeit([&] { ozaki_kernel<<<2 * sms, TM>>>(dx, dy, n, dg, mode, R); });
      if (mode == 7) e_oz = check(names[mode], R);
      std::printf("  ozaki %-36s %.3f ms  %.2f G line-stages/s  (%.2fx the butterfly time)\n", names[mode], t,
                  (double)n * R / t / 1e6, t / t_bf);
    }
    std::printf("RESULT R=%d butterfly_ms %.4f ozaki_ms_full see above butterfly_rel_err %.3e ozaki_rel_err %.3e "
                "(target 1e-9)\n", R, t_bf, e_bf, e_oz);
  }
  return 0;
}
