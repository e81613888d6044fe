// Microbenchmark: FP64 tensor (DMMA m8n8k4) and FP64 FMA (DFMA) peak on this GPU,
// plus a fragment-layout check of mma.m8n8k4.f64. Used to fix the roofline
// denominator for the FP64-bound fused FFT-stencil kernel.
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
               : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}

template <int CH>
__global__ void dmma_loop(double* out, int iters, double a0, double b0) {
  double c[CH][2];
#pragma unroll
  for (int i = 0; i < CH; ++i) { c[i][0] = 0; c[i][1] = 0; }
  double a = a0 * threadIdx.x, b = b0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) dmma(c[i][0], c[i][1], a, b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += c[i][0] + c[i][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int CH>
__global__ void dfma_loop(double* out, int iters, double a0, double b0) {
  double c[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) c[i] = threadIdx.x * 1e-3 + i;
  double a = a0, b = b0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) c[i] = fma(c[i], a, b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += c[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// Per-instruction FP64 rate of DADD / DMUL / an FFT-like mix (2 DADD : 1 DMUL : 1 DFMA): does
// every FP64 instruction take one pipe slot (the ALU roofline of bench.py assumes so)?
// OP 0 = DADD, 1 = DMUL, 2 = mix.  CH independent chains per thread.
template <int CH, int OP>
__global__ void op_loop(double* out, int iters, double a0, double b0) {
  double c[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) c[i] = threadIdx.x * 1e-3 + i;
  const double a = a0, b = b0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      if (OP == 0) c[i] = c[i] + b;
      else if (OP == 1) c[i] = c[i] * a;
      else {   // 4 instructions per chain step
        c[i] = __dadd_rn(c[i], b);   // _rn intrinsics: no FMA contraction
        c[i] = __dmul_rn(c[i], a);
        c[i] = __dsub_rn(c[i], b);
        c[i] = fma(c[i], a, b);
      }
    }
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += c[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// DMMA and DFMA interleaved in one warp stream (independent accumulators): tells whether
// the tensor DMMA path and the FP64 FMA units share throughput on this GPU.
template <int CH, int NF>
__global__ void mix_loop(double* out, int iters, double a0, double b0) {
  double c[CH][2], f[NF > 0 ? NF : 1];
#pragma unroll
  for (int i = 0; i < CH; ++i) { c[i][0] = 0; c[i][1] = 0; }
#pragma unroll
  for (int i = 0; i < NF; ++i) f[i] = threadIdx.x * 1e-3 + i;
  double a = a0 * threadIdx.x, b = b0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      dmma(c[i][0], c[i][1], a, b);
#pragma unroll
      for (int k = 0; k < NF / CH; ++k) f[i * (NF / CH) + k] = fma(f[i * (NF / CH) + k], a0, b0);
    }
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += c[i][0] + c[i][1];
#pragma unroll
  for (int i = 0; i < NF; ++i) s += f[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void layout_probe(double* A, double* B, double* C) {
  int lane = threadIdx.x;
  // A[8][4] row-major, B[4][8] row-major (k, n), fragment per documented layout
  double a = A[(lane >> 2) * 4 + (lane & 3)];
  double b = B[(lane & 3) * 8 + (lane >> 2)];
  double c0 = 0, c1 = 0;
  dmma(c0, c1, a, b);
  C[(lane >> 2) * 8 + (lane & 3) * 2 + 0] = c0;
  C[(lane >> 2) * 8 + (lane & 3) * 2 + 1] = c1;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("SMs %d clock(kHz) %d\n", sms, clk);
  double *out; cudaMalloc(&out, sizeof(double) * 148 * 64 * 1024);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int iters = 20000;
  for (int wpb : {4, 8, 16, 32}) {
    for (int rep = 0; rep < 2; ++rep) {
      int blocks = sms * 2;
      cudaEventRecord(e0);
      dmma_loop<8><<<blocks, wpb * 32>>>(out, iters, 1.0, 1e-9);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double flops = 2.0 * 256 * 8 * (double)iters * blocks * wpb;
      if (rep) printf("DMMA m8n8k4: warps/block %d blocks %d -> %.2f TFLOP/s (%.3f ms)\n", wpb, blocks, flops / ms / 1e9, ms);
    }
  }
  for (int wpb : {8, 16, 32}) {
    for (int rep = 0; rep < 2; ++rep) {
      int blocks = sms * 2;
      cudaEventRecord(e0);
      dfma_loop<8><<<blocks, wpb * 32>>>(out, iters, 1.0000001, 1e-9);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double flops = 2.0 * 8 * (double)iters * blocks * wpb * 32;
      if (rep) printf("DFMA: warps/block %d blocks %d -> %.2f TFLOP/s (%.3f ms)\n", wpb, blocks, flops / ms / 1e9, ms);
    }
  }
  {
    const int wpb = 32, blocks = sms * 2;
    auto run_op = [&](auto kern, const char* name, double instr_per_iter) {
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0);
        kern<<<blocks, wpb * 32>>>(out, iters, 1.0000001, 1e-9);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        const double ins = instr_per_iter * (double)iters * blocks * wpb * 32;
        if (rep) printf("%s: %.3f ms  %.2f T FP64 instructions/s (DFMA equivalent %.2f TF)\n", name, ms, ins / ms / 1e9,
                        2 * ins / ms / 1e9);
      }
    };
    run_op(op_loop<8, 0>, "DADD x8 chains       ", 8.0);
    run_op(op_loop<8, 1>, "DMUL x8 chains       ", 8.0);
    run_op(op_loop<8, 2>, "mix add/mul/sub/fma  ", 32.0);
    run_op(dfma_loop<8>, "DFMA x8 chains       ", 8.0);
  }
  // shared or separate FP64 throughput: CH DMMA + NF DFMA per iteration and warp
  {
    const int wpb = 16, blocks = sms * 2;
    auto run = [&](auto kern, const char* name, double dm_flops, double fm_flops) {
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0);
        kern<<<blocks, wpb * 32>>>(out, iters, 1.0000001, 1e-9);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        const double w = (double)iters * blocks * wpb;
        if (rep) printf("%s: %.3f ms  DMMA %.2f TF + DFMA %.2f TF = %.2f TF\n", name, ms, dm_flops * w / ms / 1e9,
                        fm_flops * w / ms / 1e9, (dm_flops + fm_flops) * w / ms / 1e9);
      }
    };
    run(mix_loop<8, 0>, "mix DMMA x8 only      ", 2.0 * 256 * 8, 0.0);
    run(mix_loop<8, 32>, "mix DMMA x8 + DFMA x32", 2.0 * 256 * 8, 2.0 * 32 * 32);
    run(mix_loop<8, 16>, "mix DMMA x8 + DFMA x16", 2.0 * 256 * 8, 2.0 * 32 * 16);
  }
  // layout probe
  double hA[32], hB[32], hC[64], ref[64];
  for (int i = 0; i < 32; ++i) { hA[i] = (i * 7 % 11) - 5; hB[i] = (i * 5 % 13) - 6; }
  for (int m = 0; m < 8; ++m) for (int n = 0; n < 8; ++n) { double s = 0; for (int k = 0; k < 4; ++k) s += hA[m*4+k] * hB[k*8+n]; ref[m*8+n] = s; }
  double *dA, *dB, *dC; cudaMalloc(&dA, 256); cudaMalloc(&dB, 256); cudaMalloc(&dC, 512);
  cudaMemcpy(dA, hA, 256, cudaMemcpyHostToDevice); cudaMemcpy(dB, hB, 256, cudaMemcpyHostToDevice);
  layout_probe<<<1, 32>>>(dA, dB, dC);
  cudaMemcpy(hC, dC, 512, cudaMemcpyDeviceToHost);
  double err = 0; for (int i = 0; i < 64; ++i) err += fabs(hC[i] - ref[i]);
  printf("layout probe abs err sum: %g (%s)\n", err, err == 0 ? "LAYOUT OK" : "LAYOUT MISMATCH");
  printf("last error: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
