// Device helpers shared by the fused FFT-tile kernels (sm_100a).
//
// FP64 tensor-core MMA on B200: PTX mma.sync m8n8k4 .f64 lowers to SASS DMMA.8x8x4
// (tcgen05 has no FP64 kind).  Fragment layout (verified on the
// B200 by tools/fp64_peak.cu, profiles/r01_fp64_peak.txt):
//   lane = 4*g + q   (g = lane>>2 in 0..7, q = lane&3 in 0..3)
//   A (8x4): a = A[g][q]          B (4x8): b = B[q][g]
//   C (8x8): c[j] = C[g][2q+j], j = 0,1
// Register chaining (§3.3 "Swizzling Fragments", L266-L272): the C fragment of
// M is, element for element, a B fragment of M^T when the contraction index of the next
// product visits the 8 columns of a C tile as two k-chunks {0,2,4,6} and {1,3,5,7}.  The
// DFT matrix side (A operand) is read with the same column permutation, which we bake into
// the shared-memory layout of every matrix (perm8 below), so every fragment load is "row
// g, four consecutive doubles" and bank-conflict free with a row stride of L+4 doubles.
#pragma once

#include <cstdint>

namespace fstencil {
namespace dev {

__device__ __forceinline__ void dmma(double (&c)[2], double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
      : "+d"(c[0]), "+d"(c[1])
      : "d"(a), "d"(b));
}

// Complex 8x8x8 product C = A . B on DMMA, A given as per-thread A fragments (two k-chunks),
// B as B fragments; CONJ multiplies by conj(A).  4 DMMA per k-chunk (4M form).
template <bool CONJ>
__device__ __forceinline__ void cgemm8(const double (&ar)[2], const double (&ai)[2], const double (&br)[2],
                                       const double (&bi)[2], double (&cr)[2], double (&ci)[2]) {
  cr[0] = cr[1] = ci[0] = ci[1] = 0.0;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    if (CONJ) {
      dmma(cr, ar[j], br[j]);
      dmma(cr, ai[j], bi[j]);
      dmma(ci, ar[j], bi[j]);
      dmma(ci, -ai[j], br[j]);
    } else {
      dmma(cr, ar[j], br[j]);
      dmma(cr, -ai[j], bi[j]);
      dmma(ci, ar[j], bi[j]);
      dmma(ci, ai[j], br[j]);
    }
  }
}

// Physical column of logical column c inside its group of 8: even columns first.
__host__ __device__ __forceinline__ int perm8(int c) {
  return (c & ~7) | ((c & 1) << 2) | ((c & 7) >> 1);
}

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

}  // namespace dev
}  // namespace fstencil
