// Arithmetic type of the nets ("precision 32 switches nets and P to fp32"; reading Z22).
//
// nets.cu and emb.cu (with gemm.cuh / emb.cuh) are written once over `real` and compiled twice:
//   nets.cu, emb.cu      -> namespace fekf::n64, real = double (the paper's precision)
//   nets32.cu, emb32.cu  -> namespace fekf::n32, real = float  (FEKF_NETS32)
// Everything a net pass hands back to the filter or the caller stays fp64: the weight gradient g, the
// error sums, energies, forces and virials (fp32 values widened on store); coordinates, labels and the
// geometry are fp64 and the fp32 nets read fp32 copies of R~, its Jacobian and the weights.
//
// The fp32 tensor path: the nets' 8x8x4 fragment product (fp64: one DMMA m8n8k4) is, for fp32, two
// mma.sync.m16n8k4 tf32 products with the operands split into tf32 hi + lo parts: A's hi part in rows
// 0-7 and its lo part in rows 8-15 of the m16 operand, so the two MMAs (B_hi, then B_lo) accumulate
//   rows 0-7:  A_hi B_hi + A_hi B_lo      rows 8-15:  A_lo B_hi + A_lo B_lo
// and the 8x8 result is the sum of the two halves (same thread, same columns: the m16n8k4 C fragment
// of rows g and g + 8 sits in one thread).  The split keeps 22 of fp32's 24 mantissa bits of each
// operand, every product of the splits is exact in fp32 and the sum runs in fp32: an fp32-accurate
// product on the tensor cores ("3xTF32" with the fourth term for free).
#pragma once
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#ifdef FEKF_NETS32
#define FEKF_NETNS n32
#else
#define FEKF_NETNS n64
#endif

namespace fekf {
namespace FEKF_NETNS {

#ifdef FEKF_NETS32
using real = float;
using real2 = float2;
__host__ __device__ __forceinline__ float2 make_real2(float a, float b) { return make_float2(a, b); }
#else
using real = double;
using real2 = double2;
__host__ __device__ __forceinline__ double2 make_real2(double a, double b) { return make_double2(a, b); }
#endif

__device__ __forceinline__ void dmma884(double& d0, double& d1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
      : "+d"(d0), "+d"(d1)
      : "d"(a), "d"(b));
}

__device__ __forceinline__ uint32_t to_tf32(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return r;
}
// tf32 hi + lo split of an fp32 operand
struct Split32 {
  uint32_t hi, lo;
};
__device__ __forceinline__ Split32 split32(float x) {
  const uint32_t h = to_tf32(x);
  return Split32{h, to_tf32(x - __uint_as_float(h))};
}
// d[0..1] += a (8x4 fragment, row = lane/4, k = lane%4) * b (4x8, k = lane%4, n = lane/4), fp32-accurate
__device__ __forceinline__ void dmma884(float& d0, float& d1, Split32 a, Split32 b) {
  float e0 = 0.f, e1 = 0.f;
  asm("mma.sync.aligned.m16n8k4.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
      : "+f"(d0), "+f"(d1), "+f"(e0), "+f"(e1)
      : "r"(a.hi), "r"(a.lo), "r"(b.hi));
  asm("mma.sync.aligned.m16n8k4.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
      : "+f"(d0), "+f"(d1), "+f"(e0), "+f"(e1)
      : "r"(a.hi), "r"(a.lo), "r"(b.lo));
  d0 += e0;
  d1 += e1;
}
__device__ __forceinline__ void dmma884(float& d0, float& d1, float a, float b) {
  dmma884(d0, d1, split32(a), split32(b));
}

// a fragment operand prepared once for all the products it enters (fp32: its tf32 split)
#ifdef FEKF_NETS32
using frag_t = Split32;
__device__ __forceinline__ Split32 frag(float x) { return split32(x); }
#else
using frag_t = double;
__device__ __forceinline__ double frag(double x) { return x; }
#endif
// byte mask of the alignment a two-element copy needs
constexpr size_t PAIR_MASK = 2 * sizeof(real) - 1;

// one element / two consecutive elements global -> shared (cp.async; src-size 0 zero-fills)
__device__ __forceinline__ void cp_async1(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(d), "l"(src), "r"(valid ? 8 : 0) : "memory");
}
__device__ __forceinline__ void cp_async1(float* dst, const float* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(d), "l"(src), "r"(valid ? 4 : 0) : "memory");
}
__device__ __forceinline__ void cp_async2(double* dst, const double* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(d), "l"(src), "r"(valid ? 16 : 0) : "memory");
}
__device__ __forceinline__ void cp_async2(float* dst, const float* src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(d), "l"(src), "r"(valid ? 8 : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

}  // namespace FEKF_NETNS
}  // namespace fekf
