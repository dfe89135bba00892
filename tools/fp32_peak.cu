// Microbenchmark for the fp32 nets variant (reading Z22): FP32 FFMA rate, the legacy tensor path
// mma.sync.m16n8k4 tf32 rate, the split-operand "fp32 m8n8k4" product built from two of them (fp32.cuh),
// and the fp32 tanh cost, on sm_100a.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/fp32_peak.cu -o /tmp/fp32_peak && /tmp/fp32_peak
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void ffma_kernel(float* out, int iters) {
  float a[16], b = 1.0000001f, c = 0.9999999f;
#pragma unroll
  for (int k = 0; k < 16; ++k) a[k] = threadIdx.x * 1e-3f + k;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 16; ++k) a[k] = fmaf(a[k], b, c);
  }
  float s = 0;
#pragma unroll
  for (int k = 0; k < 16; ++k) s += a[k];
  if (s == 12345.0f) out[0] = s;
}

__device__ __forceinline__ uint32_t tf32(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return r;
}

__global__ void hmma_kernel(float* out, int iters) {
  const uint32_t a0 = tf32(threadIdx.x * 1e-3f), a1 = tf32(1.5f), b = tf32(1.0001f);
  float d[4][4];
#pragma unroll
  for (int k = 0; k < 4; ++k) d[k][0] = d[k][1] = d[k][2] = d[k][3] = k;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k)
      asm volatile("mma.sync.aligned.m16n8k4.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                   : "+f"(d[k][0]), "+f"(d[k][1]), "+f"(d[k][2]), "+f"(d[k][3]) : "r"(a0), "r"(a1), "r"(b));
  }
  float s = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k) s += d[k][0] + d[k][1] + d[k][2] + d[k][3];
  if (s == 12345.0f) out[0] = s;
}

// the fp32 8x8x4 product of fp32.cuh: two m16n8k4 per call (hi/lo split of A in the two row halves)
__global__ void split_kernel(float* out, int iters) {
  float a = threadIdx.x * 1e-3f, b = 1.0001f;
  float d[4][2];
#pragma unroll
  for (int k = 0; k < 4; ++k) { d[k][0] = k; d[k][1] = -k; }
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const uint32_t ah = tf32(a), al = tf32(a - __uint_as_float(ah));
      const uint32_t bh = tf32(b), bl = tf32(b - __uint_as_float(bh));
      float e0 = 0.f, e1 = 0.f;
      asm volatile("mma.sync.aligned.m16n8k4.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                   : "+f"(d[k][0]), "+f"(d[k][1]), "+f"(e0), "+f"(e1) : "r"(ah), "r"(al), "r"(bh));
      asm volatile("mma.sync.aligned.m16n8k4.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                   : "+f"(d[k][0]), "+f"(d[k][1]), "+f"(e0), "+f"(e1) : "r"(ah), "r"(al), "r"(bl));
      d[k][0] += e0;
      d[k][1] += e1;
      a += 1e-7f;
    }
  }
  float s = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k) s += d[k][0] + d[k][1];
  if (s == 12345.0f) out[0] = s;
}

__global__ void tanh_kernel(float* out, int iters) {
  float x = threadIdx.x * 1e-4f - 0.3f, s = 0;
  for (int i = 0; i < iters; ++i) {
    s += tanhf(x);
    x += 1e-7f;
  }
  if (s == 12345.0f) out[0] = s;
}

int main() {
  float* out;
  cudaMalloc(&out, 8);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int iters = 20000;
  float ms;
  auto run = [&](auto kern) {
    kern<<<sms * 4, 256>>>(out, iters);
    cudaEventRecord(e0);
    kern<<<sms * 4, 256>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
  };
  const double thr = (double)sms * 4 * 256;
  run(ffma_kernel);
  printf("{\"ffma_tflops\": %.2f, ", 2.0 * 16 * iters * thr / ms / 1e9);
  run(hmma_kernel);
  printf("\"mma_tf32_m16n8k4_tflops\": %.2f, ", 2.0 * 16 * 8 * 4 * 4 * iters * thr / 32 / ms / 1e9);
  run(split_kernel);
  printf("\"split_fp32_884_tflops\": %.2f, ", 2.0 * 8 * 8 * 4 * 4 * iters * thr / 32 / ms / 1e9);
  run(tanh_kernel);
  printf("\"tanhf_gps\": %.2f}\n", (double)iters * thr / ms / 1e6);
  return 0;
}
