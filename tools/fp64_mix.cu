// Microbenchmark: do fp64 DMMA (mma.sync.m8n8k4.f64) and DFMA share the FP64 units on sm_100a?
// Runs DMMA-only, DFMA-only, and both at once (even warps DMMA, odd warps DFMA, same work each as the
// single runs) and the library's tanh_fp64 throughput.
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I paper_conf_ppopp_huzslmlwtj24_b200/csrc tools/fp64_mix.cu -o /tmp/fp64_mix
#include <cstdio>
#include <cuda_runtime.h>

#include "mathx.cuh"

__device__ __forceinline__ void dfma_loop(double* out, int iters) {
  double a[8], b = 1.0000001, c = 0.9999999;
#pragma unroll
  for (int k = 0; k < 8; ++k) a[k] = threadIdx.x * 1e-3 + k;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = fma(a[k], b, c);
  }
  double s = 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) s += a[k];
  if (s == 12345.0) out[0] = s;
}
__device__ __forceinline__ void dmma_loop(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0001;
  double d[4][2];
#pragma unroll
  for (int k = 0; k < 4; ++k) { d[k][0] = k; d[k][1] = -k; }
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(d[k][0]), "+d"(d[k][1]) : "d"(a), "d"(b));
  }
  double s = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k) s += d[k][0] + d[k][1];
  if (s == 12345.0) out[0] = s;
}
// mode 0: DFMA (iters_f), 1: DMMA (iters_m), 2: even warps DMMA + odd warps DFMA
__global__ void mix_kernel(double* out, int mode, int iters_m, int iters_f) {
  const int w = threadIdx.x >> 5;
  if (mode == 0 || (mode == 2 && (w & 1))) dfma_loop(out, iters_f);
  else dmma_loop(out, iters_m);
}
__global__ void tanh_kernel(double* out, int iters) {
  double x[4], s = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k) x[k] = threadIdx.x * 1e-4 - 0.3 + k;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k) { s += fekf::tanh_fp64(x[k]); x[k] += 1e-7; }
  }
  if (s == 12345.0) out[0] = s;
}

int main() {
  double* out;
  cudaMalloc(&out, 8);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int im = 20000, iff = 20000;
  const int grid = sms * 4, block = 256;
  const double threads = (double)grid * block;
  const double fl_f = 2.0 * 8 * iff * threads, fl_m = 2.0 * 256 * 4 * im * threads / 32;
  float ms[3], msf = 0.f;
  for (int rep = 0; rep < 2; ++rep)
    for (int mode = 0; mode < 3; ++mode) {
      cudaEventRecord(e0);
      mix_kernel<<<grid, block>>>(out, mode, im, iff);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&ms[mode], e0, e1);
    }
  msf = ms[0];
  printf("DFMA alone: %.2f TFLOP/s (%.3f ms)\n", fl_f / ms[0] / 1e9, ms[0]);
  printf("DMMA alone: %.2f TFLOP/s (%.3f ms)\n", fl_m / ms[1] / 1e9, ms[1]);
  printf("half warps DMMA + half DFMA: %.3f ms; sum of the halves run alone %.3f ms, max %.3f ms -> %s\n", ms[2],
         0.5 * (ms[0] + ms[1]), 0.5 * (ms[0] > ms[1] ? ms[0] : ms[1]),
         ms[2] > 0.85 * 0.5 * (ms[0] + ms[1]) ? "shared units" : "independent units");
  const int it = 5000;
  for (int rep = 0; rep < 2; ++rep) {
    cudaEventRecord(e0);
    tanh_kernel<<<grid, block>>>(out, it);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms[0], e0, e1);
  }
  const double n = 4.0 * it * threads;
  const double dfma_rate = 8.0 * iff * threads / msf;   // DFMA lane-ops per ms
  printf("tanh_fp64: %.2f Gtanh/s = %.1f DFMA lane-ops of time each\n", n / ms[0] / 1e6, dfma_rate / (n / ms[0]));
  return 0;
}
