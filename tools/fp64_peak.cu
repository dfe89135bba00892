// Microbenchmark: fp64 DFMA vs DMMA (mma.sync.m8n8k4.f64) throughput and fp64 tanh cost on sm_100a.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/fp64_peak.cu -o /tmp/fp64_peak && /tmp/fp64_peak
#include <cstdio>
#include <cuda_runtime.h>

__global__ void dfma_kernel(double* out, int iters) {
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

__global__ void dmma_kernel(double* out, int iters) {
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

__global__ void tanh_kernel(double* out, int iters) {
  double x = threadIdx.x * 1e-4 - 0.3, s = 0;
  for (int i = 0; i < iters; ++i) {
    s += tanh(x);
    x += 1e-7;
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
  const int iters = 20000;
  for (int rep = 0; rep < 2; ++rep) {
    cudaEventRecord(e0);
    dfma_kernel<<<sms * 4, 256>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    double flops = 2.0 * 8 * iters * (double)sms * 4 * 256;
    if (rep) printf("DFMA: %.2f TFLOP/s\n", flops / ms / 1e9);
    cudaEventRecord(e0);
    dmma_kernel<<<sms * 4, 256>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    flops = 2.0 * 8 * 8 * 4 * 4 * iters * (double)sms * 4 * 256 / 32;
    if (rep) printf("DMMA m8n8k4: %.2f TFLOP/s\n", flops / ms / 1e9);
    cudaEventRecord(e0);
    tanh_kernel<<<sms * 4, 256>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    double n = (double)iters * sms * 4 * 256;
    if (rep) printf("tanh f64: %.2f Gtanh/s (%.1f DFMA-equivalents each at the DFMA rate above)\n", n / ms / 1e6, 0.0);
  }
  return 0;
}
