// Probe: cost of launching a large-shared-memory kernel right after a kernel with a different L1/shared
// carve-out (does switching the carve-out stall the SMs?).
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/carveout_probe.cu -o /tmp/carveout_probe
#include <cstdio>
#include <cuda_runtime.h>

__global__ void small_k(float* p) { if (threadIdx.x == 0 && p) p[blockIdx.x] = 1.f; }
__global__ void big_k(float* p) {
  extern __shared__ float s[];
  s[threadIdx.x] = threadIdx.x;
  __syncthreads();
  if (threadIdx.x == 0 && p) p[blockIdx.x] = s[5];
}

int main() {
  float* p;
  cudaMalloc(&p, 1 << 20);
  const int big = 225 * 1024;
  cudaFuncSetAttribute(big_k, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaEvent_t e[4];
  for (auto& x : e) cudaEventCreate(&x);
  for (int mode = 0; mode < 3; ++mode) {
    if (mode == 2) cudaFuncSetAttribute(small_k, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    float tot_b = 0.f, tot_s = 0.f;
    for (int it = 0; it < 200; ++it) {
      cudaEventRecord(e[0]);
      if (mode == 0) big_k<<<148, 768, big>>>(p); else small_k<<<148 * 4, 256>>>(p);
      cudaEventRecord(e[1]);
      big_k<<<148, 768, big>>>(p);
      cudaEventRecord(e[2]);
      cudaEventSynchronize(e[2]);
      float a, b;
      cudaEventElapsedTime(&a, e[0], e[1]);
      cudaEventElapsedTime(&b, e[1], e[2]);
      if (it >= 10) { tot_s += a; tot_b += b; }
    }
    printf("%s: first kernel %.2f us, big-smem kernel after it %.2f us\n",
           mode == 0 ? "big after big" : (mode == 1 ? "big after small (default carve-out)" : "big after small (small forced to max-shared carve-out)"),
           1000 * tot_s / 190, 1000 * tot_b / 190);
  }
  return 0;
}
