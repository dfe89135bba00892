// Shared helpers of libfekf (sm_100a).  No method arithmetic lives here.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <string>
#include <vector>

#include "../../include/fekf.h"

namespace fekf {

void set_error(const std::string& msg);

#define FEKF_CHECK_CUDA(expr)                                                               \
  do {                                                                                      \
    cudaError_t e__ = (expr);                                                               \
    if (e__ != cudaSuccess) {                                                               \
      ::fekf::set_error(std::string(#expr) + ": " + cudaGetErrorString(e__));               \
      return FEKF_ECUDA;                                                                    \
    }                                                                                       \
  } while (0)

#define FEKF_LAUNCH_CHECK()                                                                 \
  do {                                                                                      \
    cudaError_t e__ = cudaGetLastError();                                                   \
    if (e__ != cudaSuccess) {                                                               \
      ::fekf::set_error(std::string("kernel launch: ") + cudaGetErrorString(e__) + " at " + \
                        __FILE__ + ":" + std::to_string(__LINE__));                         \
      return FEKF_ECUDA;                                                                    \
    }                                                                                       \
  } while (0)

#define FEKF_TRY(...)                  \
  do {                                 \
    fekf_status s__ = (__VA_ARGS__);   \
    if (s__ != FEKF_OK) return s__;    \
  } while (0)

__host__ __device__ inline int cdiv(int64_t a, int64_t b) { return (int)((a + b - 1) / b); }

// Device buffer owned by the library (cudaMalloc; freed in the owner's destructor).
struct DBuf {
  void* p = nullptr;
  size_t bytes = 0;
  template <class T> T* as() const { return reinterpret_cast<T*>(p); }
};

fekf_status dalloc(DBuf& b, size_t bytes);
void dfree(DBuf& b);

// Per-launch counter used for the launch-count instrumentation (bench.py gpu_launches).
extern thread_local int64_t g_launches;
inline void count_launch(int n = 1) { g_launches += n; }

}  // namespace fekf
