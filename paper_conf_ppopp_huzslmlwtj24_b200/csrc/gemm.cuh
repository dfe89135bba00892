// fp64 GEMM for the embedding / fitting layers (sm_100a CUDA cores; see DESIGN.md §7 for why fp64
// stays off tcgen05).  C = op(A) op(B) with a fused epilogue.
//   TA: A stored [K x M] (weight gradients, K = rows); TB: B stored [N x K] (data gradients, W^T).
//   Optional "ones" row aug_m of op(A): (k < aug_k ? 1 : 0), so [W-grad ; b-grad] = [H | 1]^T Zbar.
//   Mdev / Kdev: device-resident row counts (compacted rows); CTAs past them exit / contribute 0.
#pragma once
#include "model.cuh"

namespace fekf {

constexpr int GB_M = 64, GB_N = 64, GB_K = 16;

struct EpiStore {
  double* C; int ldc;
  __device__ void operator()(int r, int c, double v) const { C[(size_t)r * ldc + c] = v; }
};
struct EpiPartial {
  double* ws; int M, N; int zoff;
  __device__ void operator()(int r, int c, double v) const {
    ws[((size_t)(blockIdx.z + zoff) * M + r) * N + c] = v;
  }
};
// forward layer: y = tanh(z + b) (primal) or ydot = (1 - y^2) zdot (tangent); h = skip(h_prev) + dt*y
struct EpiFwd {
  double* Y; double* H; int ld;
  const double* bias; const double* dt;
  const double* Hp; int ldp; int skip; int dprev;
  const double* Yprim;    // non-null: tangent rows; primal y of row rowmap[r] (or r)
  const int* rowmap;
  __device__ void operator()(int r, int c, double v) const {
    double sk = 0.0;
    if (skip == 1) sk = Hp[(size_t)r * ldp + c];
    else if (skip == 2) sk = Hp[(size_t)r * ldp + (c % dprev)];
    double y;
    if (Yprim == nullptr) {
      y = tanh(v + bias[c]);
    } else {
      const int rp = rowmap ? rowmap[r] : r;
      const double yp = Yprim[(size_t)rp * ld + c];
      y = (1.0 - yp * yp) * v;
    }
    Y[(size_t)r * ld + c] = y;
    H[(size_t)r * ld + c] = sk + (dt ? dt[c] * y : y);
  }
};
// data gradient: hbar_prev = Zbar W^T + skip^T(hbar)
struct EpiDgrad {
  double* out; int ldo; const double* Hb; int ld; int skip; int dprev;
  __device__ void operator()(int r, int c, double v) const {
    double s = 0.0;
    if (skip == 1) s = Hb[(size_t)r * ld + c];
    else if (skip == 2) s = Hb[(size_t)r * ld + c] + Hb[(size_t)r * ld + c + dprev];
    out[(size_t)r * ldo + c] = v + s;
  }
};

template <bool TA, bool TB, class Epi>
__global__ void __launch_bounds__(256)
dgemm_kernel(int M, int N, int K, const int* __restrict__ Mdev, const int* __restrict__ Kdev,
             const double* __restrict__ A, int lda, const double* __restrict__ B, int ldb, int aug_m, int aug_k,
             int kps, Epi epi) {
  __shared__ __align__(16) double As[2][GB_K][GB_M + 2];
  __shared__ __align__(16) double Bs[2][GB_K][GB_N + 2];
  if (Mdev) M = min(M, *Mdev);
  if (Kdev) {
    const int kd = *Kdev;
    K = min(K, kd);
    aug_k = min(aug_k, kd);
  }
  const int tid = threadIdx.x;
  const int m0 = blockIdx.x * GB_M, n0 = blockIdx.y * GB_N;
  if (m0 >= M) return;
  const int kbeg = blockIdx.z * kps;
  const int kend = min(K, kbeg + kps);
  const int tm = tid >> 4, tn = tid & 15;
  double acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.0;
  double ra[4], rb[4];
  auto load = [&](int k0) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int idx = tid + 256 * q;
      int r, kk;
      if (!TA) { r = idx >> 4; kk = idx & 15; } else { kk = idx >> 6; r = idx & 63; }
      const int m = m0 + r, k = k0 + kk;
      double v = 0.0;
      if (m < M && k < kend) {
        if (m == aug_m) v = (k < aug_k) ? 1.0 : 0.0;
        else v = TA ? A[(size_t)k * lda + m] : A[(size_t)m * lda + k];
      }
      ra[q] = v;
      int c;
      if (!TB) { kk = idx >> 6; c = idx & 63; } else { c = idx >> 4; kk = idx & 15; }
      const int n = n0 + c, k2 = k0 + kk;
      double u = 0.0;
      if (n < N && k2 < kend) u = TB ? B[(size_t)n * ldb + k2] : B[(size_t)k2 * ldb + n];
      rb[q] = u;
    }
  };
  auto store = [&](int buf) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int idx = tid + 256 * q;
      if (!TA) As[buf][idx & 15][idx >> 4] = ra[q]; else As[buf][idx >> 6][idx & 63] = ra[q];
      if (!TB) Bs[buf][idx >> 6][idx & 63] = rb[q]; else Bs[buf][idx & 15][idx >> 4] = rb[q];
    }
  };
  const int nk = kend > kbeg ? (kend - kbeg + GB_K - 1) / GB_K : 0;
  if (nk > 0) {
    load(kbeg);
    store(0);
    __syncthreads();
    for (int t = 0; t < nk; ++t) {
      if (t + 1 < nk) load(kbeg + (t + 1) * GB_K);
      const int buf = t & 1;
#pragma unroll
      for (int kk = 0; kk < GB_K; ++kk) {
        const double2 a01 = *reinterpret_cast<const double2*>(&As[buf][kk][tm * 4]);
        const double2 a23 = *reinterpret_cast<const double2*>(&As[buf][kk][tm * 4 + 2]);
        const double2 b01 = *reinterpret_cast<const double2*>(&Bs[buf][kk][tn * 4]);
        const double2 b23 = *reinterpret_cast<const double2*>(&Bs[buf][kk][tn * 4 + 2]);
        const double a[4] = {a01.x, a01.y, a23.x, a23.y};
        const double b[4] = {b01.x, b01.y, b23.x, b23.y};
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[i][j] = fma(a[i], b[j], acc[i][j]);
      }
      if (t + 1 < nk) store((t + 1) & 1);
      __syncthreads();
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int r = m0 + tm * 4 + i, c = n0 + tn * 4 + j;
      if (r < M && c < N) epi(r, c, acc[i][j]);
    }
}

template <bool TA, bool TB, class Epi>
static fekf_status gemm(long long M, int N, int K, const double* A, int lda, const double* B, int ldb, Epi epi,
                        cudaStream_t s, const int* Mdev = nullptr, const int* Kdev = nullptr, int aug_m = -1,
                        int aug_k = 0, int splits = 1, int kps = 0) {
  if (M <= 0 || N <= 0) return FEKF_OK;
  if (kps <= 0) kps = K;
  dim3 grid((unsigned)cdiv(M, GB_M), (unsigned)cdiv(N, GB_N), (unsigned)splits);
  dgemm_kernel<TA, TB, Epi><<<grid, 256, 0, s>>>((int)M, N, K, Mdev, Kdev, A, lda, B, ldb, aug_m, aug_k, kps, epi);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

}  // namespace fekf
