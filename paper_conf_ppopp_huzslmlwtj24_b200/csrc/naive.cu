// Naive-EKF (the paper's fusiform-shaped minibatch EKF) on the FEKF filter's storage.
//
// P:L168 / Table 2: delta* = E(K . ABE) — every sample i of the minibatch forms its own Kalman
// gain from the shared P_t, "each sample updates independently and has an individual P matrix",
// and Fig. 5 reduces the per-sample results over the batch.  Readings N1-N4: with
// u_i = P_t g_i, A_i = 1/(c + g_i^T u_i) (Alg. 1 line 8), K_i = A_i u_i (line 9),
//   P_i = (P_t - A_i u_i u_i^T) / lambda            (line 10, per sample)
//   P_{t+1} = (1/n) sum_i P_i = (P_t - U diag(A/n) U^T) / lambda        U = [u_1 .. u_n]
//   w_{t+1} = w_t + (1/n) sum_i ABE_i A_i u_i                           (E(K . ABE), no sqrt(bs))
// so the n individual P_i of the paper's formulation are never materialised: one update is a rank-n
// correction of the shared P, and the paper's P all-reduce (Fig. 5c, (r-1) N^2 per step) becomes an
// all-reduce of the partial U (N n) when P is sharded.
//
// Unlike FEKF (one vector per pass: HBM-bound, kalman.cu), U = P G carries n <= 32 vectors per pass, so
// both passes are DMMA-bound (m8n8k4 fp64 tensor path; tcgen05 has no fp64 kind):
//   pass 1 (read-only):  per stored tile (I, J) of the upper triangle, U_I += P_IJ G_J and, off the
//                        diagonal, U_J += P_IJ^T G_I: 4 * 64^2 * NP flops (2 * 64^2 * NP on the diagonal);
//                        row partials stay in registers over the item (tile-row segment), column partials
//                        go to a workspace slot per tile and are summed per tile column in a fixed order
//                        (the FEKF plan's CSR) — deterministic, no floating-point atomics;
//   pass 2 (read-write): P_IJ <- (P_IJ - U_I diag(A/n) U_J^T) / lambda: 2 * 64^2 * NP flops per tile.
// Pending FEKF corrections (kalman.cu's deferred list) are flushed first, so P_t is the stored P.
#include <algorithm>
#include <cmath>

#include "kalman.cuh"

namespace fekf {

namespace {

constexpr int NKF_THREADS = 256;         // 8 warps, each an 8-row strip of the 64-row tile
constexpr int MV_THREADS = 512;          // pass 1: warps 0-7 the row product, warps 8-15 the column product
constexpr int LDP = KT + 4;              // SMEM row stride of a P tile: conflict-free A-fragment loads both ways
constexpr int TILE_E = KT * KT;

__device__ __forceinline__ void dmma(double& d0, double& d1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
      : "+d"(d0), "+d"(d1)
      : "d"(a), "d"(b));
}
__device__ __forceinline__ void cp16(void* dst, const void* src) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// 64 rows x NP doubles of a [Npad][NP] vector set -> SMEM rows of stride NP + 4
template <int NP, int NTH = NKF_THREADS>
__device__ __forceinline__ void stage_vec(double* dst, const double* src, int tid) {
  constexpr int C = NP / 2;  // 16-byte chunks per row
  for (int e = tid; e < KT * C; e += NTH) {
    const int r = e / C, q = e % C;
    cp16(dst + r * (NP + 4) + 2 * q, src + (size_t)r * NP + 2 * q);
  }
}
template <int NTH>
__device__ __forceinline__ void stage_tile(double* dst, const double* src, int tid) {
  for (int e = tid; e < KT * (KT / 2); e += NTH) {
    const int r = e / (KT / 2), q = e % (KT / 2);
    cp16(dst + r * LDP + 2 * q, src + (size_t)r * KT + 2 * q);
  }
}

}  // namespace

// G [n][ldg] (sample-major, flat parameter order) -> gN [Npad][NP] (position-major, blocks padded to
// whole tiles, zero padding in positions and in samples n..NP-1)
template <int NP>
__global__ void nkf_pad_kernel(const double* __restrict__ G, long long ldg, int n, double* __restrict__ gN,
                               const int* tc_blk, const int* tc_c, const long long* off, const int* nblk,
                               long long npad) {
  const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= npad * NP) return;
  const long long p = e / NP;
  const int j = (int)(e % NP);
  const long long tc = p / KT;
  const int b = tc_blk[tc];
  const int loc = tc_c[tc] * KT + (int)(p % KT);
  gN[e] = (j < n && loc < nblk[b]) ? G[(size_t)j * ldg + off[b] + loc] : 0.0;
}

// Pass 1: partial U = P G over this rank's items.  One CTA per SM pulls items (largest first) from a
// counter; each tile of an item and the G_J segment it needs are double-buffered in SMEM by cp.async.
template <int NP>
__global__ void __launch_bounds__(MV_THREADS, 1)
nkf_mv_kernel(const double* __restrict__ P, const ItemD* __restrict__ items, int n_items, int* counter,
              const double* __restrict__ gN, double* __restrict__ ws, int rps) {
  constexpr int LDG = NP + 4, NT = NP / 8;
  extern __shared__ __align__(16) double sm[];
  double* const sP = sm;                             // [2][KT * LDP]
  double* const sGJ = sm + 2 * KT * LDP;              // [2][KT * LDG]
  double* const sGI = sm + 2 * KT * LDP + 2 * KT * LDG;
  __shared__ int s_item;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, fr = lane >> 2, fk = lane & 3;
  const bool colw = warp >= 8;                       // column-product warp (warp-uniform role)
  const int m0 = 8 * (warp & 7);
  for (;;) {
    if (tid == 0) s_item = atomicAdd(counter, 1);
    __syncthreads();
    const int k = s_item;
    if (k >= n_items) break;
    const ItemD it = items[k];
    const double* Pt = P + (size_t)it.tile_off * TILE_E;
    const double* gI = gN + (size_t)(it.vbase + (long long)it.I * KT) * NP;
    stage_vec<NP, MV_THREADS>(sGI, gI, tid);
    stage_tile<MV_THREADS>(sP, Pt, tid);
    stage_vec<NP, MV_THREADS>(sGJ, gN + (size_t)(it.vbase + (long long)it.J0 * KT) * NP, tid);
    cp_commit();
    double acc[NT][2];
#pragma unroll
    for (int j = 0; j < NT; ++j) acc[j][0] = acc[j][1] = 0.0;
    for (int t = 0; t < it.nJ; ++t) {
      const int b = t & 1;
      if (t + 1 < it.nJ) {
        stage_tile<MV_THREADS>(sP + (b ^ 1) * KT * LDP, Pt + (size_t)(t + 1) * TILE_E, tid);
        stage_vec<NP, MV_THREADS>(sGJ + (b ^ 1) * KT * LDG,
                                  gN + (size_t)(it.vbase + (long long)(it.J0 + t + 1) * KT) * NP, tid);
        cp_commit();
        cp_wait<1>();
      } else {
        cp_wait<0>();
      }
      __syncthreads();
      const double* p = sP + b * KT * LDP;
      if (!colw) {
        // U_I[m0..m0+7][:] += P[m0..m0+7][:] G_J
        const double* gj = sGJ + b * KT * LDG;
#pragma unroll 4
        for (int ks = 0; ks < KT / 4; ++ks) {
          const double a = p[(m0 + fr) * LDP + 4 * ks + fk];
#pragma unroll
          for (int j = 0; j < NT; ++j) dmma(acc[j][0], acc[j][1], a, gj[(4 * ks + fk) * LDG + 8 * j + fr]);
        }
      } else if (it.J0 + t != it.I) {
        // U_J[m0..m0+7][:] = P[:][m0..m0+7]^T G_I -> the tile's column-partial slot
        double z[NT][2];
#pragma unroll
        for (int j = 0; j < NT; ++j) z[j][0] = z[j][1] = 0.0;
#pragma unroll 4
        for (int ks = 0; ks < KT / 4; ++ks) {
          const double a = p[(4 * ks + fk) * LDP + m0 + fr];
#pragma unroll
          for (int j = 0; j < NT; ++j) dmma(z[j][0], z[j][1], a, sGI[(4 * ks + fk) * LDG + 8 * j + fr]);
        }
        double* dst = ws + (size_t)(it.col_slot0 + t) * KT * NP + (m0 + fr) * NP + 2 * fk;
#pragma unroll
        for (int j = 0; j < NT; ++j) *reinterpret_cast<double2*>(dst + 8 * j) = make_double2(z[j][0], z[j][1]);
      }
      __syncthreads();   // buffer b is refilled at t + 2
    }
    if (!colw) {
      // the plan's rps row slots per item: the sum goes to the first, the others are zeroed
      double* dst = ws + (size_t)it.row_slot * rps * KT * NP + (m0 + fr) * NP + 2 * fk;
#pragma unroll
      for (int j = 0; j < NT; ++j) *reinterpret_cast<double2*>(dst + 8 * j) = make_double2(acc[j][0], acc[j][1]);
      for (int g = 1; g < rps; ++g)
#pragma unroll
        for (int j = 0; j < NT; ++j)
          *reinterpret_cast<double2*>(dst + (size_t)g * KT * NP + 8 * j) = make_double2(0.0, 0.0);
    }
  }
}

// U[tc*64 + r][j] = sum over the CSR slots of tile column tc (fixed order)
template <int NP>
__global__ void nkf_reduce_kernel(const double* __restrict__ ws, const long long* __restrict__ ptr,
                                  const long long* __restrict__ idx, double* __restrict__ U) {
  const long long tc = blockIdx.x;
  const int e = blockIdx.y * blockDim.x + threadIdx.x;   // < 64 * NP
  double a = 0.0;
  for (long long q = ptr[tc]; q < ptr[tc + 1]; ++q) a += ws[(size_t)idx[q] * KT * NP + e];
  U[(size_t)tc * KT * NP + e] = a;
}

// dotp[j][tc] = g_j . u_j over tile column tc
template <int NP>
__global__ void nkf_dot_kernel(const double* __restrict__ gN, const double* __restrict__ U, long long n_tc,
                               double* __restrict__ dotp) {
  __shared__ double red[8][NP];
  const long long tc = blockIdx.x;
  const int j = threadIdx.x % NP, r0 = threadIdx.x / NP;   // blockDim = 8 * NP
  double a = 0.0;
  for (int r = r0; r < KT; r += 8) {
    const size_t e = ((size_t)tc * KT + r) * NP + j;
    a = fma(gN[e], U[e], a);
  }
  red[r0][j] = a;
  __syncthreads();
  if (r0 == 0) {
    double s = 0.0;
    for (int q = 0; q < 8; ++q) s += red[q][j];
    dotp[(size_t)j * n_tc + tc] = s;
  }
}

// Per sample j (one CTA each): A_j = 1/(c + g_j^T u_j) (Alg. 1 line 8, c = L lambda or lambda, Z1);
// coef[j] = A_j / n (P correction), coef[NMAX + j] = ABE_j A_j / n (w increment).
__global__ void nkf_finish_kernel(const double* __restrict__ dotp, long long n_tc, int n, const KfState* st,
                                  const double* __restrict__ abe, double* __restrict__ coef, double* A_out) {
  __shared__ double red[256];
  const int j = blockIdx.x;
  double a = 0.0;
  for (long long tc = threadIdx.x; tc < n_tc; tc += blockDim.x) a += dotp[(size_t)j * n_tc + tc];
  red[threadIdx.x] = a;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if ((int)threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const double A = 1.0 / (st->c_mult * st->lambda + red[0]);
    coef[j] = A / n;
    coef[32 + j] = abe[j] * A / n;
    coef[64 + j] = A;
    if (A_out) A_out[j] = A;
  }
}

// lambda_t -> the correction scale 1/lambda_t; lambda <- nu lambda + 1 - nu (line 12, Eq. 3)
__global__ void nkf_state_kernel(KfState* st, double* __restrict__ coef, int n) {
  bool ok = true;
  for (int j = 0; j < n; ++j) ok = ok && isfinite(coef[64 + j]) && isfinite(coef[32 + j]);
  const double lam = st->lambda;
  coef[96] = 1.0 / lam;
  coef[97] = ok ? 0.0 : 1.0;   // a non-finite A_i / ABE_i: the update is a no-op (w, P, lambda kept)
  st->A_last = coef[64 + n - 1];
  if (ok) st->lambda = lam * st->nu + 1.0 - st->nu;
  st->t += 1;
  if (!ok) st->flags |= 2;
}

// w += sum_j (ABE_j A_j / n) u_j on the valid positions
template <int NP>
__global__ void nkf_vec_kernel(const double* __restrict__ U, const double* __restrict__ coef, int n, long long npad,
                               double* __restrict__ w, const int* tc_blk, const int* tc_c, const long long* off,
                               const int* nblk) {
  const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= npad) return;
  const long long tc = p / KT;
  const int b = tc_blk[tc];
  const int loc = tc_c[tc] * KT + (int)(p % KT);
  if (loc >= nblk[b] || coef[97] != 0.0) return;
  double v = 0.0;
  for (int j = 0; j < n; ++j) v = fma(coef[32 + j], U[(size_t)p * NP + j], v);
  w[off[b] + loc] += v;
}

// Pass 2: P_IJ <- (P_IJ - U_I diag(A/n) U_J^T) / lambda on this rank's tiles (one CTA per item; U_I and
// each tile's U_J staged in SMEM, the tile updated in place through double2 accesses).
template <int NP>
__global__ void __launch_bounds__(NKF_THREADS)
nkf_correct_kernel(double* __restrict__ P, const ItemD* __restrict__ items, const double* __restrict__ U,
                   const double* __restrict__ coef, int n) {
  constexpr int LDG = NP + 4;
  extern __shared__ __align__(16) double smc[];
  double* const sUI = smc;                              // [KT * LDG]
  double (*sUJ)[KT * LDG] = reinterpret_cast<double (*)[KT * LDG]>(smc + KT * LDG);   // [2][KT * LDG]
  __shared__ double sc[NP];
  if (coef[97] != 0.0) return;   // non-finite update (nkf_state_kernel): P untouched
  const ItemD it = items[blockIdx.x];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, fr = lane >> 2, fk = lane & 3;
  const int m0 = 8 * warp;
  if (tid < NP) sc[tid] = tid < n ? coef[tid] : 0.0;
  const double inv_lam = coef[96];
  stage_vec<NP>(sUI, U + (size_t)(it.vbase + (long long)it.I * KT) * NP, tid);
  stage_vec<NP>(sUJ[0], U + (size_t)(it.vbase + (long long)it.J0 * KT) * NP, tid);
  cp_commit();
  for (int t = 0; t < it.nJ; ++t) {
    const int b = t & 1;
    // this thread's 16 elements of the tile, in flight while U_J arrives and the correction is formed
    double* row = P + (size_t)(it.tile_off + t) * TILE_E + (m0 + fr) * KT + 2 * fk;
    double2 v[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) v[q] = *reinterpret_cast<const double2*>(row + 8 * q);
    if (t + 1 < it.nJ) {
      stage_vec<NP>(sUJ[b ^ 1], U + (size_t)(it.vbase + (long long)(it.J0 + t + 1) * KT) * NP, tid);
      cp_commit();
      cp_wait<1>();
    } else {
      cp_wait<0>();
    }
    __syncthreads();
    double c[8][2];
#pragma unroll
    for (int q = 0; q < 8; ++q) c[q][0] = c[q][1] = 0.0;
#pragma unroll
    for (int ks = 0; ks < NP / 4; ++ks) {
      const int kk = 4 * ks + fk;
      const double a = sc[kk] * sUI[(m0 + fr) * LDG + kk];
#pragma unroll
      for (int q = 0; q < 8; ++q) dmma(c[q][0], c[q][1], a, sUJ[b][(8 * q + fr) * LDG + kk]);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      v[q].x = (v[q].x - c[q][0]) * inv_lam;
      v[q].y = (v[q].y - c[q][1]) * inv_lam;
      *reinterpret_cast<double2*>(row + 8 * q) = v[q];
    }
    __syncthreads();   // sUJ[b] is restaged at t + 2
  }
}

static int np_for(int n) { return n <= 8 ? 8 : n <= 16 ? 16 : 32; }

static size_t mv_smem(int NP) { return (size_t)(2 * KT * LDP + 3 * KT * (NP + 4)) * sizeof(double); }

// begin: pad G, pass 1 over this rank's tiles and the per-tile-column reduction -> this rank's partial U
template <int NP>
static fekf_status naive_begin_t(Kf& k, const double* G, long long ldg, int n, cudaStream_t s) {
  const KfPlan& p = k.plan;
  const int tb = 256;
  nkf_pad_kernel<NP><<<cdiv(p.Npad * NP, tb), tb, 0, s>>>(G, ldg, n, k.nG.as<double>(), k.tc_blk.as<int>(),
                                                          k.tc_c.as<int>(), k.off_d.as<long long>(), k.n_d.as<int>(),
                                                          p.Npad);
  FEKF_LAUNCH_CHECK();
  count_launch();
  if (!p.items.empty()) {
    FEKF_CHECK_CUDA(cudaMemsetAsync(k.counter.p, 0, sizeof(int), s));
    static int sms = 0;
    if (!sms) {
      int dev = 0;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
      if (sms <= 0) sms = 148;
    }
    const size_t smem = mv_smem(NP);
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(nkf_mv_kernel<NP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int grid = std::min<int>((int)p.items.size(), sms);
    nkf_mv_kernel<NP><<<grid, MV_THREADS, smem, s>>>(k.P.as<double>(), k.items_d.as<ItemD>(), (int)p.items.size(),
                                                     k.counter.as<int>(), k.nG.as<double>(), k.nws.as<double>(), p.rps);
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  nkf_reduce_kernel<NP><<<dim3((unsigned)p.n_tc, KT * NP / 256), 256, 0, s>>>(
      k.nws.as<double>(), k.csr_ptr.as<long long>(), k.csr_idx.as<long long>(), k.nU.as<double>());
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// end: A_i, w, lambda from the (summed) U, then the rank-n correction of this rank's tiles
template <int NP>
static fekf_status naive_end_t(Kf& k, const double* abe, int n, double* w, double* A_out, cudaStream_t s) {
  const KfPlan& p = k.plan;
  nkf_dot_kernel<NP><<<(unsigned)p.n_tc, 8 * NP, 0, s>>>(k.nG.as<double>(), k.nU.as<double>(), p.n_tc,
                                                         k.ndot.as<double>());
  FEKF_LAUNCH_CHECK();
  nkf_finish_kernel<<<n, 256, 0, s>>>(k.ndot.as<double>(), p.n_tc, n, k.state.as<KfState>(), abe,
                                      k.ncoef.as<double>(), A_out);
  FEKF_LAUNCH_CHECK();
  nkf_state_kernel<<<1, 1, 0, s>>>(k.state.as<KfState>(), k.ncoef.as<double>(), n);
  FEKF_LAUNCH_CHECK();
  nkf_vec_kernel<NP><<<cdiv(p.Npad, 256), 256, 0, s>>>(k.nU.as<double>(), k.ncoef.as<double>(), n, p.Npad, w,
                                                       k.tc_blk.as<int>(), k.tc_c.as<int>(), k.off_d.as<long long>(),
                                                       k.n_d.as<int>());
  FEKF_LAUNCH_CHECK();
  count_launch(4);
  if (!p.items.empty()) {
    const size_t csm = (size_t)3 * KT * (NP + 4) * sizeof(double);
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(nkf_correct_kernel<NP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)csm));
    nkf_correct_kernel<NP><<<(unsigned)p.items.size(), NKF_THREADS, csm, s>>>(
        k.P.as<double>(), k.items_d.as<ItemD>(), k.nU.as<double>(), k.ncoef.as<double>(), n);
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  return FEKF_OK;
}

fekf_status Kf::update_naive_begin(const double* G, long long ldg, int n, cudaStream_t s) {
  if (p32) { set_error("kf_update_naive: fp64 P only"); return FEKF_EINVAL; }
  if (n < 1 || n > NAIVE_NMAX) { set_error("kf_update_naive: n must be in [1, 32]"); return FEKF_EINVAL; }
  if (ldg < plan.N) { set_error("kf_update_naive: ldg < N"); return FEKF_EINVAL; }
  if (in_update || naive_n > 0) { set_error("kf_update_naive: an update is in progress"); return FEKF_ESTATE; }
  const int NP = np_for(n);
  if (naive_np < NP) {   // workspace for the widest vector set seen so far
    for (DBuf* b : {&nG, &nU, &nws, &ndot, &ncoef}) dfree(*b);
    FEKF_TRY(dalloc(nG, (size_t)plan.Npad * NP * sizeof(double)));
    FEKF_TRY(dalloc(nU, (size_t)plan.Npad * NP * sizeof(double)));
    FEKF_TRY(dalloc(nws, (size_t)std::max<int64_t>(1, plan.ws_slots) * KT * NP * sizeof(double)));
    FEKF_TRY(dalloc(ndot, (size_t)NP * plan.n_tc * sizeof(double)));
    FEKF_TRY(dalloc(ncoef, 128 * sizeof(double)));
    naive_np = NP;
  }
  if (npend > 0) FEKF_TRY(flush(s));   // P_t is now the stored P (sigma = 1, no deferred terms)
  naive_n = n;
  if (NP == 8) return naive_begin_t<8>(*this, G, ldg, n, s);
  if (NP == 16) return naive_begin_t<16>(*this, G, ldg, n, s);
  return naive_begin_t<32>(*this, G, ldg, n, s);
}

fekf_status Kf::update_naive_end(const double* abe, double* w, double* A_out, cudaStream_t s) {
  if (naive_n <= 0) { set_error("kf_update_naive_end: no naive update begun"); return FEKF_ESTATE; }
  const int n = naive_n;
  naive_n = 0;
  const int NP = np_for(n);
  if (NP == 8) return naive_end_t<8>(*this, abe, n, w, A_out, s);
  if (NP == 16) return naive_end_t<16>(*this, abe, n, w, A_out, s);
  return naive_end_t<32>(*this, abe, n, w, A_out, s);
}

// The U layout of the partial / summed vector set: [N_pad][roundup8(n)] (position-major)
long long Kf::naive_u_len() const { return naive_n > 0 ? plan.Npad * np_for(naive_n) : 0; }

fekf_status Kf::update_naive(const double* G, long long ldg, const double* abe, int n, double* w, double* A_out,
                             cudaStream_t s) {
  FEKF_TRY(update_naive_begin(G, ldg, n, s));
  if (comm && !replicated) FEKF_TRY(comm_allreduce(comm, nU.as<double>(), naive_u_len(), s));
  return update_naive_end(abe, w, A_out, s);
}

}  // namespace fekf
