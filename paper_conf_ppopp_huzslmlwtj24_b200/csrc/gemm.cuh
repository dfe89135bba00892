// GEMM for the embedding / fitting layers in the nets' type (real.cuh).  fp64: the sm_100a FP64 tensor path
// (DMMA, mma.sync.m8n8k4.f64; measured on B200 at the same 37 TFLOP/s as FP64 FFMA but with ~5x less
// shared-memory traffic per FMA); tcgen05 has no fp64 kind, and TF32 would break the fp64 parity.
// fp32: the same fragments through real.cuh's split-tf32 pair of mma.sync.m16n8k4 (fp32-accurate).
// C = op(A) op(B) with a fused epilogue:
//   TA: A stored [K x M] (weight gradients, K = rows); TB: B stored [N x K] (data gradients, W^T).
//   Optional "ones" row aug_m of op(A): (k < aug_k ? 1 : 0), so [W-grad ; b-grad] = [H | 1]^T Zbar.
//   Mdev / Kdev: device-resident row counts (compacted rows); CTAs past them exit.
// CTA tile BM x BN x 16, 8 warps each WM x WN (WM/8 x WN/8 DMMA tiles), operands staged in SMEM
// k-contiguous with a 20-element row stride (conflict-free fragment loads), 3-stage cp.async ring.
#pragma once
#include <algorithm>
#include <cstdlib>

#include "model.cuh"
#include "mathx.cuh"
#include "real.cuh"

namespace fekf {
namespace FEKF_NETNS {

constexpr int GB_K = 16;
constexpr int GB_LDS = GB_K + 4;

// Every epilogue gets split(z) (the CTA's split-K index) before its first use.
template <class O>
struct EpiStore {   // O = double: a weight gradient straight into g (fp64 whatever the nets' precision)
  O* C; int ldc;
  __device__ void split(int) {}
  __device__ void operator()(int r, int c, real v) const { C[(size_t)r * ldc + c] = (O)v; }
};
struct EpiPartial {
  real* ws; int M, N; int zoff;
  __device__ void split(int z) { zoff += z; }
  __device__ void operator()(int r, int c, real v) const {
    ws[((size_t)zoff * M + r) * N + c] = v;
  }
};
// forward layer: y = tanh(z + b) (primal) or ydot = (1 - y^2) zdot (tangent); h = skip(h_prev) + dt*y
struct EpiFwd {
  __device__ void split(int) {}
  real* Y; real* H; int ld;
  const real* bias; const real* dt;
  const real* Hp; int ldp; int skip; int dprev;
  const real* Yprim;    // non-null: tangent rows; primal y of row rowmap[r] (or r)
  const int* rowmap;
  __device__ void operator()(int r, int c, real v) const {
    real sk = 0.0;
    if (skip == 1) sk = Hp[(size_t)r * ldp + c];
    else if (skip == 2) sk = Hp[(size_t)r * ldp + (c % dprev)];
    real y;
    if (Yprim == nullptr) {
      y = tanh_r(v + bias[c]);
    } else {
      const int rp = rowmap ? rowmap[r] : r;
      const real yp = Yprim[(size_t)rp * ld + c];
      y = (real(1) - yp * yp) * v;
    }
    Y[(size_t)r * ld + c] = y;
    H[(size_t)r * ld + c] = sk + (dt ? dt[c] * y : y);
  }
};
// data gradient: hbar_prev = Zbar W^T + skip^T(hbar)
struct EpiDgrad {
  __device__ void split(int) {}
  real* out; int ldo; const real* Hb; int ld; int skip; int dprev;
  __device__ void operator()(int r, int c, real v) const {
    real s = 0.0;
    if (skip == 1) s = Hb[(size_t)r * ld + c];
    else if (skip == 2) s = Hb[(size_t)r * ld + c] + Hb[(size_t)r * ld + c + dprev];
    out[(size_t)r * ldo + c] = v + s;
  }
};

// data gradient fused with the previous layer's activation adjoint (embedding, no timestep):
//   hbar_prev = Zbar W^T + skip^T(hbar);  zbar_prev = (1 - y^2) hbar_prev [- 2 y ydot hdotbar_prev]
// primal launch: the tangent rows of the same layer are done first (tpos / Yt / Hbt);
// tangent launch: y of the primal row rowmap[r].
struct EpiDgradAct {
  __device__ void split(int) {}
  real* out; int ldo; const real* Hb; int ld; int skip; int dprev;
  const real* Y; real* Zb;
  const int* tpos; const real* Yt; const real* Hbt;
  const int* rowmap;
  __device__ void operator()(int r, int c, real v) const {
    real s = 0.0;
    if (skip == 1) s = Hb[(size_t)r * ld + c];
    else if (skip == 2) s = Hb[(size_t)r * ld + c] + Hb[(size_t)r * ld + c + dprev];
    const real hb = v + s;
    const size_t o = (size_t)r * ldo + c;
    out[o] = hb;
    const real y = Y[(rowmap ? (size_t)rowmap[r] : (size_t)r) * ldo + c];
    real z = (real(1) - y * y) * hb;
    if (tpos) {
      const int tr = tpos[r];
      if (tr >= 0) {
        const size_t ot = (size_t)tr * ldo + c;
        z -= real(2) * y * Yt[ot] * Hbt[ot];
      }
    }
    Zb[o] = z;
  }
};

constexpr int GB_STAGES = 3;

// A group of up to GG_MAX independent GEMMs of the same shape class in one launch (e.g. one fitting
// layer of every atom type): CTAs are numbered across the problems' tile grids.
constexpr int GG_MAX = 8;
template <class Epi>
struct GemmProb {
  int M, N, K;
  const int* Mdev;   // device row count (compacted rows) or nullptr
  const int* Kdev;   // device K (split-K over rows) or nullptr
  const real* A; int lda;
  const real* B; int ldb;
  int aug_m, aug_k;  // "ones" row of op(A) (bias gradient), -1: none
  int kps, splits;   // K per split, number of splits
  Epi epi;
};
template <class Epi>
struct GemmGroup {
  int n;
  int start[GG_MAX + 1];   // first CTA of each problem
  int mt[GG_MAX], nt[GG_MAX];
  GemmProb<Epi> p[GG_MAX];
};
template <class Epi>
__device__ __forceinline__ GemmProb<Epi> pick(const GemmGroup<Epi>& G, int q) {
  // static indices only (a dynamic index into the parameter struct would copy it to local memory)
  switch (q) {
    case 0: return G.p[0];
    case 1: return G.p[1];
    case 2: return G.p[2];
    case 3: return G.p[3];
    case 4: return G.p[4];
    case 5: return G.p[5];
    case 6: return G.p[6];
    default: return G.p[7];
  }
}

// Mainloop: GB_STAGES-deep cp.async ring (global -> SMEM without register staging), one
// __syncthreads per BK slice, warp tiles of (WM/8) x (WN/8) DMMA 8x8 tiles.
template <int BM, int BN, int WM, int WN, bool TA, bool TB, class Epi, int NW = 8>
__global__ void __launch_bounds__(32 * NW)
dgemm_kernel(const __grid_constant__ GemmGroup<Epi> G) {
  constexpr int NT = 32 * NW;
  constexpr int NWN = BN / WN;
  static_assert((BM / WM) * NWN == NW, "warp grid");
  constexpr int TI = WM / 8, TJ = WN / 8;
  constexpr int AE = (BM * GB_K + NT - 1) / NT, BE = (BN * GB_K + NT - 1) / NT;
  // SMEM layout follows the operand's global layout so consecutive threads copy consecutive
  // addresses: k-contiguous [mn][GB_LDS] (A row-major / B given as [N x K]) or mn-contiguous
  // [k][MN + 4] (A given as [K x M] / B row-major [K x N]).  Both strides make the 8x4 DMMA fragment
  // loads bank-conflict free.
  constexpr int ASZ = TA ? GB_K * (BM + 4) : BM * GB_LDS;
  constexpr int BSZ = TB ? BN * GB_LDS : GB_K * (BN + 4);
  extern __shared__ __align__(16) real gsm[];
  real* As0 = gsm;
  real* Bs0 = gsm + GB_STAGES * ASZ;
  auto a_at = [&](int buf, int m, int k) -> real& {
    return TA ? As0[buf * ASZ + k * (BM + 4) + m] : As0[buf * ASZ + m * GB_LDS + k];
  };
  auto b_at = [&](int buf, int n, int k) -> real& {
    return TB ? Bs0[buf * BSZ + n * GB_LDS + k] : Bs0[buf * BSZ + k * (BN + 4) + n];
  };
  int q = 0;
#pragma unroll
  for (int k = 1; k < GG_MAX; ++k)
    if (k < G.n && (int)blockIdx.x >= G.start[k]) q = k;
  const GemmProb<Epi> P = pick(G, q);
  const int local = blockIdx.x - G.start[q];
  int mtq = G.mt[0], ntq = G.nt[0];
#pragma unroll
  for (int k = 1; k < GG_MAX; ++k)
    if (q == k) { mtq = G.mt[k]; ntq = G.nt[k]; }
  const int bm = local % mtq, bn = (local / mtq) % ntq, bz = local / (mtq * ntq);
  int M = P.M, K = P.K, aug_k = P.aug_k;
  const int N = P.N, lda = P.lda, ldb = P.ldb, aug_m = P.aug_m, kps = P.kps;
  const real* __restrict__ A = P.A;
  const real* __restrict__ B = P.B;
  Epi epi = P.epi;
  epi.split(bz);
  if (P.Mdev) M = min(M, *P.Mdev);
  if (P.Kdev) {
    const int kd = *P.Kdev;
    K = min(K, kd);
    aug_k = min(aug_k, kd);
  }
  const int tid = threadIdx.x;
  const int m0 = bm * BM, n0 = bn * BN;
  const int kbeg = bz * kps;
  if (m0 >= M || (bz > 0 && kbeg >= K)) return;  // empty split: the reduction skips it
  const int kend = min(K, kbeg + kps);
  const int warp = tid >> 5, lane = tid & 31;
  const int wm = warp / NWN, wn = warp % NWN;
  const int fr = lane >> 2, fk = lane & 3;
  real acc[TI][TJ][2];
#pragma unroll
  for (int i = 0; i < TI; ++i)
#pragma unroll
    for (int j = 0; j < TJ; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;
  // two-element copies (16 bytes fp64, 8 bytes fp32, along the contiguous dimension) when the problem's strides, bases and
  // extents keep every pair inside one row and aligned; per problem, so warp-uniform
  const bool a16 = !TA && aug_m < 0 && !(lda & 1) && !(reinterpret_cast<size_t>(A) & PAIR_MASK) && !(K & 1) && !(kps & 1);
  // TA (A stored [K x M], m-contiguous): pairs (m, m+1) of real columns go as one two-element copy; the pair
  // holding the last real column / the "ones" row is done element by element
  const bool a16t = TA && !(lda & 1) && !(reinterpret_cast<size_t>(A) & PAIR_MASK);
  const int mreal = aug_m >= 0 ? min(M, aug_m) : M;
  const bool b16 = !(ldb & 1) && !(reinterpret_cast<size_t>(B) & PAIR_MASK) && (TB ? (!(K & 1) && !(kps & 1)) : !(N & 1));
  auto issue = [&](int buf, int k0) {
    if (a16t) {
#pragma unroll
      for (int q = 0; q < (AE + 1) / 2; ++q) {
        const int idx = tid + NT * q;
        if (idx >= BM * GB_K / 2) break;
        const int kk = idx / (BM / 2), r = 2 * (idx % (BM / 2));
        const int m = m0 + r, k = k0 + kk;
        const bool kin = k < kend;
        if (m + 1 < mreal) {
          cp_async2(&a_at(buf, r, kk), kin ? A + (size_t)k * lda + m : A, kin);
        } else {
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            real* dst = &a_at(buf, r + h, kk);
            if (m + h == aug_m) {
              *dst = (k < aug_k) ? real(1) : real(0);
            } else {
              const bool ok = m + h < M && kin;
              cp_async1(dst, ok ? A + (size_t)k * lda + m + h : A, ok);
            }
          }
        }
      }
    } else if (a16) {
#pragma unroll
      for (int q = 0; q < (AE + 1) / 2; ++q) {
        const int idx = tid + NT * q;
        if (idx >= BM * GB_K / 2) break;
        const int r = idx / (GB_K / 2), kk = 2 * (idx % (GB_K / 2));
        const int m = m0 + r, k = k0 + kk;
        const bool ok = m < M && k < kend;
        cp_async2(&a_at(buf, r, kk), ok ? A + (size_t)m * lda + k : A, ok);
      }
    } else {
#pragma unroll
    for (int q = 0; q < AE; ++q) {
      const int idx = tid + NT * q;
      if (BM * GB_K % NT && idx >= BM * GB_K) break;
      int r, kk;
      if (!TA) { r = idx / GB_K; kk = idx % GB_K; } else { kk = idx / BM; r = idx % BM; }
      const int m = m0 + r, k = k0 + kk;
      real* dst = &a_at(buf, r, kk);
      if (m == aug_m) {
        *dst = (k < aug_k) ? real(1) : real(0);
      } else {
        const bool ok = m < M && k < kend;
        const real* src = ok ? (TA ? A + (size_t)k * lda + m : A + (size_t)m * lda + k) : A;
        cp_async1(dst, src, ok);
      }
    }
    }
    if (b16) {
#pragma unroll
      for (int q = 0; q < (BE + 1) / 2; ++q) {
        const int idx = tid + NT * q;
        if (idx >= BN * GB_K / 2) break;
        int c, kk;
        if (!TB) { kk = idx / (BN / 2); c = 2 * (idx % (BN / 2)); } else { c = idx / (GB_K / 2); kk = 2 * (idx % (GB_K / 2)); }
        const int n = n0 + c, k = k0 + kk;
        const bool ok = n < N && k < kend;
        cp_async2(&b_at(buf, c, kk), ok ? (TB ? B + (size_t)n * ldb + k : B + (size_t)k * ldb + n) : B, ok);
      }
      return;
    }
#pragma unroll
    for (int q = 0; q < BE; ++q) {
      const int idx = tid + NT * q;
      if (BN * GB_K % NT && idx >= BN * GB_K) break;
      int c, kk;
      if (!TB) { kk = idx / BN; c = idx % BN; } else { c = idx / GB_K; kk = idx % GB_K; }
      const int n = n0 + c, k = k0 + kk;
      const bool ok = n < N && k < kend;
      const real* src = ok ? (TB ? B + (size_t)n * ldb + k : B + (size_t)k * ldb + n) : B;
      cp_async1(&b_at(buf, c, kk), src, ok);
    }
  };
  const int nk = kend > kbeg ? (kend - kbeg + GB_K - 1) / GB_K : 0;
#pragma unroll
  for (int st = 0; st < GB_STAGES - 1; ++st) {
    if (st < nk) issue(st, kbeg + st * GB_K);
    cp_async_commit();
  }
  for (int t = 0; t < nk; ++t) {
    cp_async_wait<GB_STAGES - 2>();
    __syncthreads();  // slice t visible to all; slice t-1's buffer free for reuse
    const int tn = t + GB_STAGES - 1;
    if (tn < nk) issue(tn % GB_STAGES, kbeg + tn * GB_K);
    cp_async_commit();
    const int buf = t % GB_STAGES;
#pragma unroll
    for (int ks = 0; ks < GB_K; ks += 4) {
      frag_t a[TI], b[TJ];
#pragma unroll
      for (int i = 0; i < TI; ++i) a[i] = frag(a_at(buf, wm * WM + i * 8 + fr, ks + fk));
#pragma unroll
      for (int j = 0; j < TJ; ++j) b[j] = frag(b_at(buf, wn * WN + j * 8 + fr, ks + fk));
#pragma unroll
      for (int i = 0; i < TI; ++i)
#pragma unroll
        for (int j = 0; j < TJ; ++j) dmma884(acc[i][j][0], acc[i][j][1], a[i], b[j]);
    }
  }
  cp_async_wait<0>();
#pragma unroll
  for (int i = 0; i < TI; ++i)
#pragma unroll
    for (int j = 0; j < TJ; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int r = m0 + wm * WM + i * 8 + fr, c = n0 + wn * WN + j * 8 + 2 * fk + h;
        if (r < M && c < N) epi(r, c, acc[i][j][h]);
      }
}

#ifdef FEKF_NETS32
// fp32 nets: the same GEMM on the FP32 FFMA pipe (measured 71.5 TFLOP/s on B200, vs 34.6 for an
// fp32-accurate product on the split-tf32 mma.sync pair; tools/fp32_peak.cu).  256 threads as a 16 x 16
// grid, each a TM x TN register micro-tile (TM = BM/16 rows, TN = BN/16 columns strided by 16), the k loop
// four at a time.  Operands stay in SMEM in their global orientation: an operand contiguous along k (A
// row-major, B given as [N x K]) as [row][k] (stride BK + 4, 16-byte cp.async; a thread's rows strided by
// 16 so the two row groups of a warp hit different banks), one contiguous along m / n as [k][mn] (stride
// MN + 4; A's TM rows of a thread consecutive and read as float4 along m).  Same GemmGroup / split-K /
// device row-count / "ones" row semantics as dgemm_kernel; the epilogue gets every element of the tile.
__device__ __forceinline__ void cp_async16n(float* dst, const float* src, int nbytes) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(d), "l"(src), "r"(nbytes) : "memory");
}
template <int BM, int BN, bool TA, bool TB, class Epi>
__global__ void __launch_bounds__(256)
sgemm_kernel(const __grid_constant__ GemmGroup<Epi> G) {
  constexpr int NT = 256, TM = BM / 16, TN = BN / 16, LK = GB_K + 4, LA = BM + 4, LB = BN + 4;
  constexpr bool AK = !TA, BK = TB;   // operand contiguous along k
  constexpr int ASZ = AK ? BM * LK : GB_K * LA, BSZ = BK ? BN * LK : GB_K * LB;
  static_assert(TM % 4 == 0 && BN % 16 == 0, "sgemm micro-tile");
  extern __shared__ __align__(16) real gsm[];
  real* As0 = gsm;
  real* Bs0 = gsm + GB_STAGES * ASZ;
  int q = 0;
#pragma unroll
  for (int k = 1; k < GG_MAX; ++k)
    if (k < G.n && (int)blockIdx.x >= G.start[k]) q = k;
  const GemmProb<Epi> P = pick(G, q);
  const int local = blockIdx.x - G.start[q];
  int mtq = G.mt[0], ntq = G.nt[0];
#pragma unroll
  for (int k = 1; k < GG_MAX; ++k)
    if (q == k) { mtq = G.mt[k]; ntq = G.nt[k]; }
  const int bm = local % mtq, bn = (local / mtq) % ntq, bz = local / (mtq * ntq);
  int M = P.M, K = P.K, aug_k = P.aug_k;
  const int N = P.N, lda = P.lda, ldb = P.ldb, aug_m = P.aug_m, kps = P.kps;
  const real* __restrict__ A = P.A;
  const real* __restrict__ B = P.B;
  Epi epi = P.epi;
  epi.split(bz);
  if (P.Mdev) M = min(M, *P.Mdev);
  if (P.Kdev) {
    const int kd = *P.Kdev;
    K = min(K, kd);
    aug_k = min(aug_k, kd);
  }
  const int tid = threadIdx.x;
  const int m0 = bm * BM, n0 = bn * BN;
  const int kbeg = bz * kps;
  if (m0 >= M || (bz > 0 && kbeg >= K)) return;  // empty split: the reduction skips it
  const int kend = min(K, kbeg + kps);
  const int ty = tid >> 4, tx = tid & 15;
  real acc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; ++i)
#pragma unroll
    for (int j = 0; j < TN; ++j) acc[i][j] = 0.f;
  const int mreal = aug_m >= 0 ? min(M, aug_m) : M;
  // 16-byte copies along k when the row stride, the base and the split's first k are 16-byte aligned (slices
  // advance by GB_K); a ragged end of K is zero-filled by the copy's source size
  const bool a4 = AK && aug_m < 0 && !(lda & 3) && !(reinterpret_cast<size_t>(A) & 15) && !(kbeg & 3);
  const bool b4 = BK && !(ldb & 3) && !(reinterpret_cast<size_t>(B) & 15) && !(kbeg & 3);
  const bool a2 = !AK && !(lda & 1) && !(reinterpret_cast<size_t>(A) & PAIR_MASK);
  const bool b2 = !BK && !(ldb & 1) && !(reinterpret_cast<size_t>(B) & PAIR_MASK) && !(N & 1);
  auto issue = [&](int buf, int k0) {
    real* As = As0 + buf * ASZ;
    real* Bs = Bs0 + buf * BSZ;
    if (AK) {   // A row-major [M x K] -> [m][k]
      if (a4) {
        for (int idx = tid; idx < BM * GB_K / 4; idx += NT) {
          const int r = idx / (GB_K / 4), kk = 4 * (idx % (GB_K / 4));
          const int m = m0 + r, k = k0 + kk;
          const int nb = (m < M && k < kend) ? 4 * min(4, kend - k) : 0;
          cp_async16n(As + r * LK + kk, nb ? A + (size_t)m * lda + k : A, nb);
        }
      } else {
        for (int idx = tid; idx < BM * GB_K; idx += NT) {
          const int r = idx / GB_K, kk = idx % GB_K;
          const int m = m0 + r, k = k0 + kk;
          real* dst = As + r * LK + kk;
          if (m == aug_m) *dst = (k < aug_k) ? real(1) : real(0);
          else {
            const bool ok = m < M && k < kend;
            cp_async1(dst, ok ? A + (size_t)m * lda + k : A, ok);
          }
        }
      }
    } else {    // A stored [K x M] -> [k][m]
      for (int idx = tid; idx < GB_K * BM / 2; idx += NT) {
        const int kk = idx / (BM / 2), r = 2 * (idx % (BM / 2));
        const int m = m0 + r, k = k0 + kk;
        const bool kin = k < kend;
        if (a2 && m + 1 < mreal) {
          cp_async2(As + kk * LA + r, kin ? A + (size_t)k * lda + m : A, kin);
        } else {
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            real* dst = As + kk * LA + r + h;
            if (m + h == aug_m) *dst = (k < aug_k) ? real(1) : real(0);
            else {
              const bool ok = m + h < M && kin;
              cp_async1(dst, ok ? A + (size_t)k * lda + m + h : A, ok);
            }
          }
        }
      }
    }
    if (BK) {   // B given as [N x K] -> [n][k]
      if (b4) {
        for (int idx = tid; idx < BN * GB_K / 4; idx += NT) {
          const int c = idx / (GB_K / 4), kk = 4 * (idx % (GB_K / 4));
          const int n = n0 + c, k = k0 + kk;
          const int nb = (n < N && k < kend) ? 4 * min(4, kend - k) : 0;
          cp_async16n(Bs + c * LK + kk, nb ? B + (size_t)n * ldb + k : B, nb);
        }
      } else {
        for (int idx = tid; idx < BN * GB_K; idx += NT) {
          const int c = idx / GB_K, kk = idx % GB_K;
          const int n = n0 + c, k = k0 + kk;
          const bool ok = n < N && k < kend;
          cp_async1(Bs + c * LK + kk, ok ? B + (size_t)n * ldb + k : B, ok);
        }
      }
    } else {    // B row-major [K x N] -> [k][n]
      if (b2) {
        for (int idx = tid; idx < GB_K * BN / 2; idx += NT) {
          const int kk = idx / (BN / 2), c = 2 * (idx % (BN / 2));
          const int n = n0 + c, k = k0 + kk;
          const bool ok = n < N && k < kend;
          cp_async2(Bs + kk * LB + c, ok ? B + (size_t)k * ldb + n : B, ok);
        }
      } else {
        for (int idx = tid; idx < GB_K * BN; idx += NT) {
          const int kk = idx / BN, c = idx % BN;
          const int n = n0 + c, k = k0 + kk;
          const bool ok = n < N && k < kend;
          cp_async1(Bs + kk * LB + c, ok ? B + (size_t)k * ldb + n : B, ok);
        }
      }
    }
  };
  // the thread's rows: AK strided by 16 (conflict-free float4 along k), else TM consecutive (float4 along m)
  auto row_of = [&](int i) { return AK ? ty + 16 * i : ty * TM + i; };
  const int nk = kend > kbeg ? (kend - kbeg + GB_K - 1) / GB_K : 0;
#pragma unroll
  for (int st = 0; st < GB_STAGES - 1; ++st) {
    if (st < nk) issue(st, kbeg + st * GB_K);
    cp_async_commit();
  }
  for (int t = 0; t < nk; ++t) {
    cp_async_wait<GB_STAGES - 2>();
    __syncthreads();  // slice t visible to all; slice t-1's buffer free for reuse
    const int tn = t + GB_STAGES - 1;
    if (tn < nk) issue(tn % GB_STAGES, kbeg + tn * GB_K);
    cp_async_commit();
    const real* As = As0 + (t % GB_STAGES) * ASZ;
    const real* Bs = Bs0 + (t % GB_STAGES) * BSZ;
#pragma unroll
    for (int k4 = 0; k4 < GB_K; k4 += 4) {
      real a[TM][4], b[TN][4];
#pragma unroll
      for (int i = 0; i < TM; ++i) {
        if (AK) {
          const float4 v = *reinterpret_cast<const float4*>(As + row_of(i) * LK + k4);
          a[i][0] = v.x; a[i][1] = v.y; a[i][2] = v.z; a[i][3] = v.w;
        } else if (i % 4 == 0) {
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const float4 v = *reinterpret_cast<const float4*>(As + (k4 + u) * LA + ty * TM + i);
            a[i][u] = v.x; a[i + 1][u] = v.y; a[i + 2][u] = v.z; a[i + 3][u] = v.w;
          }
        }
      }
#pragma unroll
      for (int j = 0; j < TN; ++j) {
        if (BK) {
          const float4 v = *reinterpret_cast<const float4*>(Bs + (tx + 16 * j) * LK + k4);
          b[j][0] = v.x; b[j][1] = v.y; b[j][2] = v.z; b[j][3] = v.w;
        } else {
#pragma unroll
          for (int u = 0; u < 4; ++u) b[j][u] = Bs[(k4 + u) * LB + tx + 16 * j];
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int i = 0; i < TM; ++i)
#pragma unroll
          for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(a[i][u], b[j][u], acc[i][j]);
    }
  }
  cp_async_wait<0>();
#pragma unroll
  for (int i = 0; i < TM; ++i)
#pragma unroll
    for (int j = 0; j < TN; ++j) {
      const int r = m0 + row_of(i), c = n0 + tx + 16 * j;
      if (r < M && c < N) epi(r, c, acc[i][j]);
    }
}
#endif

template <int BM, int BN, int WM, int WN, bool TA, bool TB, class Epi, int NW = 8>
static fekf_status gemm_launch(GemmGroup<Epi>& G, cudaStream_t s) {
#ifdef FEKF_NETS32
  constexpr size_t smem = sizeof(real) * GB_STAGES * ((TA ? GB_K * (BM + 4) : BM * (GB_K + 4)) +
                                                      (TB ? BN * (GB_K + 4) : GB_K * (BN + 4)));
  auto kern = sgemm_kernel<BM, BN, TA, TB, Epi>;
  constexpr int nthr = 256;
#else
  constexpr size_t asz = TA ? GB_K * (BM + 4) : BM * GB_LDS;
  constexpr size_t bsz = TB ? BN * GB_LDS : GB_K * (BN + 4);
  constexpr size_t smem = sizeof(real) * GB_STAGES * (asz + bsz);
  auto kern = dgemm_kernel<BM, BN, WM, WN, TA, TB, Epi, NW>;
  constexpr int nthr = 32 * NW;
#endif
  static bool attr = false;
  if (!attr) {
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = true;
  }
  int tot = 0;
  for (int q = 0; q < G.n; ++q) {
    G.mt[q] = cdiv(G.p[q].M, BM);
    G.nt[q] = cdiv(G.p[q].N, BN);
    G.start[q] = tot;
    tot += G.mt[q] * G.nt[q] * G.p[q].splits;
  }
  for (int q = G.n; q <= GG_MAX; ++q) G.start[q] = tot;
  if (tot == 0) return FEKF_OK;
  kern<<<tot, nthr, smem, s>>>(G);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// One launch for every problem of the group.  Tile from the group's shape: N <= 32 -> 128x32
// (embedding widths); N a multiple of 80 up to 320 (the fitting widths) -> 128x80; otherwise 64x64
// (warps 32x16) unless the group has many rows -> 128x64.
template <bool TA, bool TB, class Epi>
static fekf_status gemm_group(GemmProb<Epi>* probs, int n, cudaStream_t s) {
  GemmGroup<Epi> G{};
  long long rows = 0;
  int nmax = 0;
  for (int q = 0; q < n; ++q) {
    if (probs[q].M <= 0 || probs[q].N <= 0) continue;
    if (probs[q].kps <= 0) probs[q].kps = probs[q].K;
    if (probs[q].splits <= 0) probs[q].splits = 1;
    G.p[G.n++] = probs[q];
    rows += probs[q].M;
    nmax = std::max(nmax, probs[q].N);
  }
  if (G.n == 0) return FEKF_OK;
  if (nmax <= 32) return gemm_launch<128, 32, 32, 16, TA, TB>(G, s);
  // the fitting widths (240) over a long K (the first fitting layer, K = M M^< = 1600): 128 x 80 tiles put N
  // in 3 tiles and 6144 rows in 48, one wave of 144 CTAs on 148 SMs (64 x 64 tiles: 384 CTAs,
  // 2.6 waves): measured 220 -> 203 us (ncu); then 16 warps of 16 x 40 instead of 8 of 32 x 40 (4 warps per
  // SMSP instead of 2, at 0.7 instead of 0.45 fragment loads per DMMA): 196 -> 181 us live.  The 16-warp tile
  // also wins for the K = 240 layers (forward 47 -> 42.5 us, data gradient 36.4 -> 33.2 us; the 8-warp 128 x 80
  // tile lost to 64 x 64 there, 62 vs 49 us); 128 x 64 tiles with 16 warps measured slower on the generic path
  if (!TA && nmax % 80 == 0 && nmax <= 320 && rows >= 2048)
    return gemm_launch<128, 80, 16, 40, TA, TB, Epi, 16>(G, s);
  static const long long big_rows = [] {   // experiment knob: rows from which the generic path takes 128 x 64
    const char* v = getenv("FEKF_GEMM_BIG_ROWS");
    return v ? atoll(v) : 65536LL;
  }();
  if (rows < big_rows) return gemm_launch<64, 64, 32, 16, TA, TB>(G, s);
  return gemm_launch<128, 64, 32, 32, TA, TB>(G, s);
}

template <bool TA, bool TB, class Epi>
static fekf_status gemm(long long M, int N, int K, const real* A, int lda, const real* B, int ldb, Epi epi,
                        cudaStream_t s, const int* Mdev = nullptr, const int* Kdev = nullptr, int aug_m = -1,
                        int aug_k = 0, int splits = 1, int kps = 0) {
  GemmProb<Epi> p{(int)M, N, K, Mdev, Kdev, A, lda, B, ldb, aug_m, aug_k, kps, splits, epi};
  return gemm_group<TA, TB>(&p, 1, s);
}

}  // namespace FEKF_NETNS
}  // namespace fekf
