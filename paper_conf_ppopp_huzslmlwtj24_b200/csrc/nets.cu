// DeePMD se_a nets on sm_100a: forward, backward to coordinates, energy- and force-Jacobians.  Written over
// the nets' type `real` (real.cuh): compiled as fp64 (this file, namespace n64) and as fp32 (nets32.cu, n32).
//
//   embedding  G = E2 o E1 o E0(s)          P:L84-90 (§2.1 item 2), skip rule: reading Z12
//   descriptor X = R~^T G / N_m, D = X^T X^<   P:L92, P:L233 (Fig. 6), scale 1/N_m: reading Z13
//   fitting    E_i = F3 o F2 o F1 o F0(D)    P:L95-101, residual timestep dt: reading Z14
//   forces     F = -dE/dx via dE/dX by Eq. 4 and the R~ chain rule (Opt1)
//   force-Jacobian: d/dw of Edot = <dE/dx, v> (forward-mode tangent along v, then reverse over the
//     primal+tangent graph).  Each weight gradient is one split-K GEMM over primal + tangent rows.
//
// Row layouts:
//   embedding net (ti,tj): COMPACTED rows, valid slots only (a prefix of each type section of the
//     sorted neighbour list), ordered (b, k, s); row_start[b*n_ti + k] gives atom (b, atoms_of[ti][k]).
//     Tangent rows (force-Jacobian) are the ACTIVE rows only (i or j among the selected atoms, where
//     R~-dot = J (v_j - v_i) can be non-zero), kept in primal order: tidx[t] -> r, tpos[r] -> t | -1.
//     Row counts live on the device (graph-friendly); launches are sized for the maxima.
//   fitting net t: row r = b*n_t + k, stacked [primal rows | tangent rows] (every atom is active).
#include <algorithm>

#include "gemm.cuh"
#include "emb.cuh"

namespace fekf {
namespace FEKF_NETNS {

// =================================================================================================
// weight gradients: [W-grad ; b-grad] (din+1 x dout) = [H | 1]^T Zbar + [Hdot | 0]^T Zdotbar
// (the bias does not enter the tangent).  Two row segments (primal, tangent), split-K partials summed
// in a fixed order -> written to g at the W offset (W then b are contiguous in the layout).
// =================================================================================================
// Sum the live split-K partials in a fixed order: splits [0, S0eff) of segment 0 and
// [S0max, S0max + S1eff) of segment 1, where S*eff follow the device row counts (empty splits never
// wrote).  Two outputs per thread (16-byte loads when the workspace rows allow), the splits summed in
// index order -> deterministic.  All split loads of one thread are independent (unrolled by 4), so the
// kernel streams the (L2-resident) workspace instead of waiting on one load per split.
template <bool V2>
__global__ void __launch_bounds__(256) splitk_reduce_kernel(const real* __restrict__ ws, int S0max, int S1max,
                                                            int kps, const int* __restrict__ K0dev,
                                                            const int* __restrict__ K1dev, int M, int N,
                                                            double* __restrict__ out, int accum) {
  const long long MN = (long long)M * N;
  const long long i = 2 * ((long long)blockIdx.x * blockDim.x + threadIdx.x);
  if (i >= MN) return;
  int S0 = S0max, S1 = S1max;
  if (K0dev) S0 = min(S0max, max(1, (*K0dev + kps - 1) / kps));
  if (K1dev && S1max > 0) S1 = min(S1max, max(1, (*K1dev + kps - 1) / kps));
  const bool two = i + 1 < MN;
  real a0 = 0.0, a1 = 0.0;
  auto seg = [&](const real* base, int S) {
#pragma unroll 4
    for (int z = 0; z < S; ++z) {
      const real* p = base + (size_t)z * MN + i;
      if (V2) {
        const real2 v = *reinterpret_cast<const real2*>(p);
        a0 += v.x;
        a1 += v.y;
      } else {
        a0 += p[0];
        if (two) a1 += p[1];
      }
    }
  };
  seg(ws, S0);
  seg(ws + (size_t)S0max * MN, S1);
  out[i] = accum ? out[i] + a0 : a0;
  if (two) out[i + 1] = accum ? out[i + 1] + a1 : a1;
}
// Few outputs over many splits (the fitting output layer: 241 x 1 over 2 x 64 splits): 32 outputs x 8
// split-lanes per CTA, fixed 8-way combine.
__global__ void __launch_bounds__(256) splitk_reduce_lanes_kernel(const real* __restrict__ ws, int S0max, int S1max,
                                                                  int kps, const int* __restrict__ K0dev,
                                                                  const int* __restrict__ K1dev, int M, int N,
                                                                  double* __restrict__ out, int accum) {
  __shared__ real red[8][32];
  const int lane = threadIdx.x & 31, zl = threadIdx.x >> 5;
  const long long i = (long long)blockIdx.x * 32 + lane;
  const long long MN = (long long)M * N;
  int S0 = S0max, S1 = S1max;
  if (K0dev) S0 = min(S0max, max(1, (*K0dev + kps - 1) / kps));
  if (K1dev && S1max > 0) S1 = min(S1max, max(1, (*K1dev + kps - 1) / kps));
  real a = 0.0;
  if (i < MN) {
#pragma unroll 4
    for (int z = zl; z < S0; z += 8) a += ws[(size_t)z * MN + i];
#pragma unroll 4
    for (int z = zl; z < S1; z += 8) a += ws[(size_t)(S0max + z) * MN + i];
  }
  red[zl][lane] = a;
  __syncthreads();
  if (zl == 0 && i < MN) {
    real t = red[0][lane];
#pragma unroll
    for (int q = 1; q < 8; ++q) t += red[q][lane];
    out[i] = accum ? out[i] + t : t;
  }
}
static void splitk_reduce(const real* ws, int S0, int S1, int kps, const int* k0, const int* k1, int M, int N,
                          double* out, bool accum, cudaStream_t s) {
  const long long MN = (long long)M * N;
  if (S0 + S1 > 16) {
    splitk_reduce_lanes_kernel<<<cdiv(MN, 32), 256, 0, s>>>(ws, S0, S1, kps, k0, k1, M, N, out, accum ? 1 : 0);
    return;
  }
  const unsigned blocks = (unsigned)cdiv(cdiv(MN, 2), 256);
  if (!(MN & 1) && !(reinterpret_cast<size_t>(ws) & 15))
    splitk_reduce_kernel<true><<<blocks, 256, 0, s>>>(ws, S0, S1, kps, k0, k1, M, N, out, accum ? 1 : 0);
  else
    splitk_reduce_kernel<false><<<blocks, 256, 0, s>>>(ws, S0, S1, kps, k0, k1, M, N, out, accum ? 1 : 0);
}

struct Seg {
  const real* H; const real* Zb; long long kmax; const int* kdev; int ones;
};

// accum: add into gout (embedding nets shared by several type pairs, type_one_side) instead of writing
static fekf_status wgrad(Ctx& c, int din, int dout, Seg s0, Seg s1, double* gout, cudaStream_t s, bool accum = false) {
  const int M = din + 1, N = dout;
  const long long tiles = (long long)cdiv(M, 64) * cdiv(N, 64);
  const long long kmax = std::max(s0.kmax, s1.kmax);
  const long long budget = std::max<long long>(1, (long long)(c.splitk_elems / ((size_t)M * N)));
  long long want = std::max<long long>(1, cdiv(2 * 148, tiles));
  int kps = (int)std::max<long long>(4 * GB_K, cdiv(cdiv(kmax, want), GB_K) * GB_K);
  auto nsplit = [&](const Seg& g) { return g.kmax > 0 ? (long long)cdiv(g.kmax, kps) : 0LL; };
  while (nsplit(s0) + nsplit(s1) > budget) kps *= 2;
  const long long S0 = nsplit(s0), S1 = nsplit(s1);
  if (S0 + S1 == 0) return FEKF_OK;
  if (S0 == 1 && S1 == 0 && !accum)
    return gemm<true, false>(M, N, (int)s0.kmax, s0.H, din, s0.Zb, dout, EpiStore<double>{gout, dout}, s, nullptr, s0.kdev,
                             din, s0.ones ? (int)s0.kmax : 0);
  real* ws = c.splitk_ws.as<real>();
  if (S0) FEKF_TRY(gemm<true, false>(M, N, (int)s0.kmax, s0.H, din, s0.Zb, dout, EpiPartial{ws, M, N, 0}, s, nullptr,
                                     s0.kdev, din, s0.ones ? (int)s0.kmax : 0, (int)S0, kps));
  if (S1) FEKF_TRY(gemm<true, false>(M, N, (int)s1.kmax, s1.H, din, s1.Zb, dout, EpiPartial{ws, M, N, (int)S0}, s,
                                     nullptr, s1.kdev, din, s1.ones ? (int)s1.kmax : 0, (int)S1, kps));
  splitk_reduce(ws, (int)S0, (int)S1, kps, s0.kdev, s1.kdev, M, N, gout, accum, s);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// The weight gradients of several layers (one per atom type) in one grouped split-K launch plus one
// fixed-order reduction per layer (same partition rule as wgrad()).
struct WgradJob {
  int din, dout;
  Seg s0, s1;
  double* gout;
};
static fekf_status wgrad_group(Ctx& c, WgradJob* jobs, int n, cudaStream_t s) {
  GemmProb<EpiPartial> pr[GG_MAX];
  int np = 0;
  long long S0[FEKF_MAX_TYPES], S1[FEKF_MAX_TYPES], kps_[FEKF_MAX_TYPES];
  size_t off[FEKF_MAX_TYPES];
  size_t used = 0;
  const size_t share = c.splitk_elems / (size_t)n;
  for (int q = 0; q < n; ++q) {
    const WgradJob& J = jobs[q];
    const int M = J.din + 1, N = J.dout;
    const long long tiles = (long long)cdiv(M, 64) * cdiv(N, 64);
    const long long kmax = std::max(J.s0.kmax, J.s1.kmax);
    const long long budget = std::max<long long>(1, (long long)(share / ((size_t)M * N)));
    long long want = std::max<long long>(1, cdiv(2 * 148, tiles * n));
    int kps = (int)std::max<long long>(4 * GB_K, cdiv(cdiv(kmax, want), GB_K) * GB_K);
    auto nsplit = [&](const Seg& g) { return g.kmax > 0 ? (long long)cdiv(g.kmax, kps) : 0LL; };
    while (nsplit(J.s0) + nsplit(J.s1) > budget) kps *= 2;
    S0[q] = nsplit(J.s0);
    S1[q] = nsplit(J.s1);
    kps_[q] = kps;
    off[q] = used;
    used += (size_t)(S0[q] + S1[q]) * M * N;
    real* ws = c.splitk_ws.as<real>() + off[q];
    if (S0[q])
      pr[np++] = GemmProb<EpiPartial>{M, N, (int)J.s0.kmax, nullptr, J.s0.kdev, J.s0.H, J.din, J.s0.Zb, J.dout,
                                      J.din, J.s0.ones ? (int)J.s0.kmax : 0, kps, (int)S0[q], EpiPartial{ws, M, N, 0}};
    if (S1[q])
      pr[np++] = GemmProb<EpiPartial>{M, N, (int)J.s1.kmax, nullptr, J.s1.kdev, J.s1.H, J.din, J.s1.Zb, J.dout,
                                      J.din, J.s1.ones ? (int)J.s1.kmax : 0, kps, (int)S1[q],
                                      EpiPartial{ws, M, N, (int)S0[q]}};
  }
  FEKF_TRY(gemm_group<true, false>(pr, np, s));
  for (int q = 0; q < n; ++q) {
    const WgradJob& J = jobs[q];
    const int M = J.din + 1, N = J.dout;
    if (S0[q] + S1[q] == 0) continue;
    splitk_reduce(c.splitk_ws.as<real>() + off[q], (int)S0[q], (int)S1[q], (int)kps_[q], J.s0.kdev, J.s1.kdev, M,
                  N, J.gout, false, s);
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  return FEKF_OK;
}

// =================================================================================================
// elementwise / small kernels
// =================================================================================================
// fitting (stacked rows): zbar = (1 - y^2) ybar - 2 y ydot ydotbar, zdotbar = (1 - y^2) ydotbar;
// ybar = dt * hbar on residual layers with a timestep vector, else hbar.  One launch for every atom type of
// a layer (blockIdx.y = type; the types' layers have the same widths).
constexpr int MT = FEKF_MAX_TYPES;
struct ActArgs {
  long long R[MT];                  // primal rows per type (the tangent half follows at R)
  const real* Y[MT];
  const real* Hb[MT];
  const real* dt[MT];               // timestep vector or nullptr
  real* Zb[MT];
  real* ws[MT];                     // act_bwd_dt: per-type column-partial workspace
  double* gdt[MT];                  // act_bwd_dt: the timestep gradient (in g)
  int chunk[MT], nchunk[MT];
  int d, dual;
};
__global__ void act_bwd_kernel(const __grid_constant__ ActArgs A) {
  const int t = blockIdx.y;
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long R = A.R[t];
  const int d = A.d;
  if (i >= R * d) return;
  const int c = (int)(i % d);
  const real* __restrict__ Y = A.Y[t];
  const real* __restrict__ Hb = A.Hb[t];
  const real* __restrict__ dt = A.dt[t];
  real* __restrict__ Zb = A.Zb[t];
  const real y = Y[i];
  const real tt = real(1) - y * y;
  real yb = Hb[i];
  if (dt) yb *= dt[c];
  if (A.dual) {
    const size_t j = (size_t)R * d + i;
    const real yd = Y[j];
    real ydb = Hb[j];
    if (dt) ydb *= dt[c];
    Zb[i] = tt * yb - real(2) * y * yd * ydb;
    Zb[j] = tt * ydb;
  } else {
    Zb[i] = tt * yb;
  }
}

// embedding (compacted rows; tangent rows via tpos)
__global__ void emb_act_bwd_kernel(int Rmax, const int* __restrict__ Rdev, int d, const real* __restrict__ Y,
                                   const real* __restrict__ Hb, const int* __restrict__ tpos,
                                   const real* __restrict__ Yt, const real* __restrict__ Hbt, int dual,
                                   real* __restrict__ Zb, real* __restrict__ Zbt) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long R = min(Rmax, *Rdev);
  if (i >= R * d) return;
  const long long r = i / d;
  const int c = (int)(i % d);
  const real y = Y[i];
  const real t = real(1) - y * y;
  real z = t * Hb[i];
  if (dual) {
    const int tr = tpos[r];
    if (tr >= 0) {
      const size_t j = (size_t)tr * d + c;
      const real ydb = Hbt[j];
      z -= real(2) * y * Yt[j] * ydb;
      Zbt[j] = t * ydb;
    }
  }
  Zb[i] = z;
}

// act_bwd fused with the timestep gradient of the layer (two fixed-order stages):
//   dt[c] = sum_r y[r][c] hbar[r][c] + sum_r ydot[r][c] hdotbar[r][c]   (h = skip + dt * y)
// block (b, type): rows [b chunk, (b+1) chunk) of the type's primal half (and the same rows of its tangent
// half), one thread per column (coalesced rows); the per-block sums go to ws[type][b][c] and colsum_reduce
// adds them.
__global__ void act_bwd_dt_kernel(const __grid_constant__ ActArgs A) {
  const int t = blockIdx.y;
  if ((int)blockIdx.x >= A.nchunk[t]) return;
  const long long R = A.R[t];
  const int d = A.d, chunk = A.chunk[t];
  const long long r0 = (long long)blockIdx.x * chunk;
  const long long r1 = min(R, r0 + chunk);
  const real* __restrict__ Y = A.Y[t];
  const real* __restrict__ Hb = A.Hb[t];
  const real* __restrict__ dt = A.dt[t];
  real* __restrict__ Zb = A.Zb[t];
  for (int c = threadIdx.x; c < d; c += blockDim.x) {
    const real dtc = dt[c];
    real acc = 0.0;
#pragma unroll 4
    for (long long r = r0; r < r1; ++r) {
      const size_t i = (size_t)r * d + c;
      const real y = Y[i], hb = Hb[i];
      const real tt = real(1) - y * y;
      acc += y * hb;
      if (A.dual) {
        const size_t j = (size_t)R * d + i;
        const real yd = Y[j], hdb = Hb[j];
        const real ydb = hdb * dtc;
        Zb[i] = tt * (hb * dtc) - real(2) * y * yd * ydb;
        Zb[j] = tt * ydb;
        acc += yd * hdb;
      } else {
        Zb[i] = tt * (hb * dtc);
      }
    }
    A.ws[t][(size_t)blockIdx.x * d + c] = acc;
  }
}
// out[c] = sum_k ws[k][c]: 32 columns x 8 chunk-lanes per CTA, fixed 8-way combine (blockIdx.y = type)
__global__ void colsum_reduce_kernel(const __grid_constant__ ActArgs A) {
  __shared__ real red[8][33];
  const int t = blockIdx.y;
  const int cl = threadIdx.x & 31, z = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + cl, d = A.d, nchunk = A.nchunk[t];
  const real* __restrict__ ws = A.ws[t];
  real a = 0.0;
  if (c < d) {
#pragma unroll 4
    for (int k = z; k < nchunk; k += 8) a += ws[(size_t)k * d + c];
  }
  red[z][cl] = a;
  __syncthreads();
  if (z == 0 && c < d) {
    real v = red[0][cl];
#pragma unroll
    for (int q = 1; q < 8; ++q) v += red[q][cl];
    A.gdt[t][c] = v;
  }
}
// the activation adjoint of one fitting layer for every type (and, with timestep vectors and weight
// gradients wanted, the timestep gradients); A's per-type pointers and R filled by the caller
static fekf_status act_bwd_types(Ctx& c, ActArgs& A, int nt, bool with_dt, cudaStream_t s) {
  long long Rmax = 0;
  for (int t = 0; t < nt; ++t) Rmax = std::max(Rmax, A.R[t]);
  if (Rmax == 0) return FEKF_OK;
  if (!with_dt) {
    act_bwd_kernel<<<dim3(cdiv(Rmax * A.d, 256), nt), 256, 0, s>>>(A);
    FEKF_LAUNCH_CHECK();
    count_launch();
    return FEKF_OK;
  }
  int cmax = 1;
  for (int t = 0; t < nt; ++t) {
    A.chunk[t] = (int)std::max<long long>(4, cdiv(A.R[t], 2 * 148));
    A.nchunk[t] = A.R[t] > 0 ? (int)cdiv(A.R[t], A.chunk[t]) : 0;
    if ((size_t)A.nchunk[t] * A.d > c.colsum_elems) { set_error("colsum workspace too small"); return FEKF_EINVAL; }
    A.ws[t] = c.colsum_ws.as<real>() + (size_t)t * c.colsum_elems;
    cmax = std::max(cmax, A.nchunk[t]);
  }
  act_bwd_dt_kernel<<<dim3(cmax, nt), std::min(256, (A.d + 31) / 32 * 32), 0, s>>>(A);
  FEKF_LAUNCH_CHECK();
  colsum_reduce_kernel<<<dim3(cdiv(A.d, 32), nt), 256, 0, s>>>(A);
  FEKF_LAUNCH_CHECK();
  count_launch(2);
  return FEKF_OK;
}

constexpr int NP = FEKF_MAX_TYPES * FEKF_MAX_TYPES;

struct Geo {
  int Na, Nm, nt, M, M2, nb;
  int sec[FEKF_MAX_TYPES + 1];
  int sel[FEKF_MAX_TYPES];
  int ncnt[FEKF_MAX_TYPES];
  const int* types;
  const int* tindex;
  const int* atoms;      // concatenated atoms_of
  const int* atoms_off;  // [nt+1]
};
struct PairPtrs {
  const real* G[NP];       // primal H_last (G)
  const real* Gt[NP];      // tangent H_last (Gdot)
  const int* row_start[NP];
  const int* row_idx[NP];
  const int* tpos[NP];
  const real* sbar[NP];
};
struct FitPtrs {
  real* D[FEKF_MAX_TYPES];
  const real* Db[FEKF_MAX_TYPES];
  real* eout[FEKF_MAX_TYPES];
  real* ebar[FEKF_MAX_TYPES];
  long long F[FEKF_MAX_TYPES];
};

static Geo make_geo(Ctx& c, int nb) {
  Geo g{};
  g.Na = c.Na; g.Nm = c.Nm; g.nt = c.nt; g.M = c.M; g.M2 = c.M2; g.nb = nb;
  for (int t = 0; t <= c.nt; ++t) g.sec[t] = c.sec[t];
  for (int t = 0; t < c.nt; ++t) { g.sel[t] = c.m.sel[t]; g.ncnt[t] = (int)c.atoms_of[t].size(); }
  g.types = c.types_d.as<int>();
  g.tindex = c.tindex_d.as<int>();
  g.atoms = c.atoms_d.as<int>();
  g.atoms_off = c.atoms_off_d.as<int>();
  return g;
}
static long long pair_rows(Ctx& c, int p, int nb) {
  return (long long)nb * c.atoms_of[c.pairs[p].ti].size() * c.m.sel[c.pairs[p].tj];
}
static long long fit_rows(Ctx& c, int t, int nb) { return (long long)nb * c.atoms_of[t].size(); }
static const int* rcount(Ctx& c, int p) { return c.rowcnt.as<int>() + p; }
static const int* tcount(Ctx& c, int p) { return c.rowcnt.as<int>() + c.pairs.size() + p; }

// ---------------------------------------------------------------------------------------------
// compaction (fixed-order scans -> deterministic row order); primal rows: build_rows below
// ---------------------------------------------------------------------------------------------
// active tangent rows: v_i != 0 or v_j != 0 (R~-dot = J (v_j - v_i) vanishes otherwise).
// Three passes (chunk counts, chunk scan, scatter), chunks of 1024 rows, order = primal order.
constexpr int TCHUNK = 1024;
__device__ __forceinline__ bool row_active(int r, int Na, int Nm, const int* __restrict__ row_idx,
                                           const int* __restrict__ nl_j, const real* __restrict__ v) {
  const int idx = row_idx[r];
  const int atom = idx / Nm;
  const int b = atom / Na;
  const int j = nl_j[idx];
  const real* vi = v + (size_t)atom * 3;
  const real* vj = v + ((size_t)b * Na + j) * 3;
  return vi[0] != 0.0 || vi[1] != 0.0 || vi[2] != 0.0 || vj[0] != 0.0 || vj[1] != 0.0 || vj[2] != 0.0;
}
// every pair in one launch per pass (blockIdx.y = pair; chunks past a pair's extent exit)
struct TrowArgs {
  int Na, Nm;
  const int* nl_j; const real* v;
  int Rmax[NP];
  const int* Rdev[NP];
  const int* row_idx[NP];
  int* ck[NP];
  int* cnt[NP];
  int* tidx[NP];
  int* tpos[NP];
};
__global__ void __launch_bounds__(TCHUNK) tcount_kernel(const __grid_constant__ TrowArgs A) {
  const int p = blockIdx.y;
  if ((int)blockIdx.x >= cdiv(A.Rmax[p], TCHUNK)) return;
  const int R = min(A.Rmax[p], *A.Rdev[p]);
  const int r = blockIdx.x * TCHUNK + threadIdx.x;
  const bool a = r < R && row_active(r, A.Na, A.Nm, A.row_idx[p], A.nl_j, A.v);
  const int n = __syncthreads_count(a);
  if (threadIdx.x == 0) A.ck[p][blockIdx.x] = n;
}
// exclusive scan of one pair's chunk counts (block p): each thread owns a run of consecutive chunks
__global__ void __launch_bounds__(1024) tscan_kernel(const __grid_constant__ TrowArgs A) {
  __shared__ int wsum[32];
  const int p = blockIdx.x;
  const int nchunk = cdiv(A.Rmax[p], TCHUNK);
  int* ck = A.ck[p];
  const int per = cdiv(nchunk, 1024);
  const int k0 = min(nchunk, (int)threadIdx.x * per), k1 = min(nchunk, k0 + per);
  int mine = 0;
  for (int k = k0; k < k1; ++k) mine += ck[k];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  int incl = mine;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    int x = wsum[lane], xi = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, xi, o);
      if (lane >= o) xi += y;
    }
    wsum[lane] = xi - x;
    if (lane == 31) *A.cnt[p] = xi;
  }
  __syncthreads();
  int run = wsum[warp] + incl - mine;
  for (int k = k0; k < k1; ++k) { const int x = ck[k]; ck[k] = run; run += x; }
}
__global__ void __launch_bounds__(TCHUNK) tscatter_kernel(const __grid_constant__ TrowArgs A) {
  __shared__ int wsum[TCHUNK / 32];
  const int p = blockIdx.y;
  if ((int)blockIdx.x >= cdiv(A.Rmax[p], TCHUNK)) return;
  const int R = min(A.Rmax[p], *A.Rdev[p]);
  const int r = blockIdx.x * TCHUNK + threadIdx.x;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const bool a = r < R && row_active(r, A.Na, A.Nm, A.row_idx[p], A.nl_j, A.v);
  const unsigned bal = __ballot_sync(0xffffffffu, a);
  if (lane == 0) wsum[warp] = __popc(bal);
  __syncthreads();
  if (threadIdx.x == 0) {
    int run = 0;
    for (int w = 0; w < TCHUNK / 32; ++w) { const int x = wsum[w]; wsum[w] = run; run += x; }
  }
  __syncthreads();
  if (r < R) {
    if (a) {
      const int t = A.ck[p][blockIdx.x] + wsum[warp] + __popc(bal & ((1u << lane) - 1u));
      A.tidx[p][t] = r;
      A.tpos[p][r] = t;
    } else {
      A.tpos[p][r] = -1;
    }
  }
}

// embedding input s (primal rows) or s-dot (tangent rows) = column 0 of R~ / R~-dot
__global__ void emb_input_kernel(int Rmax, const int* __restrict__ Rdev, const int* __restrict__ row_idx,
                                 const int* __restrict__ tidx, const real* __restrict__ src, real* __restrict__ out) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= min(Rmax, *Rdev)) return;
  const int pr = tidx ? tidx[r] : r;
  out[r] = src[(size_t)row_idx[pr] * 4];
}

// embedding layer 0 (input width 1): y = tanh(s W0 + b0), h = y;  tangent: ydot = (1 - y^2) sdot W0
__global__ void emb_l0_kernel(int Rmax, const int* __restrict__ Rdev, int d, const real* __restrict__ s,
                              const real* __restrict__ W, const real* __restrict__ bias,
                              const real* __restrict__ Yprim, const int* __restrict__ rowmap, real* __restrict__ Y,
                              real* __restrict__ H) {
  const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long R = min(Rmax, *Rdev);
  if (e >= R * d) return;
  const long long r = e / d;
  const int c = (int)(e % d);
  const real z = s[r] * W[c];
  real y;
  if (Yprim == nullptr) {
    y = tanh_r(z + bias[c]);
  } else {
    const real yp = Yprim[(size_t)rowmap[r] * d + c];
    y = (real(1) - yp * yp) * z;
  }
  Y[e] = y;
  H[e] = y;
}

// X = R~^T G / N_m (4 x M) per atom and D = X^T X^< (Fig. 6); tangent: Xdot = (Rdot^T G + R~^T Gdot)/N_m,
// Ddot = Xdot^T X^< + X^T Xdot^<.  One CTA (8 warps) per atom: warp w takes the atom's rows w, w + 8, ... of
// every pair (lane l holds columns l, l + 32, l + 64, l + 96 of a row: one coalesced 8-byte load each); the
// tangent pass skips the rows with no tangent row (tpos < 0) in the same loop.  The 8 warps' partial sums
// are combined in a fixed order (deterministic).
constexpr int DESC_THREADS = 256, DESC_MC = 4;   // columns per lane: M <= 128
__global__ void __launch_bounds__(DESC_THREADS, 4)
desc_fwd_kernel(const __grid_constant__ Geo g, const __grid_constant__ PairPtrs pp, const __grid_constant__ FitPtrs fp,
                const real* __restrict__ em, const real* __restrict__ rdot, int tangent, real* __restrict__ X,
                real* __restrict__ Xd) {
  extern __shared__ real sm[];
  const int M = g.M, M2 = g.M2, Nm = g.Nm;
  real* xs = sm;            // [4][M]
  real* xds = sm + 4 * M;   // [4][M]
  real* rs = xds + 4 * M;   // [Nm][4] R~ rows of the atom (contiguous in em)
  real* rds = rs + 4 * Nm;  // [Nm][4] R~dot rows
  real* red = rds + 4 * Nm; // [8][4][128] per-warp partial sums of one column chunk
  const int atom = blockIdx.x;
  const int b = atom / g.Na, i = atom % g.Na;
  const int ti = g.types[i], k = g.tindex[i];
  const int e = b * g.ncnt[ti] + k;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int q = threadIdx.x; q < 4 * Nm; q += blockDim.x) {
    cp_async1(rs + q, em + (size_t)atom * Nm * 4 + q, true);
    if (tangent) cp_async1(rds + q, rdot + (size_t)atom * Nm * 4 + q, true);
  }
  cp_async_commit();
  cp_async_wait<0>();
  __syncthreads();
  const real inv = real(1) / g.Nm;
  real* xw = tangent ? xds : xs;
  real* xo = (tangent ? Xd : X) + (size_t)atom * 4 * M;
  for (int m0 = 0; m0 < M; m0 += 32 * DESC_MC) {   // column chunks of 128 (one pass for M <= 128)
    real acc[DESC_MC][4];
#pragma unroll
    for (int c = 0; c < DESC_MC; ++c) acc[c][0] = acc[c][1] = acc[c][2] = acc[c][3] = 0.0;
    for (int tj = 0; tj < g.nt; ++tj) {
      const int p = ti * g.nt + tj;
      const int r0 = pp.row_start[p][e], r1 = pp.row_start[p][e + 1];
      const real* er = rs + 4 * g.sec[tj];
      const real* ed = rds + 4 * g.sec[tj];
      constexpr int RS = DESC_THREADS / 32;
      if (!tangent) {   // two rows per iteration: 8 loads in flight per lane
        const real* Gp = pp.G[p];
        int r = r0 + warp;
        for (; r + RS < r1; r += 2 * RS) {
          real gv[2][DESC_MC];
#pragma unroll
          for (int u = 0; u < 2; ++u)
#pragma unroll
            for (int c = 0; c < DESC_MC; ++c) {
              const int m = m0 + lane + 32 * c;
              gv[u][c] = m < M ? Gp[(size_t)(r + u * RS) * M + m] : real(0);
            }
#pragma unroll
          for (int u = 0; u < 2; ++u) {
            const real* q = er + 4 * (r + u * RS - r0);
#pragma unroll
            for (int c = 0; c < DESC_MC; ++c)
#pragma unroll
              for (int a = 0; a < 4; ++a) acc[c][a] = fma(q[a], gv[u][c], acc[c][a]);
          }
        }
        if (r < r1) {
          const real* q = er + 4 * (r - r0);
          real gv[DESC_MC];
#pragma unroll
          for (int c = 0; c < DESC_MC; ++c) {
            const int m = m0 + lane + 32 * c;
            gv[c] = m < M ? Gp[(size_t)r * M + m] : real(0);
          }
#pragma unroll
          for (int c = 0; c < DESC_MC; ++c)
#pragma unroll
            for (int a = 0; a < 4; ++a) acc[c][a] = fma(q[a], gv[c], acc[c][a]);
        }
        continue;
      }
      // tangent: the warp's rows r0 + warp + RS*l (l = lane) are tested 32 at a time (one tpos load each, in
      // flight together); only the rows with a tangent row (R~dot, Gdot != 0) are visited
      for (int base = r0 + warp; base < r1; base += 32 * RS) {
        const int rl = base + RS * lane;
        const int tl = rl < r1 ? pp.tpos[p][rl] : -1;
        unsigned act = __ballot_sync(0xffffffffu, tl >= 0);
        while (act) {
          const int j = __ffs(act) - 1;
          act &= act - 1;
          const int r = base + RS * j;
          const int t = __shfl_sync(0xffffffffu, tl, j);
          const real* q = er + 4 * (r - r0);
          const real* qd = ed + 4 * (r - r0);
          real gv[DESC_MC], gd[DESC_MC];
#pragma unroll
          for (int c = 0; c < DESC_MC; ++c) {
            const int m = m0 + lane + 32 * c;
            gv[c] = m < M ? pp.G[p][(size_t)r * M + m] : real(0);
            gd[c] = m < M ? pp.Gt[p][(size_t)t * M + m] : real(0);
          }
#pragma unroll
          for (int c = 0; c < DESC_MC; ++c)
#pragma unroll
            for (int a = 0; a < 4; ++a) acc[c][a] = fma(qd[a], gv[c], fma(q[a], gd[c], acc[c][a]));
        }
      }
    }
#pragma unroll
    for (int c = 0; c < DESC_MC; ++c)
#pragma unroll
      for (int a = 0; a < 4; ++a) red[(warp * 4 + a) * (32 * DESC_MC) + lane + 32 * c] = acc[c][a];
    __syncthreads();
    for (int q = threadIdx.x; q < 4 * 32 * DESC_MC; q += blockDim.x) {
      const int a = q / (32 * DESC_MC), m = m0 + q % (32 * DESC_MC);
      if (m >= M) continue;
      real v = 0.0;
#pragma unroll
      for (int w = 0; w < DESC_THREADS / 32; ++w) v += red[(w * 4 + a) * (32 * DESC_MC) + q % (32 * DESC_MC)];
      xw[a * M + m] = v * inv;
      xo[a * M + m] = v * inv;
    }
    __syncthreads();
  }
  if (tangent) {
    const real* xp = X + (size_t)atom * 4 * M;
    for (int q = threadIdx.x; q < 4 * M; q += blockDim.x) xs[q] = xp[q];
  }
  __syncthreads();
  const long long row = (long long)b * g.ncnt[ti] + k;
  real* D = fp.D[ti] + (size_t)(tangent ? fp.F[ti] + row : row) * M * M2;
  for (int q = threadIdx.x; q < M * M2; q += blockDim.x) {
    const int m = q / M2, n = q % M2;
    real v;
    if (!tangent) {
      v = xs[m] * xs[n] + xs[M + m] * xs[M + n] + xs[2 * M + m] * xs[2 * M + n] + xs[3 * M + m] * xs[3 * M + n];
    } else {
      v = 0.0;
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) v += xds[kk * M + m] * xs[kk * M + n] + xs[kk * M + m] * xds[kk * M + n];
    }
    D[q] = v;
  }
}

// Eq. 4: dE/dX = X^< Dbar^T + [X Dbar into the first M^< columns].
//   Xbar = B(X, Dbar) + B(Xdot, Ddotbar) ; Xdotbar = B(X, Ddotbar)   (dual)
__global__ void desc_bwd_kernel(Geo g, FitPtrs fp, const real* __restrict__ X, const real* __restrict__ Xd, int dual,
                                real* __restrict__ Xb, real* __restrict__ Xdb) {
  extern __shared__ real sm[];
  const int M = g.M, M2 = g.M2;
  real* xs = sm;
  real* xds = xs + 4 * M;
  real* db = xds + 4 * M;
  real* ddb = db + M * (M2 + 1);
  const int atom = blockIdx.x;
  const int b = atom / g.Na, i = atom % g.Na;
  const int ti = g.types[i], k = g.tindex[i];
  const long long row = (long long)b * g.ncnt[ti] + k;
  const real* Dbp = fp.Db[ti] + (size_t)row * M * M2;
  const real* Ddbp = fp.Db[ti] + (size_t)(fp.F[ti] + row) * M * M2;
  for (int e = threadIdx.x; e < 4 * M; e += blockDim.x) {
    xs[e] = X[(size_t)atom * 4 * M + e];
    if (dual) xds[e] = Xd[(size_t)atom * 4 * M + e];
  }
  for (int e = threadIdx.x; e < M * M2; e += blockDim.x) {
    const int ep = (e / M2) * (M2 + 1) + e % M2;  // row stride M2 + 1: conflict-free in both loops below
    db[ep] = Dbp[e];
    if (dual) ddb[ep] = Ddbp[e];
  }
  __syncthreads();
  for (int e = threadIdx.x; e < 4 * M; e += blockDim.x) {
    const int kk = e / M, p = e % M;
    const real* x = xs + kk * M;
    real a = 0.0, ad = 0.0;
    for (int n = 0; n < M2; ++n) a = fma(db[p * (M2 + 1) + n], x[n], a);
    if (p < M2)
      for (int m = 0; m < M; ++m) a = fma(db[m * (M2 + 1) + p], x[m], a);
    if (dual) {
      const real* xd = xds + kk * M;
      for (int n = 0; n < M2; ++n) { a = fma(ddb[p * (M2 + 1) + n], xd[n], a); ad = fma(ddb[p * (M2 + 1) + n], x[n], ad); }
      if (p < M2)
        for (int m = 0; m < M; ++m) { a = fma(ddb[m * (M2 + 1) + p], xd[m], a); ad = fma(ddb[m * (M2 + 1) + p], x[m], ad); }
      Xdb[(size_t)atom * 4 * M + e] = ad;
    }
    Xb[(size_t)atom * 4 * M + e] = a;
  }
}

// Eq. 4 per atom (as desc_bwd_kernel), then the fused embedding backward's per-row seeds:
//   Gbar_r = (R~_r Xbar + R~dot_r Xdotbar) / N_m        (primal rows; R~dot = 0 off the tangent rows)
//   Gdotbar_t = R~_r Xdotbar / N_m                      (tangent rows t = tpos[r], into hdotbar_{L-1})
//   dR_r = G_r Xbar^T / N_m                             (forces: the R~ adjoint less sbar e_0)
// One CTA (8 warps) per centre atom; the atom's R~ (and R~dot) rows are contiguous and staged once.
struct SeedOut {
  real* gbar[NP];
  real* hbt[NP];
  real* dr[NP];
};
template <bool dual, bool force, bool sel>
__global__ void __launch_bounds__(256, dual ? 2 : 4)
desc_bwd_seed_kernel(const __grid_constant__ Geo g, const __grid_constant__ FitPtrs fp,
                     const __grid_constant__ PairPtrs pp, const __grid_constant__ SeedOut so,
                     const real* __restrict__ X, const real* __restrict__ Xd, const real* __restrict__ em,
                     const real* __restrict__ rdot, real* __restrict__ Xb, real* __restrict__ Xdb) {
  extern __shared__ real sm[];
  const int M = g.M, M2 = g.M2, Nm = g.Nm;
  real* xs = sm;               // [4][M]
  real* xds = xs + 4 * M;      // [4][M]
  real* db = xds + 4 * M;      // [M][M2 + 1]
  real* ddb = db + M * (M2 + 1);  // [M][M2 + 1]
  real* xbs = ddb + M * (M2 + 1);  // [4][M]  Xbar
  real* xdbs = xbs + 4 * M;    // [4][M]  Xdotbar
  real* rs = xdbs + 4 * M;     // [Nm][4] R~ rows of the atom
  real* rds = rs + 4 * Nm;     // [Nm][4] R~dot rows
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int atom = blockIdx.x;
  const int b = atom / g.Na, i = atom % g.Na;
  const int ti = g.types[i], k = g.tindex[i];
  const long long row = (long long)b * g.ncnt[ti] + k;
  const real* Dbp = fp.Db[ti] + (size_t)row * M * M2;
  const real* Ddbp = fp.Db[ti] + (size_t)(fp.F[ti] + row) * M * M2;
  // staging with cp.async: every copy of the CTA in flight at once (no per-element load -> store latency)
  for (int e = tid; e < 4 * M; e += blockDim.x) {
    cp_async1(xs + e, X + (size_t)atom * 4 * M + e, true);
    if (dual) cp_async1(xds + e, Xd + (size_t)atom * 4 * M + e, true);
  }
  for (int e = tid; e < M * M2; e += blockDim.x) {
    const int ep = (e / M2) * (M2 + 1) + e % M2;  // row stride M2 + 1: conflict-free in both loops below
    cp_async1(db + ep, Dbp + e, true);
    if (dual) cp_async1(ddb + ep, Ddbp + e, true);
  }
  for (int e = tid; e < 4 * Nm; e += blockDim.x) {
    cp_async1(rs + e, em + (size_t)atom * Nm * 4 + e, true);
    if (dual) cp_async1(rds + e, rdot + (size_t)atom * Nm * 4 + e, true);
  }
  cp_async_commit();
  cp_async_wait<0>();
  __syncthreads();
  // Eq. 4 in two phases so no thread runs a long serial chain: (A) the M-term sums of the first M^<
  // columns, T[kk][p] = sum_m Dbar[m][p] x[kk][m] (p < M^<), by 4 threads each (M/4 terms, combined by
  // shuffles in a fixed order); (B) the M^<-term sums of every (kk, p) plus T.  ta/td hold T in xbs/xdbs.
  {
    const int no = 4 * M2, part = tid & 3, no8 = (no + 7) & ~7;   // whole warps run the shuffles
    for (int o = tid >> 2; o < no8; o += blockDim.x >> 2) {
      const bool valid = o < no;
      const int kk = valid ? o / M2 : 0, p = valid ? o % M2 : 0;
      const real* x = xs + kk * M;
      const real* xd = xds + kk * M;
      real a = 0.0, ad = 0.0;
      for (int m = part; valid && m < M; m += 4) {
        a = fma(db[m * (M2 + 1) + p], x[m], a);
        if (dual) {
          a = fma(ddb[m * (M2 + 1) + p], xd[m], a);
          ad = fma(ddb[m * (M2 + 1) + p], x[m], ad);
        }
      }
      a += __shfl_xor_sync(0xffffffffu, a, 1);
      a += __shfl_xor_sync(0xffffffffu, a, 2);
      ad += __shfl_xor_sync(0xffffffffu, ad, 1);
      ad += __shfl_xor_sync(0xffffffffu, ad, 2);
      if (part == 0 && valid) {
        xbs[kk * M + p] = a;
        if (dual) xdbs[kk * M + p] = ad;
      }
    }
  }
  __syncthreads();
  for (int e = tid; e < 4 * M; e += blockDim.x) {
    const int kk = e / M, p = e % M;
    const real* x = xs + kk * M;
    real a = p < M2 ? xbs[e] : real(0), ad = (dual && p < M2) ? xdbs[e] : real(0);
    for (int n = 0; n < M2; ++n) a = fma(db[p * (M2 + 1) + n], x[n], a);
    if (dual) {
      const real* xd = xds + kk * M;
      for (int n = 0; n < M2; ++n) { a = fma(ddb[p * (M2 + 1) + n], xd[n], a); ad = fma(ddb[p * (M2 + 1) + n], x[n], ad); }
    }
    Xb[(size_t)atom * 4 * M + e] = a;
    if (dual) Xdb[(size_t)atom * 4 * M + e] = ad;
  }
  __syncthreads();   // every T read before the final values overwrite xbs / xdbs
  for (int e = tid; e < 4 * M; e += blockDim.x) {
    xbs[e] = Xb[(size_t)atom * 4 * M + e];
    if (dual) xdbs[e] = Xdb[(size_t)atom * 4 * M + e];
  }
  __syncthreads();
  const real inv = real(1) / Nm;
  const int e0 = b * g.ncnt[ti] + k;
  // per row: Gbar = (R~ Xbar [+ R~dot Xdotbar]) / N_m, [Hdotbar = R~ Xdotbar / N_m on tangent rows],
  // [dR = G Xbar^T / N_m]; the lane's Xbar (Xdotbar) columns m = m0 + lane + 32 u stay in registers
  for (int m0 = 0; m0 < M; m0 += 128) {
    real xb[4][4], xdb[4][4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int m = m0 + lane + 32 * u;
#pragma unroll
      for (int a = 0; a < 4; ++a) {
        xb[u][a] = m < M ? xbs[a * M + m] : real(0);
        xdb[u][a] = (dual && m < M) ? xdbs[a * M + m] : real(0);
      }
    }
    for (int tj = 0; tj < g.nt; ++tj) {
      const int p = ti * g.nt + tj;
      const int r0 = pp.row_start[p][e0], nr = pp.row_start[p][e0 + 1] - r0;
      const int* __restrict__ tpos = pp.tpos[p];
      real* __restrict__ gbar = so.gbar[p];
      real* __restrict__ hbt = so.hbt[p];
      real* __restrict__ dr = so.dr[p];
      const real* __restrict__ Gp = pp.G[p];
      const real* rsj = rs + g.sec[tj] * 4;
      const real* rdsj = rds + g.sec[tj] * 4;
      auto row_body = [&](int s_, int t) {
        const int r = r0 + s_;
        const real* q = rsj + s_ * 4;
        const real q0 = q[0], q1 = q[1], q2 = q[2], q3 = q[3];
        real d0 = 0.0, d1 = 0.0, d2 = 0.0, d3 = 0.0;
        if (dual && t >= 0) { const real* qd = rdsj + s_ * 4; d0 = qd[0]; d1 = qd[1]; d2 = qd[2]; d3 = qd[3]; }
        real gv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int m = m0 + lane + 32 * u;
          gv[u] = (force && m < M) ? Gp[(size_t)r * M + m] : real(0);
        }
        real pk0 = 0.0, pk1 = 0.0, pk2 = 0.0, pk3 = 0.0;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int m = m0 + lane + 32 * u;
          if (m >= M) continue;
          real v = q0 * xb[u][0] + q1 * xb[u][1] + q2 * xb[u][2] + q3 * xb[u][3];
          if (dual && t >= 0) {
            v += d0 * xdb[u][0] + d1 * xdb[u][1] + d2 * xdb[u][2] + d3 * xdb[u][3];
            hbt[(size_t)t * M + m] = (q0 * xdb[u][0] + q1 * xdb[u][1] + q2 * xdb[u][2] + q3 * xdb[u][3]) * inv;
          }
          gbar[(size_t)r * M + m] = v * inv;
          if (force) {
            pk0 = fma(gv[u], xb[u][0], pk0);
            pk1 = fma(gv[u], xb[u][1], pk1);
            pk2 = fma(gv[u], xb[u][2], pk2);
            pk3 = fma(gv[u], xb[u][3], pk3);
          }
        }
        if (force) {
          for (int o = 16; o > 0; o >>= 1) {
            pk0 += __shfl_xor_sync(0xffffffffu, pk0, o);
            pk1 += __shfl_xor_sync(0xffffffffu, pk1, o);
            pk2 += __shfl_xor_sync(0xffffffffu, pk2, o);
            pk3 += __shfl_xor_sync(0xffffffffu, pk3, o);
          }
          if (lane < 4) {
            const real pv = lane == 0 ? pk0 : lane == 1 ? pk1 : lane == 2 ? pk2 : pk3;
            if (m0 == 0) dr[(size_t)r * 4 + lane] = pv * inv;
            else dr[(size_t)r * 4 + lane] += pv * inv;
          }
        }
      };
      constexpr int RS = 8;   // warps
      if (sel || dual) {
        // rows tested 32 at a time per warp (tpos loads in flight together); MODE_FORCE_SEL visits only the
        // rows touching the selected atoms, the dual pass every row with its tangent row (or -1)
        for (int base = warp; base < nr; base += 32 * RS) {
          const int sl = base + RS * lane;
          const int tl = sl < nr ? tpos[r0 + sl] : -1;
          unsigned act = __ballot_sync(0xffffffffu, sel ? tl >= 0 : sl < nr);
          while (act) {
            const int j = __ffs(act) - 1;
            act &= act - 1;
            row_body(base + RS * j, __shfl_sync(0xffffffffu, tl, j));
          }
        }
      } else {
        for (int s_ = warp; s_ < nr; s_ += RS) row_body(s_, -1);
      }
    }
  }
}

// adjoint of G (and Gdot) per embedding row from the atom's Xbar (and Xdotbar):
//   Gbar = (R~ Xbar + Rdot Xdotbar)/N_m ; Gdotbar = R~ Xdotbar / N_m
// fused with the last layer's activation adjoint (G = skip + y, no timestep):
//   zbar = (1 - y^2) Gbar - 2 y ydot Gdotbar ; zdotbar = (1 - y^2) Gdotbar
__global__ void emb_seed_kernel(int Rmax, const int* __restrict__ Rdev, int M, int Nm,
                                const int* __restrict__ row_idx, const int* __restrict__ tpos,
                                const real* __restrict__ em, const real* __restrict__ rdot,
                                const real* __restrict__ Xb, const real* __restrict__ Xdb, int dual,
                                const real* __restrict__ Y, const real* __restrict__ Yt, real* __restrict__ Hb,
                                real* __restrict__ Zb, real* __restrict__ Hbt, real* __restrict__ Zbt) {
  const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long R = min(Rmax, *Rdev);
  if (e >= R * M) return;
  const long long r = e / M;
  const int m = (int)(e % M);
  const size_t idx = (size_t)row_idx[r];
  const size_t atom = idx / Nm;
  const real* xb = Xb + atom * 4 * M;
  const real* rr = em + idx * 4;
  real a = rr[0] * xb[m] + rr[1] * xb[M + m] + rr[2] * xb[2 * M + m] + rr[3] * xb[3 * M + m];
  const real inv = real(1) / Nm;
  const size_t o = (size_t)r * M + m;
  const real y = Y[o];
  const real t = real(1) - y * y;
  const int tr = dual ? tpos[r] : -1;
  if (tr >= 0) {
    const real* xdb = Xdb + atom * 4 * M;
    const real* rd = rdot + idx * 4;
    a += rd[0] * xdb[m] + rd[1] * xdb[M + m] + rd[2] * xdb[2 * M + m] + rd[3] * xdb[3 * M + m];
    const real ad = (rr[0] * xdb[m] + rr[1] * xdb[M + m] + rr[2] * xdb[2 * M + m] + rr[3] * xdb[3 * M + m]) * inv;
    const size_t od = (size_t)tr * M + m;
    Hbt[od] = ad;
    Zbt[od] = t * ad;
    a *= inv;
    Hb[o] = a;
    Zb[o] = t * a - real(2) * y * Yt[od] * ad;
  } else {
    a *= inv;
    Hb[o] = a;
    Zb[o] = t * a;
  }
}

// Same as emb_seed_kernel, one CTA per centre atom for all its rows of every pair: the atom's Xbar
// (and Xdotbar) are staged once in SMEM instead of being re-read for every (row, m).
struct SeedPtrs {
  const real* Y[NP];
  const real* Yt[NP];
  real* Hb[NP];
  real* Zb[NP];
  real* Hbt[NP];
  real* Zbt[NP];
};
__global__ void __launch_bounds__(128)
emb_seed_atom_kernel(Geo g, PairPtrs pp, SeedPtrs sp, const real* __restrict__ em, const real* __restrict__ rdot,
                     const real* __restrict__ Xb, const real* __restrict__ Xdb, int dual) {
  extern __shared__ real sm[];
  const int M = g.M;
  real* xb = sm;
  real* xdb = sm + 4 * M;
  const int atom = blockIdx.x;
  const int b = atom / g.Na, i = atom % g.Na;
  const int ti = g.types[i], k = g.tindex[i];
  const int e = b * g.ncnt[ti] + k;
  for (int q = threadIdx.x; q < 4 * M; q += blockDim.x) {
    xb[q] = Xb[(size_t)atom * 4 * M + q];
    if (dual) xdb[q] = Xdb[(size_t)atom * 4 * M + q];
  }
  __syncthreads();
  const real inv = real(1) / g.Nm;
  for (int tj = 0; tj < g.nt; ++tj) {
    const int p = ti * g.nt + tj;
    const int r0 = pp.row_start[p][e], r1 = pp.row_start[p][e + 1];
    const int n = (r1 - r0) * M;
    for (int q = threadIdx.x; q < n; q += blockDim.x) {
      const int s = q / M, m = q % M;
      const int r = r0 + s;
      const size_t idx = (size_t)atom * g.Nm + g.sec[tj] + s;
      const real* rr = em + idx * 4;
      real a = rr[0] * xb[m] + rr[1] * xb[M + m] + rr[2] * xb[2 * M + m] + rr[3] * xb[3 * M + m];
      const size_t o = (size_t)r * M + m;
      const real y = sp.Y[p][o];
      const real t = real(1) - y * y;
      const int tr = dual ? pp.tpos[p][r] : -1;
      if (tr >= 0) {
        const real* rd = rdot + idx * 4;
        a += rd[0] * xdb[m] + rd[1] * xdb[M + m] + rd[2] * xdb[2 * M + m] + rd[3] * xdb[3 * M + m];
        const real ad = (rr[0] * xdb[m] + rr[1] * xdb[M + m] + rr[2] * xdb[2 * M + m] + rr[3] * xdb[3 * M + m]) * inv;
        const size_t od = (size_t)tr * M + m;
        sp.Hbt[p][od] = ad;
        sp.Zbt[p][od] = t * ad;
        a *= inv;
        sp.Hb[p][o] = a;
        sp.Zb[p][o] = t * a - real(2) * y * sp.Yt[p][od] * ad;
      } else {
        a *= inv;
        sp.Hb[p][o] = a;
        sp.Zb[p][o] = t * a;
      }
    }
  }
}

// prod_force (per-layer embedding path): dE/dR~_row = G Xbar^T / N_m + sbar e_0 ; f = dE/dd = (dE/dR~) J per
// slot into frow (the forces / virials are gathered by force_gather_kernel).  One CTA (4 warps) per atom.
__global__ void __launch_bounds__(128)
prod_force_kernel(Geo g, PairPtrs pp, const real* __restrict__ Xb, const real* __restrict__ jac,
                  const int* __restrict__ nl_j, real* __restrict__ frow) {
  const int atom = blockIdx.x;
  const int b = atom / g.Na, i = atom % g.Na;
  const int ti = g.types[i], k = g.tindex[i];
  const int e = b * g.ncnt[ti] + k;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int M = g.M;
  const real* xb = Xb + (size_t)atom * 4 * M;
  const real inv = real(1) / g.Nm;
  for (int slot = warp; slot < g.Nm; slot += 4) {
    const size_t idx = (size_t)atom * g.Nm + slot;
    if (nl_j[idx] < 0) continue;
    int tj = 0;
    while (slot >= g.sec[tj + 1]) ++tj;
    const int p = ti * g.nt + tj;
    const long long r = pp.row_start[p][e] + (slot - g.sec[tj]);
    const real* gr = pp.G[p] + (size_t)r * M;
    real a0 = 0, a1 = 0, a2 = 0, a3 = 0;
    for (int m = lane; m < M; m += 32) {
      const real gv = gr[m];
      a0 = fma(gv, xb[m], a0); a1 = fma(gv, xb[M + m], a1); a2 = fma(gv, xb[2 * M + m], a2); a3 = fma(gv, xb[3 * M + m], a3);
    }
    for (int o = 16; o > 0; o >>= 1) {
      a0 += __shfl_xor_sync(0xffffffffu, a0, o);
      a1 += __shfl_xor_sync(0xffffffffu, a1, o);
      a2 += __shfl_xor_sync(0xffffffffu, a2, o);
      a3 += __shfl_xor_sync(0xffffffffu, a3, o);
    }
    if (lane < 3) {
      const real rb0 = a0 * inv + pp.sbar[p][r], rb1 = a1 * inv, rb2 = a2 * inv, rb3 = a3 * inv;
      const real* J = jac + idx * 12;
      frow[idx * 3 + lane] = rb0 * J[lane] + rb1 * J[3 + lane] + rb2 * J[6 + lane] + rb3 * J[9 + lane];
    }
  }
}

// ---------------------------------------------------------------------------------------------
// Atomics-free force / virial scatter.  Per slot (atom i, neighbour j, d = x_j + S - x_i) the reverse pass
// stores f = dE/dd; F = -dE/dx gives F_i += f and F_j -= f, W_i -= d (x) f.  The reverse
// neighbour map lists, for every atom j of an image, the slots whose neighbour is j in slot order, so every
// force is a fixed-order sum (bit-reproducible run to run, graph or eager).
// ---------------------------------------------------------------------------------------------
// rev_cnt[b][i][j] = number of slots of atom i with neighbour j (order-free integer counts)
__global__ void __launch_bounds__(256) rev_count_kernel(int nb, int Na, int Nm, const int* __restrict__ nl_j,
                                                        int* __restrict__ cnt) {
  const int a = blockIdx.x * 8 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (a >= nb * Na) return;
  int* row = cnt + (size_t)a * Na;
  for (int s0 = lane; s0 < Nm; s0 += 32) {
    const int j = nl_j[(size_t)a * Nm + s0];
    if (j >= 0) atomicAdd(row + j, 1);
  }
}
// per (image, j): exclusive prefix over the centre atoms i in place (cnt -> first position of atom i's
// entries inside bucket j) and the bucket size
__global__ void rev_prefix_kernel(int nb, int Na, int* __restrict__ cnt, int* __restrict__ tot) {
  const int q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= nb * Na) return;
  const int b = q / Na, j = q % Na;
  int run = 0;
  for (int i = 0; i < Na; ++i) {
    int* c = cnt + ((size_t)b * Na + i) * Na + j;
    const int v = *c;
    *c = run;
    run += v;
  }
  tot[q] = run;
}
// exclusive scan of the bucket sizes (one CTA, fixed order) -> rev_off[0 .. nb*Na]
__global__ void __launch_bounds__(1024) rev_scan_kernel(int n, int* __restrict__ off) {
  __shared__ int wsum[32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int per = (n + 1023) / 1024;
  const int a0 = min(n, (int)threadIdx.x * per), a1 = min(n, a0 + per);
  int local = 0;
  for (int e = a0; e < a1; ++e) local += off[e];
  int x = local;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[warp] = x;
  __syncthreads();
  if (warp == 0) {
    int w = wsum[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= o) w += y;
    }
    wsum[lane] = w;
  }
  __syncthreads();
  int run = x - local + (warp > 0 ? wsum[warp - 1] : 0);
  for (int e = a0; e < a1; ++e) {
    const int c = off[e];
    off[e] = run;
    run += c;
  }
  if (threadIdx.x == 1023) off[n] = wsum[31];
}
// fill: one warp per centre atom walks its slots in order; lanes with the same neighbour j inside a chunk
// are ranked by lane (match_any), and the atom's own cursor row of rev_cnt (touched by this warp only)
// carries the count across chunks -> every bucket in (i, slot) order, deterministic
__global__ void __launch_bounds__(256) rev_fill_kernel(int nb, int Na, int Nm, const int* __restrict__ nl_j,
                                                       int* __restrict__ cnt, const int* __restrict__ off,
                                                       int* __restrict__ idx) {
  const int a = blockIdx.x * 8 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (a >= nb * Na) return;
  const int b = a / Na;
  int* cur = cnt + (size_t)a * Na;
  for (int s0 = 0; s0 < Nm; s0 += 32) {
    const int sl = s0 + lane;
    const int j = sl < Nm ? nl_j[(size_t)a * Nm + sl] : -1;
    const unsigned grp = __match_any_sync(0xffffffffu, j);
    const int rk = __popc(grp & ((1u << lane) - 1u));
    int base = 0;
    if (j >= 0) base = off[(size_t)b * Na + j] + cur[j];
    __syncwarp();
    if (j >= 0) {
      idx[base + rk] = (int)((size_t)a * Nm + sl);
      if (rk == 0) cur[j] += __popc(grp);
    }
    __syncwarp();
  }
}

fekf_status build_reverse(Ctx& c, int nb, cudaStream_t s) {
  const int na = c.Na, n = nb * na;
  int* cnt = c.rev_cnt.as<int>();
  int* off = c.rev_off.as<int>();
  FEKF_CHECK_CUDA(cudaMemsetAsync(cnt, 0, sizeof(int) * (size_t)n * na, s));
  rev_count_kernel<<<cdiv(n, 8), 256, 0, s>>>(nb, na, c.Nm, c.nl_j.as<int>(), cnt);
  FEKF_LAUNCH_CHECK();
  rev_prefix_kernel<<<cdiv(n, 128), 128, 0, s>>>(nb, na, cnt, off);
  FEKF_LAUNCH_CHECK();
  rev_scan_kernel<<<1, 1024, 0, s>>>(n, off);
  FEKF_LAUNCH_CHECK();
  rev_fill_kernel<<<cdiv(n, 8), 256, 0, s>>>(nb, na, c.Nm, c.nl_j.as<int>(), cnt, off, c.rev_idx.as<int>());
  FEKF_LAUNCH_CHECK();
  count_launch(4);
  return FEKF_OK;
}

// F_i = sum_{own slots} f - sum_{slots with neighbour i} f ;  W_i = - sum_{own slots} d (x) f.
// One warp per atom (all atoms, or the listed ones of every image); lane-strided sums combined by a fixed
// butterfly: deterministic.
__global__ void __launch_bounds__(256) force_gather_kernel(int nb, int Na, int Nm, const int* __restrict__ sel,
                                                           int n_sel, const int* __restrict__ nl_j,
                                                           const real* __restrict__ rij,
                                                           const real* __restrict__ frow,
                                                           const int* __restrict__ off, const int* __restrict__ idx,
                                                           double* __restrict__ force, double* __restrict__ vatom) {
  const int w = blockIdx.x * 8 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  const int nw = sel ? nb * n_sel : nb * Na;
  if (w >= nw) return;
  const int a = sel ? (w / n_sel) * Na + sel[w % n_sel] : w;
  real v[12];
#pragma unroll
  for (int q = 0; q < 12; ++q) v[q] = 0.0;
  for (int sl = lane; sl < Nm; sl += 32) {
    const size_t e = (size_t)a * Nm + sl;
    if (nl_j[e] < 0) continue;
    const real f0 = frow[e * 3], f1 = frow[e * 3 + 1], f2 = frow[e * 3 + 2];
    const real d0 = rij[e * 3], d1 = rij[e * 3 + 1], d2 = rij[e * 3 + 2];
    v[0] += f0; v[1] += f1; v[2] += f2;
    v[3] -= d0 * f0; v[4] -= d0 * f1; v[5] -= d0 * f2;
    v[6] -= d1 * f0; v[7] -= d1 * f1; v[8] -= d1 * f2;
    v[9] -= d2 * f0; v[10] -= d2 * f1; v[11] -= d2 * f2;
  }
  for (int q = off[a] + lane; q < off[a + 1]; q += 32) {
    const size_t e = (size_t)idx[q];
    v[0] -= frow[e * 3];
    v[1] -= frow[e * 3 + 1];
    v[2] -= frow[e * 3 + 2];
  }
#pragma unroll
  for (int q = 0; q < 12; ++q)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v[q] += __shfl_xor_sync(0xffffffffu, v[q], o);
  if (lane < 3) force[(size_t)a * 3 + lane] = lane == 0 ? v[0] : (lane == 1 ? v[1] : v[2]);
  else if (lane < 12) {
    real x = 0.0;
#pragma unroll
    for (int q = 3; q < 12; ++q) if (lane == q) x = v[q];
    vatom[(size_t)a * 9 + lane - 3] = x;
  }
}

// per-image virial = sum of the atoms' contributions in atom order (deterministic)
__global__ void virial_reduce_kernel(const double* __restrict__ vatom, int Na, double* __restrict__ virial) {
  const int b = blockIdx.x, q = threadIdx.x;
  if (q >= 9) return;
  double a = 0.0;
  for (int i = 0; i < Na; ++i) a += vatom[((size_t)b * Na + i) * 9 + q];
  virial[(size_t)b * 9 + q] = a;
}

// E_i = h_F W_out + b_out (primal rows), Edot_i = hdot_F W_out (tangent rows); one warp per row; every type
// in one launch (blockIdx.y = type)
struct OutArgs {
  long long rows[MT], F[MT];
  const real* H[MT];
  const real* W[MT];
  const real* b[MT];
  real* out[MT];
  const real* ebar[MT];
  real* Hb[MT];
  int h;
};
__global__ void fit_out_kernel(const __grid_constant__ OutArgs A) {
  const int t = blockIdx.y;
  const long long r = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31, h = A.h;
  if (r >= A.rows[t]) return;
  const real* __restrict__ H = A.H[t];
  const real* __restrict__ W = A.W[t];
  real a = 0.0;
  for (int c = lane; c < h; c += 32) a = fma(H[(size_t)r * h + c], W[c], a);
  for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
  if (lane == 0) A.out[t][r] = a + (r < A.F[t] ? A.b[t][0] : real(0));
}
// adjoint of h_F from the output seeds: Hbar = ebar (x) W_out
__global__ void fit_out_bwd_kernel(const __grid_constant__ OutArgs A) {
  const int t = blockIdx.y;
  const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const int h = A.h;
  if (e >= A.rows[t] * h) return;
  A.Hb[t][e] = A.ebar[t][e / h] * A.W[t][e % h];
}

// per-atom energies back into [nb][Na] and E_b = sum_i E_i, fixed order
__global__ void energy_scatter_kernel(Geo g, FitPtrs fp, double* __restrict__ eatom, double* __restrict__ etot) {
  const int b = blockIdx.x;
  for (int i = threadIdx.x; i < g.Na; i += blockDim.x) {
    const int t = g.types[i];
    eatom[(size_t)b * g.Na + i] = fp.eout[t][(size_t)b * g.ncnt[t] + g.tindex[i]];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double a = 0.0;
    for (int i = 0; i < g.Na; ++i) a += eatom[(size_t)b * g.Na + i];
    etot[b] = a;
  }
}

// energy update errors (Alg. 1 lines 3-6): e_b = (Y_b - E_b)/N_a, flip when E_b >= Y_b; seeds s_b/N_a
// (any local batch: the seed of row r is formed from its image's energy directly, no per-image staging)
__global__ void energy_error_kernel(Geo g, FitPtrs fp, const double* __restrict__ etot, const double* __restrict__ label,
                                    double seed_scale, double* __restrict__ abs_sum) {
  if (threadIdx.x == 0) {
    double a = 0.0;
    for (int b = 0; b < g.nb; ++b) a += fabs((label[b] - etot[b]) / g.Na);
    *abs_sum = a;
  }
  for (int t = 0; t < g.nt; ++t) {
    const long long F = (long long)g.nb * g.ncnt[t];
    for (long long r = threadIdx.x; r < F; r += blockDim.x) {
      const long long b = r / g.ncnt[t];
      fp.ebar[t][r] = (real)((etot[b] >= label[b] ? -1.0 : 1.0) * seed_scale / g.Na);
    }
  }
}

// force update errors on the selected atoms (Alg. 1 lines 3-6 applied to force components):
// e = F_label - F_pred, flip when F_pred >= F_label; v[b][a] accumulates the signs (tangent direction);
// seeds: Ebar = 0, Edotbar = -1/(N_a n_sel 3) because sum s F = -Edot.
__global__ void __launch_bounds__(1024) force_error_kernel(Geo g, const double* __restrict__ force,
                                                           const double* __restrict__ label,
                                                           const int* __restrict__ atom_idx, int n_sel, double seed,
                                                           real* __restrict__ v, FitPtrs fp,
                                                           double* __restrict__ abs_sum) {
  __shared__ double red[1024];
  for (long long e = threadIdx.x; e < (long long)g.nb * g.Na * 3; e += blockDim.x) v[e] = 0.0;
  __syncthreads();
  // one thread per (image, selected atom, component); the signs are integers, so their atomic sums
  // (duplicate atoms in the list) are exact and order-free; |e| is reduced in a fixed tree
  double a = 0.0;
  const int n = g.nb * n_sel * 3;
  for (int e = threadIdx.x; e < n; e += blockDim.x) {
    const int b = e / (n_sel * 3), q = (e / 3) % n_sel, al = e % 3;
    const size_t o = ((size_t)b * g.Na + atom_idx[q]) * 3 + al;
    const double fpred = force[o], fl = label[o];
    a += fabs(fl - fpred);
    atomicAdd(v + o, fpred >= fl ? real(-1) : real(1));
  }
  red[threadIdx.x] = a;
  __syncthreads();
  for (int w = blockDim.x / 2; w > 0; w >>= 1) {
    if ((int)threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
    __syncthreads();
  }
  if (threadIdx.x == 0) *abs_sum = red[0];
  for (int t = 0; t < g.nt; ++t) {
    const long long F = (long long)g.nb * g.ncnt[t];
    for (long long r = threadIdx.x; r < 2 * F; r += blockDim.x) fp.ebar[t][r] = r < F ? real(0) : (real)seed;
  }
}

// tangent of R~ along v: ddot = v_j - v_i ; Rdot = J ddot
__global__ void tangent_env_kernel(const real* __restrict__ jac, const int* __restrict__ nl_j, const real* __restrict__ v,
                                   int Na, int Nm, long long nslots, real* __restrict__ rdot) {
  const long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= nslots) return;
  const int j = nl_j[idx];
  real* o = rdot + idx * 4;
  if (j < 0) { o[0] = o[1] = o[2] = o[3] = 0.0; return; }
  const long long bi = idx / Nm;
  const int b = (int)(bi / Na);
  const real* vi = v + bi * 3;
  const real* vj = v + ((size_t)b * Na + j) * 3;
  const real dd[3] = {vj[0] - vi[0], vj[1] - vi[1], vj[2] - vi[2]};
  const real* J = jac + idx * 12;
#pragma unroll
  for (int k = 0; k < 4; ++k) o[k] = J[3 * k] * dd[0] + J[3 * k + 1] * dd[1] + J[3 * k + 2] * dd[2];
}

__global__ void fill_kernel(real* p, long long n, real v) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = v;
}

// =================================================================================================
// host orchestration
// =================================================================================================
static PairPtrs make_pp(Ctx& c) {
  PairPtrs pp{};
  for (size_t p = 0; p < c.pairs.size(); ++p) {
    PairNet& P = c.pairs[p];
    pp.G[p] = P.H.back().as<real>();
    pp.Gt[p] = P.Ht.back().as<real>();
    pp.row_start[p] = P.row_start.as<int>();
    pp.row_idx[p] = P.row_idx.as<int>();
    pp.tpos[p] = P.tpos.as<int>();
    pp.sbar[p] = P.sbar.as<real>();
  }
  return pp;
}
static FitPtrs make_fp(Ctx& c, int nb) {
  FitPtrs fp{};
  for (int t = 0; t < c.nt; ++t) {
    fp.D[t] = c.fits[t].D.as<real>();
    fp.Db[t] = c.fits[t].Db.as<real>();
    fp.eout[t] = c.fits[t].eout.as<real>();
    fp.ebar[t] = c.fits[t].ebar.as<real>();
    fp.F[t] = fit_rows(c, t, nb);
  }
  return fp;
}

// Row compaction for all pairs at once, three launches (blockIdx.y = pair): per-atom valid-slot
// counts (a warp per centre atom, ballots over its sorted section), one CTA per pair scanning the counts
// into row_start (fixed order: deterministic row order), then the row -> slot scatter (a warp per atom).
struct RowsArgs {
  int ti[NP], tj[NP];
  int* row_start[NP];
  int* row_idx[NP];
  int* cnt;
};
__device__ __forceinline__ size_t rows_base(const Geo& g, int ti, int tj, int e) {
  const int b = e / g.ncnt[ti], k = e % g.ncnt[ti];
  const int i = g.atoms[g.atoms_off[ti] + k];
  return ((size_t)b * g.Na + i) * g.Nm + g.sec[tj];
}
__global__ void __launch_bounds__(256) rows_count_kernel(Geo g, RowsArgs ra, const int* __restrict__ nl_j) {
  const int p = blockIdx.y, ti = ra.ti[p], tj = ra.tj[p];
  const int e = blockIdx.x * 8 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (e >= g.nb * g.ncnt[ti]) return;
  const size_t base = rows_base(g, ti, tj, e);
  const int sel = g.sel[tj];
  int c = 0;
  for (int s0 = 0; s0 < sel; s0 += 32) c += __popc(__ballot_sync(0xffffffffu, s0 + lane < sel && nl_j[base + s0 + lane] >= 0));
  if (lane == 0) ra.row_start[p][e] = c;
}
__global__ void __launch_bounds__(1024) rows_scan_kernel(Geo g, RowsArgs ra) {
  __shared__ int wsum[32];
  const int p = blockIdx.x, E = g.nb * g.ncnt[ra.ti[p]];
  int* rs = ra.row_start[p];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int per = (E + 1023) / 1024;
  const int a0 = min(E, (int)threadIdx.x * per), a1 = min(E, a0 + per);
  int local = 0;
  for (int e = a0; e < a1; ++e) local += rs[e];
  int x = local;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[warp] = x;
  __syncthreads();
  if (warp == 0) {
    int w = wsum[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= o) w += y;
    }
    wsum[lane] = w;
  }
  __syncthreads();
  int run = x - local + (warp > 0 ? wsum[warp - 1] : 0);
  for (int e = a0; e < a1; ++e) {
    const int c = rs[e];
    rs[e] = run;
    run += c;
  }
  if (threadIdx.x == 1023) {
    rs[E] = wsum[31];
    ra.cnt[p] = wsum[31];
  }
}
__global__ void __launch_bounds__(256) rows_scatter_kernel(Geo g, RowsArgs ra) {
  const int p = blockIdx.y, ti = ra.ti[p], tj = ra.tj[p];
  const int e = blockIdx.x * 8 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (e >= g.nb * g.ncnt[ti]) return;
  const int r0 = ra.row_start[p][e], n = ra.row_start[p][e + 1] - r0;
  const size_t base = rows_base(g, ti, tj, e);
  for (int s0 = lane; s0 < n; s0 += 32) ra.row_idx[p][r0 + s0] = (int)(base + s0);
}

fekf_status build_rows(Ctx& c, int nb, cudaStream_t s) {
  Geo g = make_geo(c, nb);
  RowsArgs ra{};
  int emax = 0;
  const int np = (int)c.pairs.size();
  for (int p = 0; p < np; ++p) {
    PairNet& P = c.pairs[p];
    ra.ti[p] = P.ti;
    ra.tj[p] = P.tj;
    ra.row_start[p] = P.row_start.as<int>();
    ra.row_idx[p] = P.row_idx.as<int>();
    emax = std::max(emax, nb * (int)c.atoms_of[P.ti].size());
  }
  ra.cnt = c.rowcnt.as<int>();
  if (emax == 0) return FEKF_OK;
  const dim3 grid(cdiv(emax, 8), np);
  rows_count_kernel<<<grid, 256, 0, s>>>(g, ra, c.nl_j.as<int>());
  FEKF_LAUNCH_CHECK();
  rows_scan_kernel<<<np, 1024, 0, s>>>(g, ra);
  FEKF_LAUNCH_CHECK();
  rows_scatter_kernel<<<grid, 256, 0, s>>>(g, ra);
  FEKF_LAUNCH_CHECK();
  count_launch(3);
  return FEKF_OK;
}

static fekf_status build_trows(Ctx& c, int nb, cudaStream_t s) {
  TrowArgs A{};
  A.Na = c.Na;
  A.Nm = c.Nm;
  A.nl_j = c.nl_j.as<int>();
  A.v = c.vdir.as<real>();
  int np = 0, cmax = 0;
  for (size_t p = 0; p < c.pairs.size(); ++p) {
    PairNet& P = c.pairs[p];
    const long long Rmax = pair_rows(c, (int)p, nb);
    if (Rmax == 0) continue;
    A.Rmax[np] = (int)Rmax;
    A.Rdev[np] = rcount(c, (int)p);
    A.row_idx[np] = P.row_idx.as<int>();
    A.ck[np] = c.chunks.as<int>() + p * c.max_chunks;
    A.cnt[np] = c.rowcnt.as<int>() + c.pairs.size() + p;
    A.tidx[np] = P.tidx.as<int>();
    A.tpos[np] = P.tpos.as<int>();
    cmax = std::max(cmax, cdiv(Rmax, TCHUNK));
    ++np;
  }
  if (np == 0) return FEKF_OK;
  tcount_kernel<<<dim3(cmax, np), TCHUNK, 0, s>>>(A);
  FEKF_LAUNCH_CHECK();
  tscan_kernel<<<np, 1024, 0, s>>>(A);
  FEKF_LAUNCH_CHECK();
  tscatter_kernel<<<dim3(cmax, np), TCHUNK, 0, s>>>(A);
  FEKF_LAUNCH_CHECK();
  count_launch(3);
  return FEKF_OK;
}

// one layer of the forward: primal rows (tanh(z + b)) or tangent rows ((1 - y^2) zdot)
static fekf_status layer_fwd(const Layer& L, const real* w, long long Rmax, const int* Rdev, const real* A,
                             const real* Hprev, real* Y, real* H, const real* Yprim, const int* rowmap,
                             cudaStream_t s) {
  EpiFwd e;
  e.Y = Y;
  e.H = H;
  e.ld = L.dout;
  e.bias = w + L.b;
  e.dt = L.dt >= 0 ? w + L.dt : nullptr;
  e.Hp = Hprev;
  e.ldp = L.din;
  e.skip = Hprev ? L.skip : 0;
  e.dprev = L.din;
  e.Yprim = Yprim;
  e.rowmap = rowmap;
  return gemm<false, false>(Rmax, L.dout, L.din, A, L.din, w + L.W, L.dout, e, s, Rdev);
}

// v = 1 on the selected atoms of every image (0 elsewhere) and the active-row sets of every pair.
// force_error later sets v = +-1 on the same atoms, so the tangent forward reuses these row sets.
__global__ void mark_sel_kernel(int nb, int Na, const int* __restrict__ atom_idx, int n_sel, real* __restrict__ v) {
  for (int e = threadIdx.x; e < nb * Na * 3; e += blockDim.x) v[e] = 0.0;
  __syncthreads();
  for (int e = threadIdx.x; e < nb * n_sel * 3; e += blockDim.x) {
    const int b = e / (n_sel * 3), q = (e / 3) % n_sel, al = e % 3;
    v[((size_t)b * Na + atom_idx[q]) * 3 + al] = real(1);
  }
}

fekf_status mark_selected(Ctx& c, int nb, const int* atom_idx, int n_sel, cudaStream_t s) {
  c.sel_atoms = atom_idx;
  c.n_sel_atoms = n_sel;
  mark_sel_kernel<<<1, 1024, 0, s>>>(nb, c.Na, atom_idx, n_sel, c.vdir.as<real>());
  FEKF_LAUNCH_CHECK();
  count_launch();
  FEKF_TRY(build_trows(c, nb, s));
  c.trows_ready = true;
  return FEKF_OK;
}

// The embedding launches of every type pair side by side (one stream per pair, forked from and joined back
// into s), each persistent grid capped at the pair's share of the SMs by its row bound; serial when the
// context has no pair streams.  fn(p, stream) issues pair p's launch.
template <class Fn>
static fekf_status pairs_concurrent(Ctx& c, int nb, cudaStream_t s, Fn fn) {
  const int np = (int)c.pairs.size();
  long long tot = 0;
  int live = 0;
  for (int p = 0; p < np; ++p) {
    const long long r = pair_rows(c, p, nb);
    tot += r;
    live += r > 0;
  }
  if (c.pstreams.empty() || live < 2) {
    for (int p = 0; p < np; ++p)
      if (pair_rows(c, p, nb) > 0) FEKF_TRY(fn(p, s));
    return FEKF_OK;
  }
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  FEKF_CHECK_CUDA(cudaEventRecord(c.pev[0], s));
  for (int p = 0; p < np; ++p) {
    const long long r = pair_rows(c, p, nb);
    if (r == 0) continue;
    cudaStream_t ps = c.pstreams[p];
    FEKF_CHECK_CUDA(cudaStreamWaitEvent(ps, c.pev[0], 0));
    c.emb_grid_cap = (int)std::max<long long>(1, (long long)sms * r / tot);
    const fekf_status st = fn(p, ps);
    c.emb_grid_cap = 0;
    FEKF_TRY(st);
    FEKF_CHECK_CUDA(cudaEventRecord(c.pev[1 + p], ps));
  }
  for (int p = 0; p < np; ++p)
    if (pair_rows(c, p, nb) > 0) FEKF_CHECK_CUDA(cudaStreamWaitEvent(s, c.pev[1 + p], 0));
  return FEKF_OK;
}

// fp32 nets: fp32 copies of the fp64 inputs (R~, its Jacobian, d: once per geometry; the weights: before
// every primal forward, i.e. after every Kalman update)
#ifdef FEKF_NETS32
__global__ void to_real_kernel(const double* __restrict__ src, real* __restrict__ dst, long long n) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[i] = (real)src[i];
}
static fekf_status to_real(const DBuf& src, const DBuf& dst, long long n, cudaStream_t s) {
  if (src.p == dst.p || n <= 0) return FEKF_OK;
  to_real_kernel<<<cdiv(n, 256), 256, 0, s>>>(src.as<double>(), dst.as<real>(), n);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}
#endif

fekf_status prepare_geometry(Ctx& c, int nb, cudaStream_t s) {
#ifdef FEKF_NETS32
  const long long n = (long long)nb * c.Na * c.Nm;
  FEKF_TRY(to_real(c.em, c.em32, 4 * n, s));
  FEKF_TRY(to_real(c.jac, c.jac32, 12 * n, s));
  FEKF_TRY(to_real(c.rij, c.rij32, 3 * n, s));
#else
  (void)c; (void)nb; (void)s;
#endif
  return FEKF_OK;
}

fekf_status model_forward(Ctx& c, int nb, bool tangent, cudaStream_t s) {
#ifdef FEKF_NETS32
  if (!tangent) FEKF_TRY(to_real(c.w, c.w32, c.Np, s));
#endif
  const real* w = w_of(c);
  Geo g = make_geo(c, nb);
  if (tangent && !c.trows_ready) FEKF_TRY(build_trows(c, nb, s));
  if (tangent) c.trows_ready = false;
  // embedding nets (compacted rows)
  const bool fused = emb_fused_ok(c);
  if (fused)
    FEKF_TRY(pairs_concurrent(c, nb, s, [&](int p, cudaStream_t ps) {
      return emb_forward(c, p, pair_rows(c, p, nb), tangent, ps);
    }));
  for (size_t p = 0; p < c.pairs.size() && !fused; ++p) {
    PairNet& P = c.pairs[p];
    const long long Rmax = pair_rows(c, (int)p, nb);
    if (Rmax == 0) continue;
    const int* cnt = tangent ? tcount(c, (int)p) : rcount(c, (int)p);
    real* hin = tangent ? P.hin_t.as<real>() : P.hin.as<real>();
    emb_input_kernel<<<cdiv(Rmax, 256), 256, 0, s>>>((int)Rmax, cnt, P.row_idx.as<int>(),
                                                     tangent ? P.tidx.as<int>() : nullptr,
                                                     tangent ? c.rdot.as<real>() : em_of(c), hin);
    FEKF_LAUNCH_CHECK();
    count_launch();
    for (size_t l = 0; l < P.L.size(); ++l) {
      if (l == 0 && P.L[0].din == 1) {
        const Layer& L = P.L[0];
        emb_l0_kernel<<<cdiv(Rmax * L.dout, 256), 256, 0, s>>>(
            (int)Rmax, cnt, L.dout, hin, w + L.W, w + L.b, tangent ? P.Y[0].as<real>() : nullptr,
            tangent ? P.tidx.as<int>() : nullptr, tangent ? P.Yt[0].as<real>() : P.Y[0].as<real>(),
            tangent ? P.Ht[0].as<real>() : P.H[0].as<real>());
        FEKF_LAUNCH_CHECK();
        count_launch();
        continue;
      }
      if (!tangent) {
        const real* A = l == 0 ? hin : P.H[l - 1].as<real>();
        FEKF_TRY(layer_fwd(P.L[l], w, Rmax, cnt, A, l == 0 ? nullptr : P.H[l - 1].as<real>(), P.Y[l].as<real>(),
                           P.H[l].as<real>(), nullptr, nullptr, s));
      } else {
        const real* A = l == 0 ? hin : P.Ht[l - 1].as<real>();
        FEKF_TRY(layer_fwd(P.L[l], w, Rmax, cnt, A, l == 0 ? nullptr : P.Ht[l - 1].as<real>(), P.Yt[l].as<real>(),
                           P.Ht[l].as<real>(), P.Y[l].as<real>(), P.tidx.as<int>(), s));
      }
    }
  }
  // descriptor
  PairPtrs pp = make_pp(c);
  FitPtrs fp = make_fp(c, nb);
  const size_t smem = (8 * (size_t)c.M + 8 * (size_t)c.Nm + 4 * 32 * DESC_MC * (DESC_THREADS / 32)) * sizeof(real);
  const size_t Xoff = (size_t)c.B * c.Na * 4 * c.M;
  static size_t dattr = 0;
  if (smem > dattr) {
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(desc_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    dattr = smem;
  }
  desc_fwd_kernel<<<nb * c.Na, DESC_THREADS, smem, s>>>(g, pp, fp, em_of(c), c.rdot.as<real>(),
                                                        tangent ? 1 : 0, c.X.as<real>(), c.X.as<real>() + Xoff);
  FEKF_LAUNCH_CHECK();
  count_launch();
  // fitting nets (stacked rows: the tangent half starts at row F); one grouped GEMM per layer over types
  const size_t nfl = c.fits[0].L.size();
  for (size_t l = 0; l < nfl; ++l) {
    GemmProb<EpiFwd> pr[GG_MAX];
    int n = 0;
    for (int t = 0; t < c.nt; ++t) {
      FitNet& Fn = c.fits[t];
      const long long F = fit_rows(c, t, nb);
      if (F == 0) continue;
      const Layer& L = Fn.L[l];
      const real* Ain = l == 0 ? Fn.D.as<real>() : Fn.H[l - 1].as<real>();
      const real* Hprev = l == 0 ? nullptr : Fn.H[l - 1].as<real>();
      const size_t oi = tangent ? (size_t)F * L.din : 0, oo = tangent ? (size_t)F * L.dout : 0;
      EpiFwd e;
      e.Y = Fn.Y[l].as<real>() + oo;
      e.H = Fn.H[l].as<real>() + oo;
      e.ld = L.dout;
      e.bias = w + L.b;
      e.dt = L.dt >= 0 ? w + L.dt : nullptr;
      e.Hp = Hprev ? Hprev + oi : nullptr;
      e.ldp = L.din;
      e.skip = Hprev ? L.skip : 0;
      e.dprev = L.din;
      e.Yprim = tangent ? Fn.Y[l].as<real>() : nullptr;
      e.rowmap = nullptr;
      pr[n++] = GemmProb<EpiFwd>{(int)F, L.dout, L.din, nullptr, nullptr, Ain + oi, L.din, w + L.W, L.dout, -1, 0, 0, 1, e};
    }
    FEKF_TRY(gemm_group<false, false>(pr, n, s));
  }
  {
    OutArgs A{};
    long long Fmax = 0;
    A.h = c.fits[0].L.back().dout;
    for (int t = 0; t < c.nt; ++t) {
      FitNet& Fn = c.fits[t];
      const long long F = fit_rows(c, t, nb);
      const real* Hl = Fn.H.back().as<real>();
      real* eo = Fn.eout.as<real>();
      A.rows[t] = F;
      A.F[t] = F;
      A.H[t] = tangent ? Hl + (size_t)F * A.h : Hl;
      A.W[t] = w + Fn.Wout;
      A.b[t] = w + Fn.bout;
      A.out[t] = tangent ? eo + F : eo;
      Fmax = std::max(Fmax, F);
    }
    if (Fmax > 0) {
      fit_out_kernel<<<dim3(cdiv(Fmax * 32, 256), c.nt), 256, 0, s>>>(A);
      FEKF_LAUNCH_CHECK();
      count_launch();
    }
  }
  return FEKF_OK;
}

fekf_status energy_outputs(Ctx& c, int nb, cudaStream_t s) {
  Geo g = make_geo(c, nb);
  FitPtrs fp = make_fp(c, nb);
  energy_scatter_kernel<<<nb, 128, 0, s>>>(g, fp, c.eatom.as<double>(), c.etot.as<double>());
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

fekf_status energy_error(Ctx& c, int nb, const double* e_label, double* abs_sum, cudaStream_t s) {
  Geo g = make_geo(c, nb);
  FitPtrs fp = make_fp(c, nb);
  const double scale = c.o.grad_reduce == 1 ? 1.0 / c.Bg : 1.0;
  energy_error_kernel<<<1, 256, 0, s>>>(g, fp, c.etot.as<double>(), e_label, scale, abs_sum);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

fekf_status seed_force(Ctx& c, int nb, cudaStream_t s) {
  // dE_tot/dE_i = 1 for every atom: F = -dE/dx
  for (int t = 0; t < c.nt; ++t) {
    const long long F = fit_rows(c, t, nb);
    if (F == 0) continue;
    fill_kernel<<<cdiv(F, 256), 256, 0, s>>>(c.fits[t].ebar.as<real>(), F, real(1));
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  return FEKF_OK;
}

fekf_status force_error(Ctx& c, int nb, const double* f_label, const int* atom_idx, int n_sel, double* abs_sum,
                        cudaStream_t s) {
  Geo g = make_geo(c, nb);
  FitPtrs fp = make_fp(c, nb);
  double seed = -1.0 / ((double)c.Na * n_sel * 3);
  if (c.o.grad_reduce == 1) seed /= c.Bg;
  force_error_kernel<<<1, 1024, 0, s>>>(g, c.force.as<double>(), f_label, atom_idx, n_sel, seed, c.vdir.as<real>(), fp,
                                       abs_sum);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

fekf_status tangent_env(Ctx& c, int nb, cudaStream_t s) {
  const long long n = (long long)nb * c.Na * c.Nm;
  tangent_env_kernel<<<cdiv(n, 256), 256, 0, s>>>(jac_of(c), c.nl_j.as<int>(), c.vdir.as<real>(), c.Na, c.Nm,
                                                  n, c.rdot.as<real>());
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// Reverse pass from the fitting-output seeds (ebar).  MODE_ENERGY_GRAD: weight gradients of the
// primal graph.  MODE_FORCE: adjoints down to s and R~, then forces/virials.  MODE_FORCE_JAC: weight
// gradients of the dual (primal+tangent) graph.
static int sm_count() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

fekf_status model_backward(Ctx& c, int nb, Mode mode, double* gout, cudaStream_t s) {
  const real* w = w_of(c);
  const bool dual = mode == MODE_FORCE_JAC;
  if (mode == MODE_FORCE_SEL && !emb_fused_ok(c)) mode = MODE_FORCE;   // per-layer path: every row
  const bool force = mode == MODE_FORCE || mode == MODE_FORCE_SEL;
  const bool want_w = !force;
  Geo g = make_geo(c, nb);
  PairPtrs pp = make_pp(c);
  FitPtrs fp = make_fp(c, nb);
  // ---- fitting nets (stacked rows); weight and data gradients grouped over types per layer ----
  const size_t nfl = c.fits[0].L.size();
  {
    // output layer of every type: Hbar = ebar (x) W_out in one launch, [W_out ; b_out] gradients grouped
    OutArgs A{};
    WgradJob jobs[FEKF_MAX_TYPES];
    int nj = 0;
    long long rmax = 0;
    const int h = c.fits[0].L.back().dout;
    A.h = h;
    for (int t = 0; t < c.nt; ++t) {
      FitNet& Fn = c.fits[t];
      const long long F = fit_rows(c, t, nb);
      A.rows[t] = dual ? 2 * F : F;
      A.ebar[t] = Fn.ebar.as<real>();
      A.W[t] = w + Fn.Wout;
      A.Hb[t] = Fn.Hb.back().as<real>();
      rmax = std::max(rmax, A.rows[t]);
      if (want_w && F > 0) {
        const real* Hl = Fn.H.back().as<real>();
        const real* eb = Fn.ebar.as<real>();
        jobs[nj++] = WgradJob{h, 1, Seg{Hl, eb, F, nullptr, 1},
                              Seg{dual ? Hl + (size_t)F * h : nullptr, dual ? eb + F : nullptr, dual ? F : 0, nullptr, 0},
                              gout + Fn.Wout};
      }
    }
    if (rmax > 0) {
      fit_out_bwd_kernel<<<dim3(cdiv(rmax * h, 256), c.nt), 256, 0, s>>>(A);
      FEKF_LAUNCH_CHECK();
      count_launch();
    }
    if (nj) FEKF_TRY(wgrad_group(c, jobs, nj, s));
  }
  for (int l = (int)nfl - 1; l >= 0; --l) {
    WgradJob jobs[FEKF_MAX_TYPES];
    GemmProb<EpiDgrad> dg[GG_MAX];
    int nj = 0, nd = 0;
    {
      // the layer's activation adjoint (and timestep gradient) for every type in one launch
      ActArgs A{};
      A.d = c.fits[0].L[l].dout;
      A.dual = dual ? 1 : 0;
      const bool has_dt = c.fits[0].L[l].dt >= 0;
      for (int t = 0; t < c.nt; ++t) {
        FitNet& Fn = c.fits[t];
        const Layer& L = Fn.L[l];
        A.R[t] = fit_rows(c, t, nb);
        A.Y[t] = Fn.Y[l].as<real>();
        A.Hb[t] = Fn.Hb[l].as<real>();
        A.dt[t] = has_dt ? w + L.dt : nullptr;
        A.Zb[t] = Fn.Zb[l].as<real>();
        A.gdt[t] = has_dt ? gout + L.dt : nullptr;
      }
      FEKF_TRY(act_bwd_types(c, A, c.nt, want_w && has_dt, s));
    }
    for (int t = 0; t < c.nt; ++t) {
      FitNet& Fn = c.fits[t];
      const long long F = fit_rows(c, t, nb);
      if (F == 0) continue;
      const long long nF = dual ? 2 * F : F;
      const Layer& L = Fn.L[l];
      const real* Hprev = l == 0 ? Fn.D.as<real>() : Fn.H[l - 1].as<real>();
      if (want_w) {
        // stacked rows; the ones column covers the primal half only (bias not in the tangent)
        jobs[nj++] = WgradJob{L.din, L.dout, Seg{Hprev, Fn.Zb[l].as<real>(), F, nullptr, 1},
                              Seg{dual ? Hprev + (size_t)F * L.din : nullptr,
                                  dual ? Fn.Zb[l].as<real>() + (size_t)F * L.dout : nullptr, dual ? F : 0, nullptr, 0},
                              gout + L.W};
      }
      real* out = l == 0 ? Fn.Db.as<real>() : Fn.Hb[l - 1].as<real>();
      EpiDgrad e{out, L.din, Fn.Hb[l].as<real>(), L.dout, l == 0 ? 0 : L.skip, L.din};
      dg[nd++] = GemmProb<EpiDgrad>{(int)nF, L.din, L.dout, nullptr, nullptr, Fn.Zb[l].as<real>(), L.dout, w + L.W,
                                    L.dout, -1, 0, 0, 1, e};
    }
    if (nj) FEKF_TRY(wgrad_group(c, jobs, nj, s));
    if (l == 0 && want_w && c.split_armed) {
      // the fitting blocks' gradient is final: the early P pass may start (Kf::pass); the rest of this
      // reverse pass leaves it split_sms SMs
      FEKF_CHECK_CUDA(cudaEventRecord(c.ev_fit, s));
      c.emb_sms = std::max(1, sm_count() - c.kf->split_sms);
    }
    FEKF_TRY(gemm_group<false, true>(dg, nd, s));
  }
  // ---- descriptor (Eq. 4) ----
  const size_t Xoff = (size_t)c.B * c.Na * 4 * c.M;
  if (emb_fused_ok(c)) {
    SeedOut so{};
    for (size_t p = 0; p < c.pairs.size(); ++p) {
      PairNet& P = c.pairs[p];
      so.gbar[p] = P.Hb.back().as<real>();
      so.hbt[p] = P.Hbt.back().as<real>();
      so.dr[p] = P.Zb[0].as<real>();
    }
    const size_t smem = (16 * (size_t)c.M + 2 * (size_t)c.M * (c.M2 + 1) + 8 * (size_t)c.Nm) * sizeof(real);
    auto launch = [&](auto kern) -> fekf_status {
      FEKF_CHECK_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      kern<<<nb * c.Na, 256, smem, s>>>(g, fp, pp, so, c.X.as<real>(), c.X.as<real>() + Xoff, em_of(c),
                                        c.rdot.as<real>(), c.Xb.as<real>(), c.Xb.as<real>() + Xoff);
      return FEKF_OK;
    };
    if (dual) FEKF_TRY(launch(desc_bwd_seed_kernel<true, false, false>));
    else if (mode == MODE_FORCE_SEL) FEKF_TRY(launch(desc_bwd_seed_kernel<false, true, true>));
    else if (force) FEKF_TRY(launch(desc_bwd_seed_kernel<false, true, false>));
    else FEKF_TRY(launch(desc_bwd_seed_kernel<false, false, false>));
  } else {
    const size_t smem = (8 * c.M + 2 * c.M * (c.M2 + 1)) * sizeof(real);
    desc_bwd_kernel<<<nb * c.Na, 128, smem, s>>>(g, fp, c.X.as<real>(), c.X.as<real>() + Xoff, dual ? 1 : 0,
                                                 c.Xb.as<real>(), c.Xb.as<real>() + Xoff);
  }
  FEKF_LAUNCH_CHECK();
  count_launch();
  // ---- embedding nets (compacted rows; tangent rows separately) ----
  if (emb_fused_ok(c)) {
    if (force) {   // force-only reverse (no weight gradients): on the critical path, pairs side by side
      FEKF_TRY(pairs_concurrent(c, nb, s, [&](int p, cudaStream_t ps) {
        return emb_backward(c, p, pair_rows(c, p, nb), (int)mode, gout, ps);
      }));
    } else {
      for (size_t p = 0; p < c.pairs.size(); ++p) {
        const long long Rmax = pair_rows(c, (int)p, nb);
        if (Rmax == 0) continue;
        FEKF_TRY(emb_backward(c, (int)p, Rmax, (int)mode, gout, s));
      }
    }
  } else {
  {
    SeedPtrs sp{};
    for (size_t p = 0; p < c.pairs.size(); ++p) {
      PairNet& P = c.pairs[p];
      sp.Y[p] = P.Y.back().as<real>();
      sp.Yt[p] = P.Yt.back().as<real>();
      sp.Hb[p] = P.Hb.back().as<real>();
      sp.Zb[p] = P.Zb.back().as<real>();
      sp.Hbt[p] = P.Hbt.back().as<real>();
      sp.Zbt[p] = P.Zbt.back().as<real>();
    }
    emb_seed_atom_kernel<<<nb * c.Na, 128, 8 * c.M * sizeof(real), s>>>(
        g, pp, sp, em_of(c), c.rdot.as<real>(), c.Xb.as<real>(), c.Xb.as<real>() + Xoff, dual ? 1 : 0);
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  for (size_t p = 0; p < c.pairs.size(); ++p) {
    PairNet& P = c.pairs[p];
    const long long Rmax = pair_rows(c, (int)p, nb);
    if (Rmax == 0) continue;
    const int* rc = rcount(c, (int)p);
    const int* tc = tcount(c, (int)p);
    const int nl = (int)P.L.size();
    // Zbar of the last layer comes from emb_seed; every other layer's Zbar from the fused epilogue of
    // the data-gradient GEMM one layer up (tangent rows first: the primal zbar needs their hdotbar)
    for (int l = nl - 1; l >= 0; --l) {
      const Layer& L = P.L[l];
      if (want_w) {
        const real* Hp = l == 0 ? P.hin.as<real>() : P.H[l - 1].as<real>();
        const real* Hpt = l == 0 ? P.hin_t.as<real>() : P.Ht[l - 1].as<real>();
        FEKF_TRY(wgrad(c, L.din, L.dout, Seg{Hp, P.Zb[l].as<real>(), Rmax, rc, 1},
                       Seg{dual ? Hpt : nullptr, dual ? P.Zbt[l].as<real>() : nullptr, dual ? Rmax : 0, tc, 0},
                       gout + L.W, s, true));
      }
      if (l > 0) {
        if (dual) {
          EpiDgradAct et{P.Hbt[l - 1].as<real>(), L.din, P.Hbt[l].as<real>(), L.dout, L.skip, L.din,
                         P.Y[l - 1].as<real>(), P.Zbt[l - 1].as<real>(), nullptr, nullptr, nullptr,
                         P.tidx.as<int>()};
          FEKF_TRY(gemm<false, true>(Rmax, L.din, L.dout, P.Zbt[l].as<real>(), L.dout, w + L.W, L.dout, et, s, tc));
        }
        EpiDgradAct e{P.Hb[l - 1].as<real>(), L.din, P.Hb[l].as<real>(), L.dout, L.skip, L.din,
                      P.Y[l - 1].as<real>(), P.Zb[l - 1].as<real>(), dual ? P.tpos.as<int>() : nullptr,
                      P.Yt[l - 1].as<real>(), P.Hbt[l - 1].as<real>(), nullptr};
        FEKF_TRY(gemm<false, true>(Rmax, L.din, L.dout, P.Zb[l].as<real>(), L.dout, w + L.W, L.dout, e, s, rc));
      } else if (mode == MODE_FORCE) {
        FEKF_TRY(gemm<false, true>(Rmax, 1, L.dout, P.Zb[0].as<real>(), L.dout, w + L.W, L.dout,
                                   EpiStore<real>{P.sbar.as<real>(), 1}, s, rc));
      }
    }
  }
  }
  if (force) {
    if (!emb_fused_ok(c)) {
      prod_force_kernel<<<nb * c.Na, 128, 0, s>>>(g, pp, c.Xb.as<real>(), jac_of(c), c.nl_j.as<int>(),
                                                  c.frow.as<real>());
      FEKF_LAUNCH_CHECK();
      count_launch();
    }
    // MODE_FORCE_SEL: only the selected atoms' forces are formed (their slots are exactly the active rows)
    const bool sel = mode == MODE_FORCE_SEL && c.sel_atoms;
    const int nw = sel ? nb * c.n_sel_atoms : nb * c.Na;
    force_gather_kernel<<<cdiv(nw, 8), 256, 0, s>>>(nb, c.Na, c.Nm, sel ? c.sel_atoms : nullptr, c.n_sel_atoms,
                                                    c.nl_j.as<int>(), rij_of(c), c.frow.as<real>(),
                                                    c.rev_off.as<int>(), c.rev_idx.as<int>(), c.force.as<double>(),
                                                    c.vatom.as<double>());
    FEKF_LAUNCH_CHECK();
    count_launch();
    if (!sel) {   // the force updates use the selected atoms' forces only: no virial there
      virial_reduce_kernel<<<nb, 32, 0, s>>>(c.vatom.as<double>(), c.Na, c.virial.as<double>());
      FEKF_LAUNCH_CHECK();
      count_launch();
    }
  }
  c.emb_sms = 0;
  return FEKF_OK;
}

}  // namespace FEKF_NETNS
}  // namespace fekf
