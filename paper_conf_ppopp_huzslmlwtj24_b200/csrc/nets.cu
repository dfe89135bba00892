// DeePMD se_a nets on sm_100a, fp64: forward, backward to coordinates, energy- and force-Jacobians.
//
//   embedding  G = E2 o E1 o E0(s)          P:L84-90 (§2.1 item 2), skip rule: reading Z12
//   descriptor X = R~^T G / N_m, D = X^T X^<   P:L92, P:L233 (Fig. 6), scale 1/N_m: reading Z13
//   fitting    E_i = F3 o F2 o F1 o F0(D)    P:L95-101, residual timestep dt: reading Z14
//   forces     F = -dE/dx via dE/dX by Eq. 4 and the R~ chain rule (Opt1)
//   force-Jacobian: d/dw of Edot = <dE/dx, v> (forward-mode tangent along v, then reverse over the
//     primal+tangent graph): every activation carries a tangent row stacked under its primal row
//     ([primal rows | tangent rows]), so each weight-gradient is ONE GEMM over 2R rows.
//
// Row layouts (padded slots kept: their R~ rows are 0 so they add exact zeros):
//   pair net (ti,tj): row r = (b*n_ti + k)*sel_tj + s  <->  atom atoms_of[ti][k], slot sec[tj]+s
//   fitting net t:    row r = b*n_t + k
#include <algorithm>

#include "model.cuh"

namespace fekf {

// =================================================================================================
// fp64 GEMM  C = op(A) op(B)   (64x64x16 tiles, 256 threads, 4x4 register micro-tiles, smem double
// buffering).  TA: A stored [K x M]; TB: B stored [N x K].  Optional "ones" row: op(A) row aug_m is
// (k < aug_k ? 1 : 0) so [W-grad ; b-grad] = [H | 1]^T Zbar comes out of one GEMM.
// =================================================================================================
constexpr int GB_M = 64, GB_N = 64, GB_K = 16;

struct EpiStore {
  double* C; int ldc;
  __device__ void operator()(int r, int c, double v) const { C[(size_t)r * ldc + c] = v; }
};
struct EpiPartial {
  double* ws; int M, N;
  __device__ void operator()(int r, int c, double v) const { ws[((size_t)blockIdx.z * M + r) * N + c] = v; }
};
// forward layer: y = tanh(z + b) (primal) or ydot = (1 - y^2) zdot (tangent); h = skip(h_prev) + dt*y
struct EpiFwd {
  double* Y; double* H; int ld;
  const double* bias; const double* dt;
  const double* Hp; int ldp; int skip; int dprev;
  const double* Yprim;  // non-null: tangent rows (Y/H point to the tangent half, Yprim to the primal)
  __device__ void operator()(int r, int c, double v) const {
    double sk = 0.0;
    if (skip == 1) sk = Hp[(size_t)r * ldp + c];
    else if (skip == 2) sk = Hp[(size_t)r * ldp + (c % dprev)];
    double y;
    if (Yprim == nullptr) {
      y = tanh(v + bias[c]);
    } else {
      const double yp = Yprim[(size_t)r * ld + c];
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
dgemm_kernel(int M, int N, int K, const double* __restrict__ A, int lda, const double* __restrict__ B, int ldb,
             int aug_m, int aug_k, int kps, Epi epi) {
  __shared__ __align__(16) double As[2][GB_K][GB_M + 2];
  __shared__ __align__(16) double Bs[2][GB_K][GB_N + 2];
  const int tid = threadIdx.x;
  const int m0 = blockIdx.x * GB_M, n0 = blockIdx.y * GB_N;
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
                        cudaStream_t s, int aug_m = -1, int aug_k = 0, int splits = 1, int kps = 0) {
  if (M <= 0 || N <= 0) return FEKF_OK;
  if (kps <= 0) kps = K;
  dim3 grid((unsigned)cdiv(M, GB_M), (unsigned)cdiv(N, GB_N), (unsigned)splits);
  dgemm_kernel<TA, TB, Epi><<<grid, 256, 0, s>>>((int)M, N, K, A, lda, B, ldb, aug_m, aug_k, kps, epi);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

__global__ void splitk_reduce_kernel(const double* __restrict__ ws, int splits, int M, int N, double* __restrict__ out) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (long long)M * N) return;
  double a = 0.0;
  for (int z = 0; z < splits; ++z) a += ws[(size_t)z * M * N + i];
  out[i] = a;
}

// [W-grad ; b-grad] (din+1 x dout) = [Hprev | 1]^T Zbar over `rows` rows; the ones column covers
// the first `rows_primal` rows (the bias does not enter the tangent).  Written to g at the W offset
// (W then b are contiguous in the layout).  Split-K partials are summed in a fixed order.
static fekf_status wgrad(Ctx& c, int din, int dout, long long rows, long long rows_primal, const double* Hprev,
                         const double* Zb, double* gout, cudaStream_t s) {
  const int M = din + 1, N = dout;
  const long long tiles = (long long)cdiv(M, GB_M) * cdiv(N, GB_N);
  long long splits = std::max<long long>(1, std::min<long long>(cdiv(rows, 256), cdiv(4 * 148, tiles)));
  splits = std::min<long long>(splits, (long long)(c.splitk_elems / ((size_t)M * N)));
  splits = std::max<long long>(1, splits);
  int kps = (int)(cdiv(cdiv(rows, splits), GB_K) * GB_K);
  splits = cdiv(rows, kps);
  if (splits <= 1) {
    return gemm<true, false>(M, N, (int)rows, Hprev, din, Zb, dout, EpiStore{gout, dout}, s, din, (int)rows_primal);
  }
  FEKF_TRY(gemm<true, false>(M, N, (int)rows, Hprev, din, Zb, dout, EpiPartial{c.splitk_ws.as<double>(), M, N}, s,
                             din, (int)rows_primal, (int)splits, kps));
  splitk_reduce_kernel<<<cdiv((long long)M * N, 256), 256, 0, s>>>(c.splitk_ws.as<double>(), (int)splits, M, N, gout);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// =================================================================================================
// elementwise / small kernels
// =================================================================================================
// zbar = (1 - y^2) ybar - 2 y ydot ydotbar  (primal rows), zdotbar = (1 - y^2) ydotbar  (tangent rows);
// ybar = dt * hbar (residual layers with a timestep vector) else hbar.
__global__ void act_bwd_kernel(long long R, int d, const double* __restrict__ Y, const double* __restrict__ Hb,
                               const double* __restrict__ dt, int dual, double* __restrict__ Zb) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= R * d) return;
  const int c = (int)(i % d);
  const double y = Y[i];
  const double t = 1.0 - y * y;
  double yb = Hb[i];
  if (dt) yb *= dt[c];
  if (dual) {
    const size_t j = (size_t)R * d + i;
    const double yd = Y[j];
    double ydb = Hb[j];
    if (dt) ydb *= dt[c];
    Zb[i] = t * yb - 2.0 * y * yd * ydb;
    Zb[j] = t * ydb;
  } else {
    Zb[i] = t * yb;
  }
}

// dt-grad: out[c] = sum_r A[r][c] B[r][c] (two fixed-order stages)
__global__ void colsum_prod_kernel(const double* __restrict__ A, const double* __restrict__ B, long long rows, int d,
                                   int chunk, double* __restrict__ ws) {
  const long long r0 = (long long)blockIdx.x * chunk;
  const long long r1 = min(rows, r0 + chunk);
  for (int c = threadIdx.x; c < d; c += blockDim.x) {
    double a = 0.0;
    for (long long r = r0; r < r1; ++r) a += A[(size_t)r * d + c] * B[(size_t)r * d + c];
    ws[(size_t)blockIdx.x * d + c] = a;
  }
}
__global__ void colsum_reduce_kernel(const double* __restrict__ ws, int nchunk, int d, double* __restrict__ out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= d) return;
  double a = 0.0;
  for (int k = 0; k < nchunk; ++k) a += ws[(size_t)k * d + c];
  out[c] = a;
}
static fekf_status colsum_prod(Ctx& c, const double* A, const double* B, long long rows, int d, double* out,
                               cudaStream_t s) {
  const int chunk = 64;
  int nchunk = cdiv(rows, chunk);
  if ((size_t)nchunk * d > c.colsum_elems) { set_error("colsum workspace too small"); return FEKF_EINVAL; }
  colsum_prod_kernel<<<nchunk, 256, 0, s>>>(A, B, rows, d, chunk, c.colsum_ws.as<double>());
  FEKF_LAUNCH_CHECK();
  colsum_reduce_kernel<<<cdiv(d, 256), 256, 0, s>>>(c.colsum_ws.as<double>(), nchunk, d, out);
  FEKF_LAUNCH_CHECK();
  count_launch(2);
  return FEKF_OK;
}

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
  const double* G[FEKF_MAX_TYPES * FEKF_MAX_TYPES];
  double* Gb[FEKF_MAX_TYPES * FEKF_MAX_TYPES];
  long long R[FEKF_MAX_TYPES * FEKF_MAX_TYPES];
};
struct FitPtrs {
  double* D[FEKF_MAX_TYPES];
  const double* Db[FEKF_MAX_TYPES];
  double* eout[FEKF_MAX_TYPES];
  double* ebar[FEKF_MAX_TYPES];
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

// embedding input s (primal rows) or s-dot (tangent rows) gathered from R~ / R~-dot column 0
__global__ void emb_input_kernel(Geo g, int ti, int tj, long long R, const double* __restrict__ src, double* __restrict__ out) {
  const long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= R) return;
  const int sel = g.sel[tj];
  const long long bk = r / sel;
  const int s = (int)(r % sel);
  const int b = (int)(bk / g.ncnt[ti]);
  const int k = (int)(bk % g.ncnt[ti]);
  const int i = g.atoms[g.atoms_off[ti] + k];
  const size_t idx = ((size_t)b * g.Na + i) * g.Nm + g.sec[tj] + s;
  out[r] = src[idx * 4];
}

// X = R~^T G / N_m (4 x M) per atom and D = X^T X^< (Fig. 6); tangent: Xdot = (Rdot^T G + R~^T Gdot)/N_m,
// Ddot = Xdot^T X^< + X^T Xdot^<.  One CTA per atom; fixed summation order over (tj, slot).
__global__ void desc_fwd_kernel(Geo g, PairPtrs pp, FitPtrs fp, const double* __restrict__ em,
                                const double* __restrict__ rdot, int tangent, double* __restrict__ X,
                                double* __restrict__ Xd) {
  extern __shared__ double sm[];
  const int M = g.M, M2 = g.M2;
  double* xs = sm;            // [4][M]
  double* xds = sm + 4 * M;   // [4][M]
  const int atom = blockIdx.x;
  const int b = atom / g.Na, i = atom % g.Na;
  const int ti = g.types[i], k = g.tindex[i];
  for (int m = threadIdx.x; m < M; m += blockDim.x) {
    double a0 = 0, a1 = 0, a2 = 0, a3 = 0, d0 = 0, d1 = 0, d2 = 0, d3 = 0;
    for (int tj = 0; tj < g.nt; ++tj) {
      const int p = ti * g.nt + tj;
      const int sel = g.sel[tj];
      const long long base = ((long long)b * g.ncnt[ti] + k) * sel;
      const double* G = pp.G[p];
      const long long R = pp.R[p];
      for (int s = 0; s < sel; ++s) {
        const size_t idx = ((size_t)b * g.Na + i) * g.Nm + g.sec[tj] + s;
        const double* e = em + idx * 4;
        const double gv = G[(size_t)(base + s) * M + m];
        a0 = fma(e[0], gv, a0); a1 = fma(e[1], gv, a1); a2 = fma(e[2], gv, a2); a3 = fma(e[3], gv, a3);
        if (tangent) {
          const double* ed = rdot + idx * 4;
          const double gd = G[(size_t)(R + base + s) * M + m];
          d0 = fma(ed[0], gv, fma(e[0], gd, d0));
          d1 = fma(ed[1], gv, fma(e[1], gd, d1));
          d2 = fma(ed[2], gv, fma(e[2], gd, d2));
          d3 = fma(ed[3], gv, fma(e[3], gd, d3));
        }
      }
    }
    const double inv = 1.0 / g.Nm;
    if (!tangent) {
      xs[m] = a0 * inv; xs[M + m] = a1 * inv; xs[2 * M + m] = a2 * inv; xs[3 * M + m] = a3 * inv;
      double* xo = X + (size_t)atom * 4 * M;
      xo[m] = xs[m]; xo[M + m] = xs[M + m]; xo[2 * M + m] = xs[2 * M + m]; xo[3 * M + m] = xs[3 * M + m];
    } else {
      xds[m] = d0 * inv; xds[M + m] = d1 * inv; xds[2 * M + m] = d2 * inv; xds[3 * M + m] = d3 * inv;
      double* xo = Xd + (size_t)atom * 4 * M;
      xo[m] = xds[m]; xo[M + m] = xds[M + m]; xo[2 * M + m] = xds[2 * M + m]; xo[3 * M + m] = xds[3 * M + m];
    }
  }
  __syncthreads();
  if (tangent) {
    // primal X of this atom (computed by the primal pass)
    const double* xo = X + (size_t)atom * 4 * M;
    for (int e = threadIdx.x; e < 4 * M; e += blockDim.x) xs[e] = xo[e];
    __syncthreads();
  }
  const long long row = (long long)b * g.ncnt[ti] + k;
  double* D = fp.D[ti] + (size_t)(tangent ? fp.F[ti] + row : row) * M * M2;
  for (int e = threadIdx.x; e < M * M2; e += blockDim.x) {
    const int m = e / M2, n = e % M2;
    double v;
    if (!tangent) {
      v = xs[m] * xs[n] + xs[M + m] * xs[M + n] + xs[2 * M + m] * xs[2 * M + n] + xs[3 * M + m] * xs[3 * M + n];
    } else {
      v = 0.0;
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) v += xds[kk * M + m] * xs[kk * M + n] + xs[kk * M + m] * xds[kk * M + n];
    }
    D[e] = v;
  }
}

// Eq. 4: dE/dX = X^< Dbar^T + [X Dbar into the first M^< columns].
//   Xbar = B(X, Dbar) + B(Xdot, Ddotbar) ; Xdotbar = B(X, Ddotbar)   (dual)
__global__ void desc_bwd_kernel(Geo g, FitPtrs fp, const double* __restrict__ X, const double* __restrict__ Xd, int dual,
                                double* __restrict__ Xb, double* __restrict__ Xdb) {
  extern __shared__ double sm[];
  const int M = g.M, M2 = g.M2;
  double* xs = sm;
  double* xds = xs + 4 * M;
  double* db = xds + 4 * M;
  double* ddb = db + M * M2;
  const int atom = blockIdx.x;
  const int b = atom / g.Na, i = atom % g.Na;
  const int ti = g.types[i], k = g.tindex[i];
  const long long row = (long long)b * g.ncnt[ti] + k;
  const double* Dbp = fp.Db[ti] + (size_t)row * M * M2;
  const double* Ddbp = fp.Db[ti] + (size_t)(fp.F[ti] + row) * M * M2;
  for (int e = threadIdx.x; e < 4 * M; e += blockDim.x) {
    xs[e] = X[(size_t)atom * 4 * M + e];
    if (dual) xds[e] = Xd[(size_t)atom * 4 * M + e];
  }
  for (int e = threadIdx.x; e < M * M2; e += blockDim.x) {
    db[e] = Dbp[e];
    if (dual) ddb[e] = Ddbp[e];
  }
  __syncthreads();
  for (int e = threadIdx.x; e < 4 * M; e += blockDim.x) {
    const int kk = e / M, p = e % M;
    const double* x = xs + kk * M;
    double a = 0.0, ad = 0.0;
    for (int n = 0; n < M2; ++n) a = fma(db[p * M2 + n], x[n], a);
    if (p < M2)
      for (int m = 0; m < M; ++m) a = fma(db[m * M2 + p], x[m], a);
    if (dual) {
      const double* xd = xds + kk * M;
      for (int n = 0; n < M2; ++n) { a = fma(ddb[p * M2 + n], xd[n], a); ad = fma(ddb[p * M2 + n], x[n], ad); }
      if (p < M2)
        for (int m = 0; m < M; ++m) { a = fma(ddb[m * M2 + p], xd[m], a); ad = fma(ddb[m * M2 + p], x[m], ad); }
      Xdb[(size_t)atom * 4 * M + e] = ad;
    }
    Xb[(size_t)atom * 4 * M + e] = a;
  }
}

// adjoint of G (and Gdot) per embedding row from the atom's Xbar (and Xdotbar):
//   Gbar = (R~ Xbar + Rdot Xdotbar)/N_m ; Gdotbar = R~ Xdotbar / N_m
__global__ void emb_seed_kernel(Geo g, int ti, int tj, long long R, const double* __restrict__ em,
                                const double* __restrict__ rdot, const double* __restrict__ Xb,
                                const double* __restrict__ Xdb, int dual, double* __restrict__ Hb) {
  const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const int M = g.M;
  if (e >= R * M) return;
  const long long r = e / M;
  const int m = (int)(e % M);
  const int sel = g.sel[tj];
  const long long bk = r / sel;
  const int s = (int)(r % sel);
  const int b = (int)(bk / g.ncnt[ti]);
  const int k = (int)(bk % g.ncnt[ti]);
  const int i = g.atoms[g.atoms_off[ti] + k];
  const size_t idx = ((size_t)b * g.Na + i) * g.Nm + g.sec[tj] + s;
  const size_t atom = (size_t)b * g.Na + i;
  const double* xb = Xb + atom * 4 * M;
  const double* rr = em + idx * 4;
  double a = rr[0] * xb[m] + rr[1] * xb[M + m] + rr[2] * xb[2 * M + m] + rr[3] * xb[3 * M + m];
  const double inv = 1.0 / g.Nm;
  if (dual) {
    const double* xdb = Xdb + atom * 4 * M;
    const double* rd = rdot + idx * 4;
    a += rd[0] * xdb[m] + rd[1] * xdb[M + m] + rd[2] * xdb[2 * M + m] + rd[3] * xdb[3 * M + m];
    const double ad = rr[0] * xdb[m] + rr[1] * xdb[M + m] + rr[2] * xdb[2 * M + m] + rr[3] * xdb[3 * M + m];
    Hb[(size_t)(R + r) * M + m] = ad * inv;
  }
  Hb[(size_t)r * M + m] = a * inv;
}

// prod_force / prod_virial: dE/dR~_row = G Xbar^T / N_m + sbar e_0 ; f = dE/dd = (dE/dR~) J ;
// F_i += f, F_j -= f (F = -dE/dx), W -= d (x) f.  One warp per row.
__global__ void prod_force_kernel(Geo g, int ti, int tj, long long R, const double* __restrict__ G,
                                  const double* __restrict__ Xb, const double* __restrict__ sbar,
                                  const double* __restrict__ jac, const double* __restrict__ rij,
                                  const int* __restrict__ nl_j, double* __restrict__ force, double* __restrict__ virial) {
  const long long r = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= R) return;
  const int M = g.M;
  const int sel = g.sel[tj];
  const long long bk = r / sel;
  const int s = (int)(r % sel);
  const int b = (int)(bk / g.ncnt[ti]);
  const int k = (int)(bk % g.ncnt[ti]);
  const int i = g.atoms[g.atoms_off[ti] + k];
  const size_t idx = ((size_t)b * g.Na + i) * g.Nm + g.sec[tj] + s;
  const int j = nl_j[idx];
  if (j < 0) return;
  const double* xb = Xb + ((size_t)b * g.Na + i) * 4 * M;
  const double* gr = G + (size_t)r * M;
  double a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  for (int m = lane; m < M; m += 32) {
    const double gv = gr[m];
    a0 = fma(gv, xb[m], a0); a1 = fma(gv, xb[M + m], a1); a2 = fma(gv, xb[2 * M + m], a2); a3 = fma(gv, xb[3 * M + m], a3);
  }
  for (int o = 16; o > 0; o >>= 1) {
    a0 += __shfl_xor_sync(0xffffffffu, a0, o);
    a1 += __shfl_xor_sync(0xffffffffu, a1, o);
    a2 += __shfl_xor_sync(0xffffffffu, a2, o);
    a3 += __shfl_xor_sync(0xffffffffu, a3, o);
  }
  if (lane != 0) return;
  const double inv = 1.0 / g.Nm;
  const double rb[4] = {a0 * inv + sbar[r], a1 * inv, a2 * inv, a3 * inv};
  const double* J = jac + idx * 12;
  const double* d = rij + idx * 3;
  double f[3];
#pragma unroll
  for (int be = 0; be < 3; ++be) f[be] = rb[0] * J[be] + rb[1] * J[3 + be] + rb[2] * J[6 + be] + rb[3] * J[9 + be];
  double* Fi = force + ((size_t)b * g.Na + i) * 3;
  double* Fj = force + ((size_t)b * g.Na + j) * 3;
#pragma unroll
  for (int be = 0; be < 3; ++be) {
    atomicAdd(Fi + be, f[be]);
    atomicAdd(Fj + be, -f[be]);
  }
  double* V = virial + (size_t)b * 9;
#pragma unroll
  for (int a = 0; a < 3; ++a)
#pragma unroll
    for (int be = 0; be < 3; ++be) atomicAdd(V + 3 * a + be, -d[a] * f[be]);
}

// E_i = h_F W_out + b_out (primal rows), Edot_i = hdot_F W_out (tangent rows); one warp per row
__global__ void fit_out_kernel(long long rows, long long F, int h, const double* __restrict__ H,
                               const double* __restrict__ W, const double* __restrict__ bout, double* __restrict__ out) {
  const long long r = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= rows) return;
  double a = 0.0;
  for (int c = lane; c < h; c += 32) a = fma(H[(size_t)r * h + c], W[c], a);
  for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
  if (lane == 0) out[r] = a + (r < F ? bout[0] : 0.0);
}
// adjoint of h_F from the output seeds: Hbar = ebar (x) W_out
__global__ void fit_out_bwd_kernel(long long rows, int h, const double* __restrict__ ebar, const double* __restrict__ W,
                                   double* __restrict__ Hb) {
  const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= rows * h) return;
  Hb[e] = ebar[e / h] * W[e % h];
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
__global__ void energy_error_kernel(Geo g, FitPtrs fp, const double* __restrict__ etot, const double* __restrict__ label,
                                    double seed_scale, double* __restrict__ abs_sum) {
  __shared__ double sb[1024];
  if (threadIdx.x == 0) {
    double a = 0.0;
    for (int b = 0; b < g.nb; ++b) {
      const double E = etot[b], Y = label[b];
      a += fabs((Y - E) / g.Na);
      sb[b] = (E >= Y ? -1.0 : 1.0) * seed_scale / g.Na;
    }
    *abs_sum = a;
  }
  __syncthreads();
  for (int t = 0; t < g.nt; ++t) {
    const long long F = (long long)g.nb * g.ncnt[t];
    for (long long r = threadIdx.x; r < F; r += blockDim.x) fp.ebar[t][r] = sb[r / g.ncnt[t]];
  }
}

// force update errors on the selected atoms (Alg. 1 lines 3-6 applied to force components):
// e = F_label - F_pred, flip when F_pred >= F_label; v[b][a] accumulates the signs (tangent direction);
// seeds: Ebar = 0, Edotbar = -1/(N_a n_sel 3) because sum s F = -Edot.
__global__ void force_error_kernel(Geo g, const double* __restrict__ force, const double* __restrict__ label,
                                   const int* __restrict__ atom_idx, int n_sel, double seed, double* __restrict__ v,
                                   FitPtrs fp, double* __restrict__ abs_sum) {
  for (long long e = threadIdx.x; e < (long long)g.nb * g.Na * 3; e += blockDim.x) v[e] = 0.0;
  __syncthreads();
  if (threadIdx.x == 0) {
    double a = 0.0;
    for (int b = 0; b < g.nb; ++b)
      for (int q = 0; q < n_sel; ++q) {
        const int at = atom_idx[q];
        for (int al = 0; al < 3; ++al) {
          const size_t o = ((size_t)b * g.Na + at) * 3 + al;
          const double fp = force[o], fl = label[o];
          a += fabs(fl - fp);
          v[o] += (fp >= fl ? -1.0 : 1.0);
        }
      }
    *abs_sum = a;
  }
  for (int t = 0; t < g.nt; ++t) {
    const long long F = (long long)g.nb * g.ncnt[t];
    for (long long r = threadIdx.x; r < 2 * F; r += blockDim.x) fp.ebar[t][r] = r < F ? 0.0 : seed;
  }
}

// tangent of R~ along v: ddot = v_j - v_i ; Rdot = J ddot
__global__ void tangent_env_kernel(const double* __restrict__ jac, const int* __restrict__ nl_j, const double* __restrict__ v,
                                   int Na, int Nm, long long nslots, double* __restrict__ rdot) {
  const long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= nslots) return;
  const int j = nl_j[idx];
  double* o = rdot + idx * 4;
  if (j < 0) { o[0] = o[1] = o[2] = o[3] = 0.0; return; }
  const long long bi = idx / Nm;
  const int b = (int)(bi / Na);
  const double* vi = v + bi * 3;
  const double* vj = v + ((size_t)b * Na + j) * 3;
  const double dd[3] = {vj[0] - vi[0], vj[1] - vi[1], vj[2] - vi[2]};
  const double* J = jac + idx * 12;
#pragma unroll
  for (int k = 0; k < 4; ++k) o[k] = J[3 * k] * dd[0] + J[3 * k + 1] * dd[1] + J[3 * k + 2] * dd[2];
}

// =================================================================================================
// host orchestration
// =================================================================================================
static PairPtrs make_pp(Ctx& c, int nb) {
  PairPtrs pp{};
  for (size_t p = 0; p < c.pairs.size(); ++p) {
    pp.G[p] = c.pairs[p].H.back().as<double>();
    pp.Gb[p] = c.pairs[p].Hb.back().as<double>();
    pp.R[p] = pair_rows(c, (int)p, nb);
  }
  return pp;
}
static FitPtrs make_fp(Ctx& c, int nb) {
  FitPtrs fp{};
  for (int t = 0; t < c.nt; ++t) {
    fp.D[t] = c.fits[t].D.as<double>();
    fp.Db[t] = c.fits[t].Db.as<double>();
    fp.eout[t] = c.fits[t].eout.as<double>();
    fp.ebar[t] = c.fits[t].ebar.as<double>();
    fp.F[t] = fit_rows(c, t, nb);
  }
  return fp;
}

static fekf_status layer_fwd(const Layer& L, const double* w, long long R, const double* Ain, const double* Hprev,
                             double* Y, double* H, bool tangent, cudaStream_t s) {
  // tangent: rows [R, 2R) of every stacked buffer; the primal half provides y for (1 - y^2)
  const double* A = tangent ? Ain + (size_t)R * L.din : Ain;
  EpiFwd e;
  e.Y = tangent ? Y + (size_t)R * L.dout : Y;
  e.H = tangent ? H + (size_t)R * L.dout : H;
  e.ld = L.dout;
  e.bias = w + L.b;
  e.dt = L.dt >= 0 ? w + L.dt : nullptr;
  e.Hp = Hprev ? (tangent ? Hprev + (size_t)R * L.din : Hprev) : nullptr;
  e.ldp = L.din;
  e.skip = Hprev ? L.skip : 0;
  e.dprev = L.din;
  e.Yprim = tangent ? Y : nullptr;
  return gemm<false, false>(R, L.dout, L.din, A, L.din, w + L.W, L.dout, e, s);
}

fekf_status model_forward(Ctx& c, int nb, bool tangent, cudaStream_t s) {
  const double* w = c.w.as<double>();
  Geo g = make_geo(c, nb);
  // embedding nets
  for (size_t p = 0; p < c.pairs.size(); ++p) {
    PairNet& P = c.pairs[p];
    const long long R = pair_rows(c, (int)p, nb);
    if (R == 0) continue;
    double* hin = P.hin.as<double>();
    emb_input_kernel<<<cdiv(R, 256), 256, 0, s>>>(g, P.ti, P.tj, R, tangent ? c.rdot.as<double>() : c.em.as<double>(),
                                                   tangent ? hin + R : hin);
    FEKF_LAUNCH_CHECK();
    count_launch();
    for (size_t l = 0; l < P.L.size(); ++l) {
      const double* Ain = l == 0 ? hin : P.H[l - 1].as<double>();
      const double* Hprev = l == 0 ? nullptr : P.H[l - 1].as<double>();
      FEKF_TRY(layer_fwd(P.L[l], w, R, Ain, Hprev, P.Y[l].as<double>(), P.H[l].as<double>(), tangent, s));
    }
  }
  // descriptor
  PairPtrs pp = make_pp(c, nb);
  FitPtrs fp = make_fp(c, nb);
  const size_t smem = 8 * c.M * sizeof(double);
  const size_t Xoff = (size_t)c.B * c.Na * 4 * c.M;
  desc_fwd_kernel<<<nb * c.Na, 128, smem, s>>>(g, pp, fp, c.em.as<double>(), c.rdot.as<double>(), tangent ? 1 : 0,
                                               c.X.as<double>(), c.X.as<double>() + Xoff);
  FEKF_LAUNCH_CHECK();
  count_launch();
  // fitting nets
  for (int t = 0; t < c.nt; ++t) {
    FitNet& Fn = c.fits[t];
    const long long F = fit_rows(c, t, nb);
    if (F == 0) continue;
    for (size_t l = 0; l < Fn.L.size(); ++l) {
      const double* Ain = l == 0 ? Fn.D.as<double>() : Fn.H[l - 1].as<double>();
      const double* Hprev = l == 0 ? nullptr : Fn.H[l - 1].as<double>();
      FEKF_TRY(layer_fwd(Fn.L[l], w, F, Ain, Hprev, Fn.Y[l].as<double>(), Fn.H[l].as<double>(), tangent, s));
    }
    const int h = Fn.L.back().dout;
    const double* Hl = Fn.H.back().as<double>();
    double* eo = Fn.eout.as<double>();
    fit_out_kernel<<<cdiv(F * 32, 256), 256, 0, s>>>(F, F, h, tangent ? Hl + (size_t)F * h : Hl, w + Fn.Wout, w + Fn.bout,
                                                      tangent ? eo + F : eo);
    FEKF_LAUNCH_CHECK();
    count_launch();
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

__global__ void fill_kernel(double* p, long long n, double v) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = v;
}

fekf_status seed_force(Ctx& c, int nb, cudaStream_t s) {
  // dE_tot/dE_i = 1 for every atom: F = -dE/dx
  for (int t = 0; t < c.nt; ++t) {
    const long long F = fit_rows(c, t, nb);
    if (F == 0) continue;
    fill_kernel<<<cdiv(F, 256), 256, 0, s>>>(c.fits[t].ebar.as<double>(), F, 1.0);
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
  force_error_kernel<<<1, 256, 0, s>>>(g, c.force.as<double>(), f_label, atom_idx, n_sel, seed, c.vdir.as<double>(), fp,
                                       abs_sum);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

fekf_status tangent_env(Ctx& c, int nb, cudaStream_t s) {
  const long long n = (long long)nb * c.Na * c.Nm;
  tangent_env_kernel<<<cdiv(n, 256), 256, 0, s>>>(c.jac.as<double>(), c.nl_j.as<int>(), c.vdir.as<double>(), c.Na, c.Nm,
                                                  n, c.rdot.as<double>());
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// Reverse pass from the fitting-output seeds (ebar).  MODE_ENERGY_GRAD: weight gradients of the
// primal graph.  MODE_FORCE: adjoints down to s and R~, then forces/virials.  MODE_FORCE_JAC: weight
// gradients of the dual (primal+tangent) graph.
fekf_status model_backward(Ctx& c, int nb, Mode mode, double* gout, cudaStream_t s) {
  const double* w = c.w.as<double>();
  const bool dual = mode == MODE_FORCE_JAC;
  const bool want_w = mode != MODE_FORCE;
  Geo g = make_geo(c, nb);
  PairPtrs pp = make_pp(c, nb);
  FitPtrs fp = make_fp(c, nb);
  // ---- fitting nets ----
  for (int t = 0; t < c.nt; ++t) {
    FitNet& Fn = c.fits[t];
    const long long F = fit_rows(c, t, nb);
    if (F == 0) continue;
    const long long nF = dual ? 2 * F : F;
    const int h = Fn.L.back().dout;
    fit_out_bwd_kernel<<<cdiv(nF * h, 256), 256, 0, s>>>(nF, h, Fn.ebar.as<double>(), w + Fn.Wout, Fn.Hb.back().as<double>());
    FEKF_LAUNCH_CHECK();
    count_launch();
    if (want_w) FEKF_TRY(wgrad(c, h, 1, nF, F, Fn.H.back().as<double>(), Fn.ebar.as<double>(), gout + Fn.Wout, s));
    for (int l = (int)Fn.L.size() - 1; l >= 0; --l) {
      const Layer& L = Fn.L[l];
      const double* dt = L.dt >= 0 ? w + L.dt : nullptr;
      act_bwd_kernel<<<cdiv(F * L.dout, 256), 256, 0, s>>>(F, L.dout, Fn.Y[l].as<double>(), Fn.Hb[l].as<double>(), dt,
                                                            dual ? 1 : 0, Fn.Zb[l].as<double>());
      FEKF_LAUNCH_CHECK();
      count_launch();
      const double* Hprev = l == 0 ? Fn.D.as<double>() : Fn.H[l - 1].as<double>();
      if (want_w) {
        FEKF_TRY(wgrad(c, L.din, L.dout, nF, F, Hprev, Fn.Zb[l].as<double>(), gout + L.W, s));
        if (L.dt >= 0) FEKF_TRY(colsum_prod(c, Fn.Y[l].as<double>(), Fn.Hb[l].as<double>(), nF, L.dout, gout + L.dt, s));
      }
      double* out = l == 0 ? Fn.Db.as<double>() : Fn.Hb[l - 1].as<double>();
      EpiDgrad e{out, L.din, Fn.Hb[l].as<double>(), L.dout, l == 0 ? 0 : L.skip, L.din};
      FEKF_TRY(gemm<false, true>(nF, L.din, L.dout, Fn.Zb[l].as<double>(), L.dout, w + L.W, L.dout, e, s));
    }
  }
  // ---- descriptor (Eq. 4) ----
  const size_t Xoff = (size_t)c.B * c.Na * 4 * c.M;
  const size_t smem = (8 * c.M + 2 * c.M * c.M2) * sizeof(double);
  desc_bwd_kernel<<<nb * c.Na, 128, smem, s>>>(g, fp, c.X.as<double>(), c.X.as<double>() + Xoff, dual ? 1 : 0,
                                               c.Xb.as<double>(), c.Xb.as<double>() + Xoff);
  FEKF_LAUNCH_CHECK();
  count_launch();
  if (mode == MODE_FORCE) {
    FEKF_CHECK_CUDA(cudaMemsetAsync(c.force.p, 0, sizeof(double) * nb * c.Na * 3, s));
    FEKF_CHECK_CUDA(cudaMemsetAsync(c.virial.p, 0, sizeof(double) * nb * 9, s));
  }
  // ---- embedding nets ----
  for (size_t p = 0; p < c.pairs.size(); ++p) {
    PairNet& P = c.pairs[p];
    const long long R = pair_rows(c, (int)p, nb);
    if (R == 0) continue;
    const long long nR = dual ? 2 * R : R;
    emb_seed_kernel<<<cdiv(R * c.M, 256), 256, 0, s>>>(g, P.ti, P.tj, R, c.em.as<double>(), c.rdot.as<double>(),
                                                       c.Xb.as<double>(), c.Xb.as<double>() + Xoff, dual ? 1 : 0,
                                                       P.Hb.back().as<double>());
    FEKF_LAUNCH_CHECK();
    count_launch();
    for (int l = (int)P.L.size() - 1; l >= 0; --l) {
      const Layer& L = P.L[l];
      act_bwd_kernel<<<cdiv(R * L.dout, 256), 256, 0, s>>>(R, L.dout, P.Y[l].as<double>(), P.Hb[l].as<double>(), nullptr,
                                                            dual ? 1 : 0, P.Zb[l].as<double>());
      FEKF_LAUNCH_CHECK();
      count_launch();
      const double* Hprev = l == 0 ? P.hin.as<double>() : P.H[l - 1].as<double>();
      if (want_w) FEKF_TRY(wgrad(c, L.din, L.dout, nR, R, Hprev, P.Zb[l].as<double>(), gout + L.W, s));
      if (l > 0) {
        EpiDgrad e{P.Hb[l - 1].as<double>(), L.din, P.Hb[l].as<double>(), L.dout, L.skip, L.din};
        FEKF_TRY(gemm<false, true>(nR, L.din, L.dout, P.Zb[l].as<double>(), L.dout, w + L.W, L.dout, e, s));
      } else if (mode == MODE_FORCE) {
        FEKF_TRY(gemm<false, true>(R, 1, L.dout, P.Zb[0].as<double>(), L.dout, w + L.W, L.dout,
                                   EpiStore{P.sbar.as<double>(), 1}, s));
      }
    }
    if (mode == MODE_FORCE) {
      prod_force_kernel<<<cdiv(R * 32, 256), 256, 0, s>>>(g, P.ti, P.tj, R, P.H.back().as<double>(), c.Xb.as<double>(),
                                                          P.sbar.as<double>(), c.jac.as<double>(), c.rij.as<double>(),
                                                          c.nl_j.as<int>(), c.force.as<double>(), c.virial.as<double>());
      FEKF_LAUNCH_CHECK();
      count_launch();
    }
  }
  return FEKF_OK;
}

}  // namespace fekf
