// Fused embedding-net kernels (see emb.cuh for the shared-memory layout).
//
//   forward:   y_0 = tanh(s W_0 + b_0), h_0 = y_0;
//                         y_l = tanh(h_{l-1} W_l + b_l), h_l = skip(h_{l-1}) + y_l      (reading Z12)
//   tangent rows:         ydot_l = (1 - y_l^2) (hdot_{l-1} W_l)  (y_l of the primal row), hdot_l likewise
//   backward:             hbar_{L-1} = Gbar = (R~ Xbar [+ R~dot Xdotbar]) / N_m    (row of atom i)
//                         zbar_l = (1 - y_l^2) hbar_l [- 2 y_l ydot_l hdotbar_l]    (dual rows, nets.cu)
//                         [Wbar_l ; bbar_l] += [h_{l-1} | 1]^T zbar_l                (held in registers)
//                         hbar_{l-1} = zbar_l W_l^T + skip^T(hbar_l) ;  sbar = zbar_0 . W_0 (forces)
//
// A persistent CTA walks 32-row tiles.  Each layer is a DMMA phase out of shared memory (raw products
// into the layer's output buffer) followed by an elementwise phase over all threads (bias, tanh, skip,
// activation adjoints), whose global loads are issued in batches of four per thread.
#include <algorithm>

#include "emb.cuh"
#include "gemm.cuh"

namespace fekf {

// ---------------------------------------------------------------------------------------------
// building blocks
// ---------------------------------------------------------------------------------------------
// Elementwise loop over n items: U loads in flight per thread before their uses.
template <int U, class V, class Load, class Use>
__device__ __forceinline__ void ew_loop(int n, Load load, Use use) {
  for (int base = threadIdx.x; base < n; base += blockDim.x * U) {
    V v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = base + u * blockDim.x;
      if (e < n) v[u] = load(e);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = base + u * blockDim.x;
      if (e < n) use(e, v[u]);
    }
  }
}

// out[m][n] = sum_k A[m][k] B(k, n) for the T x (8 NT) tile; A row-major (lda), B(k, n) = BT ? B[n][k] :
// B[k][n] (ldb).  K a multiple of 4, padded operands zero.  Warp tiles 2x2 (8x8 DMMA tiles) when there
// are enough of them for every warp, else 1x2.
template <bool BT>
__device__ __forceinline__ void cta_mma(const double* A, int lda, const double* B, int ldb, int MT, int NT, int K,
                                        double* out, int ldo) {
  const int nw = blockDim.x >> 5, warp = threadIdx.x >> 5, lane = threadIdx.x & 31, fr = lane >> 2, fk = lane & 3;
  const int NJ = (NT + 1) / 2;
  auto bval = [&](int k, int n) -> double { return BT ? B[n * ldb + k] : B[k * ldb + n]; };
  const int MB2 = (MT + 1) / 2;
  const bool big = MB2 * NJ >= nw;
  const int MB = big ? MB2 : MT;
  const int cnt = MB * NJ;
  for (int wt = warp; wt < cnt; wt += nw) {
    const int mi = big ? (wt % MB) * 2 : wt % MB, nj = (wt / MB) * 2;
    const bool mv = big && mi + 1 < MT, nv = nj + 1 < NT;
    double c[2][2][2];
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) c[i][j][0] = c[i][j][1] = 0.0;
#pragma unroll 2
    for (int k = 0; k < K; k += 4) {
      const double a0 = A[(mi * 8 + fr) * lda + k + fk];
      const double a1 = mv ? A[(mi * 8 + 8 + fr) * lda + k + fk] : 0.0;
      const double b0 = bval(k + fk, nj * 8 + fr);
      const double b1 = nv ? bval(k + fk, nj * 8 + 8 + fr) : 0.0;
      dmma884(c[0][0][0], c[0][0][1], a0, b0);
      if (nv) dmma884(c[0][1][0], c[0][1][1], a0, b1);
      if (mv) dmma884(c[1][0][0], c[1][0][1], a1, b0);
      if (mv && nv) dmma884(c[1][1][0], c[1][1][1], a1, b1);
    }
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        if ((i == 1 && !mv) || (j == 1 && !nv)) continue;
        const int r = (mi + i) * 8 + fr, cc = (nj + j) * 8 + 2 * fk;
        *reinterpret_cast<double2*>(out + r * ldo + cc) = make_double2(c[i][j][0], c[i][j][1]);
      }
  }
}

static int g_num_sms = 0;
static int num_sms() {
  if (!g_num_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_num_sms <= 0) g_num_sms = 148;
  }
  return g_num_sms;
}

bool emb_fused_ok(const Ctx& c) {
  for (int l = 0; l < c.m.n_emb; ++l)
    if (c.m.emb[l] > EMB_MAXW) return false;
  return true;
}

// =================================================================================================
// forward
// =================================================================================================
struct EmbFwdIO {
  int Rmax;
  const int* Rdev;                    // live rows (device)
  const int* row_idx;                 // primal row -> neighbour slot
  const int* tidx;                    // tangent row -> primal row (nullptr: primal rows)
  const double* src;                  // R~ (primal) or R~-dot (tangent): the input is column 0
  double* hin;                        // s / s-dot per row (input of the layer-0 weight gradient)
  double* Y[FEKF_MAX_LAYERS];
  double* H[FEKF_MAX_LAYERS];         // may be nullptr
  const double* Yp[FEKF_MAX_LAYERS];  // tangent: primal y_l, indexed by primal row
};

static EmbNetArgs emb_args(const PairNet& P, const double* w) {
  EmbNetArgs a{};
  a.nl = (int)P.L.size();
  int wmax[2] = {1, 1};
  for (int l = 0; l < a.nl; ++l) {
    const Layer& L = P.L[l];
    a.din[l] = L.din;
    a.dout[l] = L.dout;
    a.skip[l] = L.skip;
    a.W[l] = w + L.W;
    a.b[l] = w + L.b;
    wmax[l & 1] = std::max(wmax[l & 1], L.dout);
  }
  int off = 0;
  a.wofs[0] = off;
  off += pad8(a.dout[0]);
  for (int l = 1; l < a.nl; ++l) {
    a.wofs[l] = off;
    off += pad4(a.din[l]) * sld(a.dout[l]);
  }
  for (int l = 0; l < a.nl; ++l) {
    a.bofs[l] = off;
    off += pad8(a.dout[l]);
  }
  for (int q = 0; q < 2; ++q) {
    a.ald[q] = sld(wmax[q]);
    a.aofs[q] = off;
    off += EMB_T * a.ald[q];
  }
  a.smem_doubles = off;
  return a;
}

__global__ void __launch_bounds__(EMB_FWD_WARPS * 32) emb_fwd_kernel(EmbNetArgs a, EmbFwdIO io) {
  extern __shared__ __align__(16) double sm[];
  constexpr int T = EMB_T;
  __shared__ double s_in[T];
  __shared__ int s_prow[T];
  const int tid = threadIdx.x;
  const bool tan = io.tidx != nullptr;
  const int R = min(io.Rmax, *io.Rdev);
  // ---- stage W_l (zero-padded to [pad4(din)][sld(dout)]) and b_l
  for (int c = tid; c < pad8(a.dout[0]); c += blockDim.x) sm[a.wofs[0] + c] = c < a.dout[0] ? a.W[0][c] : 0.0;
  for (int l = 1; l < a.nl; ++l) {
    const int din = a.din[l], dout = a.dout[l], ld = sld(dout), n = pad4(din) * ld;
    const double* W = a.W[l];
    double* Ws = sm + a.wofs[l];
    for (int e = tid; e < n; e += blockDim.x) {
      const int k = e / ld, j = e % ld;
      Ws[e] = (k < din && j < dout) ? W[(size_t)k * dout + j] : 0.0;
    }
  }
  for (int l = 0; l < a.nl; ++l)
    for (int c = tid; c < pad8(a.dout[l]); c += blockDim.x) sm[a.bofs[l] + c] = c < a.dout[l] ? a.b[l][c] : 0.0;

  const int ntiles = (R + T - 1) / T;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * T;
    __syncthreads();  // weights staged / previous tile's buffers consumed
    if (tid < T) {
      const int row = r0 + tid;
      double v = 0.0;
      int pr = -1;
      if (row < R) {
        pr = tan ? io.tidx[row] : row;
        v = io.src[(size_t)io.row_idx[pr] * 4];
        io.hin[row] = v;
      }
      s_in[tid] = v;
      s_prow[tid] = pr;
    }
    __syncthreads();
    // ---- layer 0 (input width 1): elementwise
    {
      const int d = a.dout[0], w8 = pad8(d), ld = a.ald[0];
      double* out = sm + a.aofs[0];
      const double* w0 = sm + a.wofs[0];
      const double* b0 = sm + a.bofs[0];
      const double* Yp0 = io.Yp[0];
      double* Y0 = io.Y[0];
      double* H0 = io.H[0];
      ew_loop<4, double>(
          T * w8,
          [&](int e) -> double {
            const int r = e / w8, cc = e % w8;
            const int pr = s_prow[r];
            return (tan && cc < d && pr >= 0) ? Yp0[(size_t)pr * d + cc] : 0.0;
          },
          [&](int e, double yp) {
            const int r = e / w8, cc = e % w8;
            const int row = r0 + r;
            double h = 0.0;
            if (cc < d) {
              const double z = s_in[r] * w0[cc];
              const double y = tan ? (1.0 - yp * yp) * z : tanh(z + b0[cc]);
              h = y;
              if (row < R) {
                const size_t o = (size_t)row * d + cc;
                Y0[o] = y;
                if (H0) H0[o] = y;
              }
            }
            out[r * ld + cc] = h;
          });
    }
    __syncthreads();
    // ---- layers 1..nl-1: DMMA phase, then the elementwise epilogue (bias, tanh, skip) in place
    for (int l = 1; l < a.nl; ++l) {
      const int din = a.din[l], dout = a.dout[l], w8 = pad8(dout);
      const double* in = sm + a.aofs[(l - 1) & 1];
      const int ldi = a.ald[(l - 1) & 1];
      double* out = sm + a.aofs[l & 1];
      const int ldo = a.ald[l & 1];
      cta_mma<false>(in, ldi, sm + a.wofs[l], sld(dout), T / 8, w8 / 8, pad4(din), out, ldo);
      __syncthreads();
      const double* bs = sm + a.bofs[l];
      const int skip = a.skip[l];
      double* Yl = io.Y[l];
      double* Hl = io.H[l];
      const double* Ypl = io.Yp[l];
      ew_loop<4, double>(
          T * w8,
          [&](int e) -> double {
            const int r = e / w8, cc = e % w8;
            const int pr = s_prow[r];
            return (tan && cc < dout && pr >= 0) ? Ypl[(size_t)pr * dout + cc] : 0.0;
          },
          [&](int e, double yp) {
            const int r = e / w8, cc = e % w8;
            const int row = r0 + r;
            double hv = 0.0;
            if (cc < dout) {
              const double z = out[r * ldo + cc];
              const double y = tan ? (1.0 - yp * yp) * z : tanh(z + bs[cc]);
              const double sk = skip == 1 ? in[r * ldi + cc] : (skip == 2 ? in[r * ldi + (cc % din)] : 0.0);
              hv = sk + y;
              if (row < R) {
                const size_t o = (size_t)row * dout + cc;
                Yl[o] = y;
                if (Hl) Hl[o] = hv;
              }
            }
            out[r * ldo + cc] = hv;
          });
      __syncthreads();
    }
  }
}

// Forward of one pair's embedding net over its primal rows (tangent = false) or its active tangent
// rows (tangent = true).  Writes y_l and h_l of every layer and s (s-dot) per row.
fekf_status emb_forward(Ctx& c, int p, long long Rmax, bool tangent, cudaStream_t s) {
  PairNet& P = c.pairs[p];
  EmbNetArgs a = emb_args(P, c.w.as<double>());
  EmbFwdIO io{};
  io.Rmax = (int)Rmax;
  io.Rdev = c.rowcnt.as<int>() + (tangent ? c.pairs.size() + p : p);
  io.row_idx = P.row_idx.as<int>();
  io.tidx = tangent ? P.tidx.as<int>() : nullptr;
  io.src = tangent ? c.rdot.as<double>() : c.em.as<double>();
  io.hin = tangent ? P.hin_t.as<double>() : P.hin.as<double>();
  for (int l = 0; l < a.nl; ++l) {
    io.Y[l] = tangent ? P.Yt[l].as<double>() : P.Y[l].as<double>();
    io.H[l] = tangent ? P.Ht[l].as<double>() : P.H[l].as<double>();
    io.Yp[l] = P.Y[l].as<double>();
  }
  const size_t smem = sizeof(double) * a.smem_doubles;
  static size_t attr = 0;
  if (smem > attr) {
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(emb_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = smem;
  }
  int occ = 0;
  FEKF_CHECK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, emb_fwd_kernel, EMB_FWD_WARPS * 32, smem));
  if (occ < 1) { set_error("emb_fwd_kernel: does not fit on an SM"); return FEKF_EINVAL; }
  const long long tiles = (Rmax + EMB_T - 1) / EMB_T;
  const int grid = (int)std::max<long long>(1, std::min<long long>(tiles, (long long)num_sms() * occ));
  emb_fwd_kernel<<<grid, EMB_FWD_WARPS * 32, smem, s>>>(a, io);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// =================================================================================================
// backward
// =================================================================================================
struct EmbBwdIO {
  int Rmax;
  const int* Rdev;
  const int* row_idx;
  const int* tidx;                    // tangent rows: tangent row -> primal row (nullptr: primal rows)
  const int* tpos;                    // primal rows, dual: primal row -> tangent row or -1 (nullptr: none)
  const double* em;
  const double* rdot;
  const double* Xb;                   // atom X-bar
  const double* Xdb;                  // atom X-dot-bar
  const double* hin;                  // s / s-dot per row
  const double* Y[FEKF_MAX_LAYERS];   // y of this row set (h is recomputed from it)
  const double* Yp[FEKF_MAX_LAYERS];  // primal y (indexed by primal row)
  const double* Yt[FEKF_MAX_LAYERS];  // tangent y (indexed by tangent row)
  double* Hbt[FEKF_MAX_LAYERS];       // hdotbar_l: written by tangent rows, read by dual primal rows
  double* sbar;                       // forces: s-bar per primal row
  double* ws;                         // weight-gradient partials [gridDim.x][gsize] (nullptr: none)
};

static EmbBwdArgs emb_bwd_args(const Ctx& c, const PairNet& P, const double* w) {
  EmbBwdArgs a{};
  a.nl = (int)P.L.size();
  a.M = c.M;
  a.Nm = c.Nm;
  int maxw = 1;
  for (int l = 0; l < a.nl; ++l) {
    const Layer& L = P.L[l];
    a.din[l] = L.din;
    a.dout[l] = L.dout;
    a.skip[l] = L.skip;
    a.W[l] = w + L.W;
    maxw = std::max(maxw, L.dout);
  }
  int off = 0;
  a.wofs[0] = off;
  off += pad8(a.dout[0]);
  for (int l = 1; l < a.nl; ++l) {
    a.wofs[l] = off;
    off += pad8(a.din[l]) * sld(a.dout[l]);
  }
  for (int l = 0; l < a.nl; ++l) {
    a.augld[l] = sld(a.din[l] + 1);
    a.augofs[l] = off;
    off += EMB_T * a.augld[l];
  }
  a.bld = sld(maxw);
  for (int q = 0; q < 3; ++q) {
    a.bofs[q] = off;
    off += EMB_T * a.bld;
  }
  a.rofs = off;
  off += EMB_T * 8;
  a.smem_doubles = off;
  int g = 0;
  for (int l = 0; l < a.nl; ++l) {
    a.goff[l] = g;
    g += (a.din[l] + 1) * a.dout[l];
  }
  a.gsize = g;
  a.nblk = 0;
  for (int l = a.nl - 1; l >= 0; --l) {
    const int mb = (pad8(a.din[l] + 1) / 8 + 1) / 2, nb = (pad8(a.dout[l]) / 8 + 1) / 2;
    for (int i = 0; i < mb; ++i)
      for (int j = 0; j < nb; ++j) {
        if (a.nblk < EMB_BWD_WARPS * EMB_MAXB) a.blk[a.nblk] = (l << 16) | (i << 8) | j;
        ++a.nblk;
      }
  }
  return a;
}

struct ZIn { double y, yt, hbt; };

__global__ void __launch_bounds__(EMB_BWD_WARPS * 32, 1) emb_bwd_kernel(EmbBwdArgs a, EmbBwdIO io) {
  extern __shared__ __align__(16) double sm[];
  constexpr int T = EMB_T;
  constexpr int MAXB = EMB_MAXB;
  constexpr int NW = EMB_BWD_WARPS;
  __shared__ int s_slot[T], s_atom[T], s_prow[T], s_tpos[T];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, fr = lane >> 2, fk = lane & 3;
  const bool tan = io.tidx != nullptr;
  const bool wantw = io.ws != nullptr;
  const int R = min(io.Rmax, *io.Rdev);
  const int nl = a.nl, M = a.M;
  // ---- stage W (zero-padded)
  for (int c = tid; c < pad8(a.dout[0]); c += blockDim.x) sm[a.wofs[0] + c] = c < a.dout[0] ? a.W[0][c] : 0.0;
  for (int l = 1; l < nl; ++l) {
    const int din = a.din[l], dout = a.dout[l], ld = sld(dout), n = pad8(din) * ld;
    const double* W = a.W[l];
    double* Ws = sm + a.wofs[l];
    for (int e = tid; e < n; e += blockDim.x) {
      const int k = e / ld, j = e % ld;
      Ws[e] = (k < din && j < dout) ? W[(size_t)k * dout + j] : 0.0;
    }
  }
  double acc[MAXB][2][2][2];
#pragma unroll
  for (int q = 0; q < MAXB; ++q)
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) acc[q][i][j][0] = acc[q][i][j][1] = 0.0;
  const double invN = 1.0 / a.Nm;
  const double one = tan ? 0.0 : 1.0;
  double* rr = sm + a.rofs;  // [T][8]: R~ row (4) | R~-dot row (4)
  const int ntiles = (R + T - 1) / T;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * T;
    __syncthreads();
    if (tid < T) {
      const int row = r0 + tid;
      int slot = -1, atom = 0, pr = 0, tp = -1;
      if (row < R) {
        pr = tan ? io.tidx[row] : row;
        slot = io.row_idx[pr];
        atom = slot / a.Nm;
        if (io.tpos) tp = io.tpos[row];
      }
      s_slot[tid] = slot;
      s_atom[tid] = atom;
      s_prow[tid] = pr;
      s_tpos[tid] = tp;
    }
    __syncthreads();
    if (tid < T * 8) {
      const int r = tid >> 3, k = tid & 7;
      const int slot = s_slot[r];
      double v = 0.0;
      if (slot >= 0) {
        if (k < 4) v = io.em[(size_t)slot * 4 + k];
        else if (s_tpos[r] >= 0) v = io.rdot[(size_t)slot * 4 + k - 4];
      }
      rr[tid] = v;
    }
    // ---- [h_{l-1} | 1] for every layer (h recomputed from the stored y: h_0 = y_0, h_l = skip + y_l)
    if (wantw) {
      double* A0 = sm + a.augofs[0];
      if (tid < T * 8) {
        const int r = tid >> 3, cc = tid & 7;
        const int row = r0 + r;
        double v = 0.0;
        if (row < R) v = cc == 0 ? io.hin[row] : (cc == 1 ? one : 0.0);
        A0[r * a.augld[0] + cc] = v;
      }
      for (int l = 1; l < nl; ++l) {
        const int din = a.din[l], w8 = pad8(din + 1), ld = a.augld[l];
        const double* prev = sm + a.augofs[l - 1];
        const int ldp = a.augld[l - 1], skp = a.skip[l - 1], dpp = a.din[l - 1];
        const double* Yl = io.Y[l - 1];
        double* Al = sm + a.augofs[l];
        if (l >= 2) __syncthreads();  // Aug_{l-1} complete
        ew_loop<4, double>(
            T * w8,
            [&](int e) -> double {
              const int r = e / w8, cc = e % w8;
              return (r0 + r < R && cc < din) ? Yl[(size_t)(r0 + r) * din + cc] : 0.0;
            },
            [&](int e, double y) {
              const int r = e / w8, cc = e % w8;
              double v = 0.0;
              if (r0 + r < R) {
                if (cc < din) {
                  v = y;
                  if (skp == 1) v += prev[r * ldp + cc];
                  else if (skp == 2) v += prev[r * ldp + cc % dpp];
                } else if (cc == din) {
                  v = one;
                }
              }
              Al[r * ld + cc] = v;
            });
      }
    }
    __syncthreads();  // rr, Aug ready
    // ---- seed: hbar_{L-1} = Gbar
    int bx = 0, bz = 1, bn = 2;
    {
      const int w8 = pad8(M);
      double* Hb = sm + a.bofs[bx];
      double* HbtL = tan ? io.Hbt[nl - 1] : nullptr;
      const double* X1 = tan ? io.Xdb : io.Xb;
      struct XIn { double x0, x1, x2, x3, d0, d1, d2, d3; };
      ew_loop<1, XIn>(
          T * w8,
          [&](int e) -> XIn {
            const int r = e / w8, cc = e % w8;
            XIn x{};
            if (cc < M && s_slot[r] >= 0) {
              const double* xb = X1 + (size_t)s_atom[r] * 4 * M + cc;
              x.x0 = xb[0]; x.x1 = xb[M]; x.x2 = xb[2 * M]; x.x3 = xb[3 * M];
              if (!tan && s_tpos[r] >= 0) {
                const double* xd = io.Xdb + (size_t)s_atom[r] * 4 * M + cc;
                x.d0 = xd[0]; x.d1 = xd[M]; x.d2 = xd[2 * M]; x.d3 = xd[3 * M];
              }
            }
            return x;
          },
          [&](int e, const XIn& x) {
            const int r = e / w8, cc = e % w8;
            double v = 0.0;
            if (cc < M && s_slot[r] >= 0) {
              const double* q = rr + r * 8;
              v = q[0] * x.x0 + q[1] * x.x1 + q[2] * x.x2 + q[3] * x.x3;
              if (!tan && s_tpos[r] >= 0) v += q[4] * x.d0 + q[5] * x.d1 + q[6] * x.d2 + q[7] * x.d3;
              v *= invN;
              if (HbtL) HbtL[(size_t)(r0 + r) * M + cc] = v;
            }
            Hb[r * a.bld + cc] = v;
          });
    }
    __syncthreads();
    for (int l = nl - 1; l >= 0; --l) {
      const int d = a.dout[l], w8 = pad8(d);
      const double* hb = sm + a.bofs[bx];
      double* zb = sm + a.bofs[bz];
      {
        const double* Ypl = io.Yp[l];
        const double* Ytl = io.Yt[l];
        const double* Hbtl = io.Hbt[l];
        ew_loop<4, ZIn>(
            T * w8,
            [&](int e) -> ZIn {
              const int r = e / w8, cc = e % w8;
              ZIn z{0.0, 0.0, 0.0};
              if (cc < d && s_slot[r] >= 0) {
                z.y = Ypl[(size_t)s_prow[r] * d + cc];
                const int tp = s_tpos[r];
                if (tp >= 0) {
                  z.yt = Ytl[(size_t)tp * d + cc];
                  z.hbt = Hbtl[(size_t)tp * d + cc];
                }
              }
              return z;
            },
            [&](int e, const ZIn& z) {
              const int r = e / w8, cc = e % w8;
              double v = 0.0;
              if (cc < d && s_slot[r] >= 0) v = (1.0 - z.y * z.y) * hb[r * a.bld + cc] - 2.0 * z.y * z.yt * z.hbt;
              zb[r * a.bld + cc] = v;
            });
      }
      __syncthreads();
      if (wantw) {
        const double* A = sm + a.augofs[l];
        const int ldA = a.augld[l];
        const int m8 = pad8(a.din[l] + 1);
#pragma unroll
        for (int q = 0; q < MAXB; ++q) {
          const int b = warp + NW * q;
          if (b < a.nblk) {
            const int code = a.blk[b];
            if ((code >> 16) == l) {
              const int m0 = ((code >> 8) & 255) * 16, n0 = (code & 255) * 16;
              const bool mv = m0 + 8 < m8, nv = n0 + 8 < w8;
#pragma unroll 2
              for (int k = 0; k < T; k += 4) {
                const double a0 = A[(k + fk) * ldA + m0 + fr];
                const double a1 = mv ? A[(k + fk) * ldA + m0 + 8 + fr] : 0.0;
                const double b0 = zb[(k + fk) * a.bld + n0 + fr];
                const double b1 = nv ? zb[(k + fk) * a.bld + n0 + 8 + fr] : 0.0;
                dmma884(acc[q][0][0][0], acc[q][0][0][1], a0, b0);
                if (nv) dmma884(acc[q][0][1][0], acc[q][0][1][1], a0, b1);
                if (mv) dmma884(acc[q][1][0][0], acc[q][1][0][1], a1, b0);
                if (mv && nv) dmma884(acc[q][1][1][0], acc[q][1][1][1], a1, b1);
              }
            }
          }
        }
      }
      if (l > 0) {
        const int din = a.din[l], n8 = pad8(din), skip = a.skip[l];
        double* hn = sm + a.bofs[bn];
        cta_mma<true>(zb, a.bld, sm + a.wofs[l], sld(d), T / 8, n8 / 8, pad4(d), hn, a.bld);
        __syncthreads();
        double* Hbt = tan ? io.Hbt[l - 1] : nullptr;
        for (int e = tid; e < T * n8; e += blockDim.x) {
          const int r = e / n8, cc = e % n8;
          double v = 0.0;
          if (cc < din) {
            v = hn[r * a.bld + cc];
            if (skip == 1) v += hb[r * a.bld + cc];
            else if (skip == 2) v += hb[r * a.bld + cc] + hb[r * a.bld + cc + din];
            if (Hbt && r0 + r < R) Hbt[(size_t)(r0 + r) * din + cc] = v;
          }
          hn[r * a.bld + cc] = v;
        }
        __syncthreads();
        const int t = bx;
        bx = bn;
        bn = bz;
        bz = t;
      } else if (io.sbar && tid < T) {
        const int row = r0 + tid;
        if (row < R) {
          const double* w0 = sm + a.wofs[0];
          double sb = 0.0;
          for (int cc = 0; cc < d; ++cc) sb = fma(zb[tid * a.bld + cc], w0[cc], sb);
          io.sbar[row] = sb;
        }
      }
    }
  }
  if (wantw) {
    double* out = io.ws + (size_t)blockIdx.x * a.gsize;
#pragma unroll
    for (int q = 0; q < MAXB; ++q) {
      const int b = warp + NW * q;
      if (b < a.nblk) {
        const int code = a.blk[b];
        const int l = code >> 16, m0 = ((code >> 8) & 255) * 16, n0 = (code & 255) * 16;
        const int rows = a.din[l] + 1, cols = a.dout[l];
#pragma unroll
        for (int i = 0; i < 2; ++i)
#pragma unroll
          for (int j = 0; j < 2; ++j)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int m = m0 + 8 * i + fr, n = n0 + 8 * j + 2 * fk + h;
              if (m < rows && n < cols) out[a.goff[l] + m * cols + n] = acc[q][i][j][h];
            }
      }
    }
  }
}

// g[i] += sum over the partial sets in a fixed order
__global__ void emb_wgrad_reduce_kernel(const double* __restrict__ ws, int nsets, int gsize, double* __restrict__ g) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= gsize) return;
  double a = 0.0;
  for (int k = 0; k < nsets; ++k) a += ws[(size_t)k * gsize + i];
  g[i] += a;
}

static fekf_status launch_bwd(const EmbBwdArgs& a, const EmbBwdIO& io, long long Rmax, int max_grid, int* grid_out,
                              cudaStream_t s) {
  const size_t smem = sizeof(double) * a.smem_doubles;
  static size_t attr = 0;
  if (smem > attr) {
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(emb_bwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = smem;
  }
  int occ = 0;
  FEKF_CHECK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, emb_bwd_kernel, EMB_BWD_WARPS * 32, smem));
  if (occ < 1) { set_error("emb_bwd_kernel: does not fit on an SM"); return FEKF_EINVAL; }
  const long long tiles = (Rmax + EMB_T - 1) / EMB_T;
  const int grid = (int)std::max<long long>(1, std::min<long long>({tiles, (long long)num_sms() * occ, (long long)max_grid}));
  emb_bwd_kernel<<<grid, EMB_BWD_WARPS * 32, smem, s>>>(a, io);
  FEKF_LAUNCH_CHECK();
  count_launch();
  *grid_out = grid;
  return FEKF_OK;
}

bool emb_bwd_fused_ok(const Ctx& c) {
  if (!emb_fused_ok(c) || c.pairs.empty()) return false;
  EmbBwdArgs a = emb_bwd_args(c, c.pairs[0], nullptr);
  int dev = 0, maxsm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  return a.nblk <= EMB_BWD_WARPS * EMB_MAXB && sizeof(double) * a.smem_doubles <= (size_t)maxsm;
}

fekf_status emb_backward(Ctx& c, int p, long long Rmax, int mode, double* g, cudaStream_t s) {
  PairNet& P = c.pairs[p];
  EmbBwdArgs a = emb_bwd_args(c, P, c.w.as<double>());
  const bool dual = mode == MODE_FORCE_JAC, wantw = mode != MODE_FORCE;
  const size_t Xoff = (size_t)c.B * c.Na * 4 * c.M;
  EmbBwdIO io{};
  io.Rmax = (int)Rmax;
  io.row_idx = P.row_idx.as<int>();
  io.em = c.em.as<double>();
  io.rdot = c.rdot.as<double>();
  io.Xb = c.Xb.as<double>();
  io.Xdb = c.Xb.as<double>() + Xoff;
  for (int l = 0; l < a.nl; ++l) {
    io.Yp[l] = P.Y[l].as<double>();
    io.Yt[l] = P.Yt[l].as<double>();
    io.Hbt[l] = P.Hbt[l].as<double>();
  }
  const int cap = (int)std::min<size_t>(1 << 20, c.splitk_elems / (2 * (size_t)a.gsize));
  double* ws = c.splitk_ws.as<double>();
  int nsets = 0;
  if (dual) {
    EmbBwdIO t = io;
    t.Rdev = c.rowcnt.as<int>() + c.pairs.size() + p;
    t.tidx = P.tidx.as<int>();
    t.hin = P.hin_t.as<double>();
    for (int l = 0; l < a.nl; ++l) t.Y[l] = P.Yt[l].as<double>();
    t.ws = ws;
    int gt = 0;
    FEKF_TRY(launch_bwd(a, t, Rmax, cap, &gt, s));
    nsets += gt;
  }
  io.Rdev = c.rowcnt.as<int>() + p;
  io.tpos = dual ? P.tpos.as<int>() : nullptr;
  io.hin = P.hin.as<double>();
  for (int l = 0; l < a.nl; ++l) io.Y[l] = P.Y[l].as<double>();
  io.sbar = mode == MODE_FORCE ? P.sbar.as<double>() : nullptr;
  io.ws = wantw ? ws + (size_t)nsets * a.gsize : nullptr;
  int gp = 0;
  FEKF_TRY(launch_bwd(a, io, Rmax, cap, &gp, s));
  if (wantw) {
    nsets += gp;
    emb_wgrad_reduce_kernel<<<cdiv(a.gsize, 256), 256, 0, s>>>(ws, nsets, a.gsize, g + P.L[0].W);
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  return FEKF_OK;
}

}  // namespace fekf
