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
// into the layer's output buffer) followed by an elementwise phase (bias, tanh, skip, activation
// adjoints) in which warp w owns rows w, w + NW, ... and the lanes own columns, with every global
// load of the phase issued before the first use.
#include <algorithm>

#include "emb.cuh"
#include "gemm.cuh"
#include "mathx.cuh"

namespace fekf {
namespace FEKF_NETNS {

// C[m][n] = sum_k A[m][k] B(k, n) over a (8 MT) x (8 NT) tile; A row-major (LDA), B(k, n) = BT ?
// B[n][k] : B[k][n] (LDB); K a multiple of 4, padded operands zero.  Warp tiles of 2x2 DMMA tiles when
// there are enough of them for every warp, else 1x2.  epi(r, c, C[r][c], C[r][c+1]) (c even) straight
// from the accumulators.
struct XfId {
  __device__ real operator()(int, int, real v) const { return v; }
};
template <bool BT, int MT, int NT, int K, int LDA, int LDB, int NW, class Epi, class Xf = XfId>
__device__ __forceinline__ void cta_mma(const real* A, const real* B, Epi epi, Xf xf = Xf()) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, fr = lane >> 2, fk = lane & 3;
  constexpr int NJ = (NT + 1) / 2;
  constexpr bool big = ((MT + 1) / 2) * NJ >= NW;
  constexpr int MB = big ? (MT + 1) / 2 : MT;
  constexpr int CNT = MB * NJ;
  for (int wt = warp; wt < CNT; wt += NW) {
    const int mi = big ? (wt % MB) * 2 : wt % MB, nj = (wt / MB) * 2;
    const bool mv = big && mi + 1 < MT, nv = nj + 1 < NT;
    real c[2][2][2];
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) c[i][j][0] = c[i][j][1] = 0.0;
    const real* a0p = A + (mi * 8 + fr) * LDA + fk;
    const real* b0p = BT ? B + (nj * 8 + fr) * LDB + fk : B + fk * LDB + nj * 8 + fr;
#pragma unroll 4
    for (int k = 0; k < K; k += 4) {
      const frag_t a0 = frag(a0p[k]);
      const frag_t a1 = frag(mv ? a0p[8 * LDA + k] : real(0));
      const frag_t b0 = frag(BT ? b0p[k] : b0p[k * LDB]);
      const frag_t b1 = frag(nv ? (BT ? b0p[8 * LDB + k] : b0p[k * LDB + 8]) : real(0));
      dmma884(c[0][0][0], c[0][0][1], a0, b0);
      if (nv) dmma884(c[0][1][0], c[0][1][1], a0, b1);
      if (mv) dmma884(c[1][0][0], c[1][0][1], a1, b0);
      if (mv && nv) dmma884(c[1][1][0], c[1][1][1], a1, b1);
    }
    // pure per-value transform of the whole warp tile first (independent chains interleave), then stores
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int h = 0; h < 2; ++h)
          if ((i == 0 || mv) && (j == 0 || nv))
            c[i][j][h] = xf((mi + i) * 8 + fr, (nj + j) * 8 + 2 * fk + h, c[i][j][h]);
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        if ((i == 1 && !mv) || (j == 1 && !nv)) continue;
        epi((mi + i) * 8 + fr, (nj + j) * 8 + 2 * fk, c[i][j][0], c[i][j][1]);
      }
  }
}

__device__ __forceinline__ void l2_prefetch(const void* p, unsigned bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// dense W [din][d] -> zero-padded SMEM image [ROWS][sld(d)], every global load of a thread issued before its
// first store (a plain strided loop serialises one L2 round trip per element)
template <int din, int d, int ROWS, int NTH>
__device__ __forceinline__ void stage_mat(real* __restrict__ dst, const real* __restrict__ src, int tid) {
  constexpr int ld = sld(d), n = ROWS * ld, IT = (n + NTH - 1) / NTH;
  real v[IT];
#pragma unroll
  for (int i = 0; i < IT; ++i) {
    const int e = tid + i * NTH, k = e / ld, j = e % ld;
    v[i] = (e < n && k < din && j < d) ? __ldg(src + k * d + j) : real(0);
  }
#pragma unroll
  for (int i = 0; i < IT; ++i) {
    const int e = tid + i * NTH;
    if (e < n) dst[e] = v[i];
  }
}
template <class W, int L, int NTH>
__device__ __forceinline__ void stage_fwd_w(real* sm, const real* __restrict__ wp, int tid) {
  if constexpr (L < W::NL) {
    stage_mat<W::din(L), W::d(L), pad4(W::din(L)), NTH>(sm + W::fW(L), wp + W::goff(L), tid);
    stage_fwd_w<W, L + 1, NTH>(sm, wp, tid);
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

// =================================================================================================
// forward
// =================================================================================================
struct EmbFwdIO {
  int Rmax;
  const int* Rdev;                    // live rows (device)
  const int* row_idx;                 // primal row -> neighbour slot
  const int* tidx;                    // tangent row -> primal row (nullptr: primal rows)
  const real* src;                  // R~ (primal) or R~-dot (tangent): the input is column 0
  real* hin;                        // s / s-dot per row (input of the layer-0 weight gradient)
  real* Y[FEKF_MAX_LAYERS];
  real* H[FEKF_MAX_LAYERS];         // may be nullptr
  const real* Yp[FEKF_MAX_LAYERS];  // tangent: primal y_l, indexed by primal row
};

// Forward, warp-tiled: every warp runs all layers of its own RT-row tiles (RT / 8 DMMA strips of 8 rows)
// with no CTA-wide barrier; W_l and b_l are staged once per (persistent, one per SM) CTA in SMEM, a
// layer's accumulators live in registers and its epilogue (bias, tanh, skip, the y / h stores) works on
// them directly, the next layer's A operand goes through the warp's own SMEM buffer (__syncwarp only).
// The next tile's inputs (row -> primal row -> slot -> s) are fetched in three dependent steps spread over
// the current tile's layers.  Tangent rows: ydot = (1 - y^2) zdot with y of the primal row, no bias.
template <class W, int L, bool tan>
__device__ __forceinline__ void wfwd_layer(const real* __restrict__ sm, real* __restrict__ wb,
                                           const EmbFwdIO& io, int r0, int R, const int (&prs)[W::RT / 8]) {
  constexpr int MS = W::RT / 8;   // 8-row DMMA strips per warp tile
  constexpr int din = W::din(L), d = W::d(L), K4 = pad4(din), NT = pad8(d) / 8, skip = W::skip(L);
  constexpr bool last = L + 1 == W::NL;
  constexpr int LDI = W::wALD((L - 1) & 1), LDO = W::wALD(L & 1), LDB = sld(d);
  const int lane = threadIdx.x & 31, fr = lane >> 2, fk = lane & 3;
  const real* in = wb + ((L - 1) & 1) * W::RT * W::wALD(0);
  real* out = wb + (L & 1) * W::RT * W::wALD(0);
  const real* Bw = sm + W::fW(L);
  const real* bs = sm + W::fB(L);
  real acc[MS][NT][2];
#pragma unroll
  for (int i = 0; i < MS; ++i)
#pragma unroll
    for (int j = 0; j < NT; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;
#pragma unroll
  for (int k = 0; k < K4; k += 4) {
    frag_t a[MS];
#pragma unroll
    for (int i = 0; i < MS; ++i) a[i] = frag(in[(8 * i + fr) * LDI + k + fk]);
#pragma unroll
    for (int j = 0; j < NT; ++j) {
      const frag_t b = frag(Bw[(k + fk) * LDB + 8 * j + fr]);
#pragma unroll
      for (int i = 0; i < MS; ++i) dmma884(acc[i][j][0], acc[i][j][1], a[i], b);
    }
  }
  real* Yl = io.Y[L];
  real* Hl = io.H[L];
  const real* Ypl = io.Yp[L];
#pragma unroll
  for (int i = 0; i < MS; ++i) {
    const int r = 8 * i + fr, row = r0 + r;
    const bool live = row < R;
    const int pr = prs[i];
    // tangent rows: the primal row's y of every output of this strip, all gathers in flight at once
    real ypv[tan ? NT : 1][2];
    if constexpr (tan) {
#pragma unroll
      for (int j = 0; j < NT; ++j)
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          const int cc = 8 * j + 2 * fk + q;
          ypv[j][q] = (cc < d && pr >= 0) ? Ypl[(size_t)pr * d + cc] : real(0);
        }
    }
#pragma unroll
    for (int j = 0; j < NT; ++j) {
      const int c = 8 * j + 2 * fk;
      real y[2], h[2];
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const int cc = c + q;
        if constexpr (tan) {
          const real yp = ypv[j][q];
          y[q] = (real(1) - yp * yp) * acc[i][j][q];
        } else {
          y[q] = tanh_r(acc[i][j][q] + bs[cc]);
        }
        const real sk = skip == 1 ? in[r * LDI + cc] : (skip == 2 ? in[r * LDI + (cc % din)] : real(0));
        h[q] = cc < d ? sk + y[q] : real(0);
      }
      if (live) {
        if ((d & 1) == 0 && c < d) {
          *reinterpret_cast<real2*>(Yl + (size_t)row * d + c) = make_real2(y[0], y[1]);
          if (last) *reinterpret_cast<real2*>(Hl + (size_t)row * d + c) = make_real2(h[0], h[1]);
        } else {
#pragma unroll
          for (int q = 0; q < 2; ++q)
            if (c + q < d) {
              Yl[(size_t)row * d + c + q] = y[q];
              if (last) Hl[(size_t)row * d + c + q] = h[q];
            }
        }
      }
      if (!last) *reinterpret_cast<real2*>(out + r * LDO + c) = make_real2(h[0], h[1]);
    }
  }
  __syncwarp();
}

// warps per CTA: the primal forward fills the SM; the tangent forward (a few % of the rows, no tanh,
// gathers of the primal y) runs 12 warps with the register room to keep a strip's gathers in flight
template <class W, bool tan>
__host__ __device__ constexpr int fwd_warps() { return tan ? (W::WNW < 12 ? W::WNW : 12) : W::WNW; }

template <class W, bool tan>
__global__ void __launch_bounds__(fwd_warps<W, tan>() * 32, 1) emb_fwd_kernel(const real* __restrict__ wp, EmbFwdIO io) {
  extern __shared__ __align__(16) real sm[];
  constexpr int NL = W::NL, RT = W::RT, NW = fwd_warps<W, tan>(), d0 = W::d(0), d0p = pad8(d0), LD0 = W::wALD(0);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, fr = lane >> 2;
  const int R = min(io.Rmax, *io.Rdev);
  // ---- stage W_l [pad4(din)][sld(d)] (zero padded) and b_l once per CTA
  for (int c = tid; c < d0p; c += NW * 32) sm[W::fW(0) + c] = c < d0 ? __ldg(wp + W::goff(0) + c) : real(0);
  if constexpr (NL >= 2) stage_fwd_w<W, 1, NW * 32>(sm, wp, tid);
#pragma unroll
  for (int l = 0; l < NL; ++l)
    for (int c = tid; c < pad8(W::d(l)); c += NW * 32)
      sm[W::fB(l) + c] = c < W::d(l) ? __ldg(wp + W::goff(l) + W::din(l) * W::d(l) + c) : real(0);
  real* wb = sm + W::WS + warp * W::WRP;
  __syncthreads();
  const int ntiles = (R + RT - 1) / RT;
  const int gw = blockIdx.x * NW + warp, nwt = gridDim.x * NW;
  // lanes 0..15 carry row lane of the tile: primal row, slot, input s (current and next tile)
  int nx_pr = -1, nx_slot = -1;
  real nx_v = 0.0;
  auto fetch_a = [&](int rn) { nx_pr = (lane < RT && rn + lane < R) ? (tan ? io.tidx[rn + lane] : rn + lane) : -1; };
  static_assert(RT == 8 || RT == 16, "warp tile rows");
  auto fetch_b = [&]() { nx_slot = nx_pr >= 0 ? io.row_idx[nx_pr] : -1; };
  auto fetch_c = [&]() { nx_v = nx_slot >= 0 ? io.src[(size_t)nx_slot * 4] : real(0); };
  if (gw < ntiles) {
    fetch_a(gw * RT);
    fetch_b();
    fetch_c();
  }
  for (int tile = gw; tile < ntiles; tile += nwt) {
    const int r0 = tile * RT, rn = r0 + nwt * RT;
    const real s_in = nx_v;
    const int cur_pr = nx_pr;
    if (lane < RT && r0 + lane < R) io.hin[r0 + lane] = s_in;
    fetch_a(rn);
    int prs[RT / 8];
#pragma unroll
    for (int i = 0; i < RT / 8; ++i) prs[i] = __shfl_sync(0xffffffffu, cur_pr, 8 * i + fr);
    // ---- layer 0 (input width 1): elementwise into buffer 0
    {
      const real* w0 = sm + W::fW(0);
      const real* b0 = sm + W::fB(0);
      constexpr int E0 = (RT * d0p + 31) / 32;
      real yp0[tan ? E0 : 1];
      if constexpr (tan) {   // the primal y_0 of every element first (gathers in flight together)
#pragma unroll
        for (int u = 0; u < E0; ++u) {
          const int e = lane + 32 * u, r = e / d0p, c = e % d0p;
          const int pr = __shfl_sync(0xffffffffu, cur_pr, r & (RT - 1));
          yp0[u] = (e < RT * d0p && c < d0 && pr >= 0) ? io.Yp[0][(size_t)pr * d0 + c] : real(0);
        }
      }
#pragma unroll
      for (int u = 0; u < E0; ++u) {
        const int e = lane + 32 * u;
        if (e >= RT * d0p) break;
        const int r = e / d0p, c = e % d0p;
        const real sv = __shfl_sync(0xffffffffu, s_in, r);
        real h = 0.0;
        if (c < d0) {
          const real z = sv * w0[c];
          if constexpr (tan) {
            h = (real(1) - yp0[u] * yp0[u]) * z;
          } else {
            h = tanh_r(z + b0[c]);
          }
          if (r0 + r < R) {
            io.Y[0][(size_t)(r0 + r) * d0 + c] = h;
            if (NL == 1) io.H[0][(size_t)(r0 + r) * d0 + c] = h;
          }
        }
        if (NL > 1) wb[r * LD0 + c] = h;
      }
      __syncwarp();
    }
    if constexpr (NL >= 2) wfwd_layer<W, 1, tan>(sm, wb, io, r0, R, prs);
    fetch_b();
    if constexpr (NL >= 3) wfwd_layer<W, 2, tan>(sm, wb, io, r0, R, prs);
    if constexpr (NL >= 4) wfwd_layer<W, 3, tan>(sm, wb, io, r0, R, prs);
    fetch_c();
  }
}

template <class W>
static fekf_status emb_forward_t(Ctx& c, int p, long long Rmax, bool tangent, cudaStream_t s) {
  PairNet& P = c.pairs[p];
  EmbFwdIO io{};
  io.Rmax = (int)Rmax;
  io.Rdev = c.rowcnt.as<int>() + (tangent ? c.pairs.size() + p : p);
  io.row_idx = P.row_idx.as<int>();
  io.tidx = tangent ? P.tidx.as<int>() : nullptr;
  io.src = tangent ? c.rdot.as<real>() : em_of(c);
  io.hin = tangent ? P.hin_t.as<real>() : P.hin.as<real>();
  for (int l = 0; l < W::NL; ++l) {
    io.Y[l] = tangent ? P.Yt[l].as<real>() : P.Y[l].as<real>();
    // only h_{L-1} (G, G-dot) is read back (descriptor); earlier h are recomputed from y where needed
    io.H[l] = l + 1 < W::NL ? nullptr : (tangent ? P.Ht[l].as<real>() : P.H[l].as<real>());
    io.Yp[l] = P.Y[l].as<real>();
  }
  static_assert(W::WNW >= 4, "emb_fwd_kernel: too few warps fit");
  const real* wp = w_of(c) + P.L[0].W;
  const long long wtiles = (Rmax + W::RT - 1) / W::RT;
  auto launch = [&](auto kern, int nw) -> fekf_status {
    const size_t smem = sizeof(real) * (W::WS + (size_t)nw * W::WRP);
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int sms = c.emb_grid_cap > 0 ? std::min(c.emb_grid_cap, num_sms()) : num_sms();
    const int grid = (int)std::max<long long>(1, std::min<long long>((wtiles + nw - 1) / nw, (long long)sms));
    kern<<<grid, nw * 32, smem, s>>>(wp, io);
    return FEKF_OK;
  };
  if (tangent) FEKF_TRY(launch(emb_fwd_kernel<W, true>, fwd_warps<W, true>()));
  else FEKF_TRY(launch(emb_fwd_kernel<W, false>, fwd_warps<W, false>()));
  FEKF_LAUNCH_CHECK();
  count_launch(1);
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
  const int* rmap;                    // MODE_FORCE_SEL: row -> primal row (active rows only; nullptr: all)
  const real* Gbar;                 // primal rows: Gbar (desc_bwd_seed_kernel)
  const real* dR;                   // forces: per-row R~ adjoint less sbar e_0 [R][4]
  const real* hin;                  // s / s-dot per row
  const real* Y[FEKF_MAX_LAYERS];   // y of this row set (h is recomputed from it)
  const real* Yp[FEKF_MAX_LAYERS];  // primal y (indexed by primal row)
  const real* Yt[FEKF_MAX_LAYERS];  // tangent y (indexed by tangent row)
  real* Hbt[FEKF_MAX_LAYERS];       // hdotbar_l: written by tangent rows, read by dual primal rows
  real* sbar;                       // forces: s-bar per primal row
  real* ws;                         // weight-gradient partials [gridDim.x][GS] (nullptr: none)
  // forces (MODE_FORCE / MODE_FORCE_SEL): dE/dR~_row = dR + sbar e_0 ; f = dE/dd = (dE/dR~) J per slot
  const real* jac;
  real* frow;
};

// weight-gradient blocks of layer L: [Wbar_L ; bbar_L] += [h_{L-1} | 1]^T zbar_L over the tile's rows
template <class W, int L>
__device__ __forceinline__ void wgrad_layer(real (&acc)[W::MAXB][2][2][2], const real* sm, int zbuf) {
  constexpr int NW = EMB_BWD_WARPS, T = W::T;
  constexpr int first = W::blk_first(L), nb = W::mblk(L) * W::nblk(L), LDA = W::augld(L), LDB = W::BLD;
  constexpr int m8 = pad8(W::din(L) + 1), n8 = pad8(W::d(L));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, fr = lane >> 2, fk = lane & 3;
  const real* A = sm + W::bAug(L);
  const real* Z = sm + W::bBuf(0) + zbuf * T * W::BLD;
#pragma unroll
  for (int q = 0; q < W::MAXB; ++q) {
    const int b = warp + NW * q - first;
    if (b >= 0 && b < nb) {
      const int m0 = (b / W::nblk(L)) * 16, n0 = (b % W::nblk(L)) * 16;
      const bool mv = m0 + 8 < m8, nv = n0 + 8 < n8;
      const real* ap = A + fk * LDA + m0 + fr;
      const real* bp = Z + fk * LDB + n0 + fr;
#pragma unroll
      for (int k = 0; k < T; k += 4) {
        const frag_t a0 = frag(ap[k * LDA]);
        const frag_t a1 = frag(mv ? ap[k * LDA + 8] : real(0));
        const frag_t b0 = frag(bp[k * LDB]);
        const frag_t b1 = frag(nv ? bp[k * LDB + 8] : real(0));
        dmma884(acc[q][0][0][0], acc[q][0][0][1], a0, b0);
        if (nv) dmma884(acc[q][0][1][0], acc[q][0][1][1], a0, b1);
        if (mv) dmma884(acc[q][1][0][0], acc[q][1][0][1], a1, b0);
        if (mv && nv) dmma884(acc[q][1][1][0], acc[q][1][1][1], a1, b1);
      }
    }
  }
}

template <class W, int L>
__device__ __forceinline__ void write_partials(const real (&acc)[W::MAXB][2][2][2], real* out) {
  constexpr int NW = EMB_BWD_WARPS;
  constexpr int first = W::blk_first(L), nb = W::mblk(L) * W::nblk(L);
  constexpr int rows = W::din(L) + 1, cols = W::d(L);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, fr = lane >> 2, fk = lane & 3;
#pragma unroll
  for (int q = 0; q < W::MAXB; ++q) {
    const int b = warp + NW * q - first;
    if (b >= 0 && b < nb) {
      const int m0 = (b / W::nblk(L)) * 16, n0 = (b % W::nblk(L)) * 16;
#pragma unroll
      for (int i = 0; i < 2; ++i)
#pragma unroll
        for (int j = 0; j < 2; ++j)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int m = m0 + 8 * i + fr, n = n0 + 8 * j + 2 * fk + h;
            if (m < rows && n < cols) out[W::goff(L) + m * cols + n] = acc[q][i][j][h];
          }
    }
  }
}

// One layer L of the reverse chain on the current tile (buffers rotate with the step from the top).
template <class W, int L>
__device__ __forceinline__ void bwd_layer(real (&acc)[W::MAXB][2][2][2], real* sm, const EmbBwdIO& io, int r0, int R,
                                          bool tan, bool wantw, const int* s_slot, const int* s_prow,
                                          const int* s_tpos, const real* s_dr) {
  constexpr int T = W::T, NW = EMB_BWD_WARPS, RPW = T / NW, BLD = W::BLD;
  constexpr int step = W::NL - 1 - L;
  constexpr int bx = (3 - step % 3) % 3, bz = (bx + 1) % 3, bn = (bx + 2) % 3;
  constexpr int d = W::d(L), w8 = pad8(d), CJ = (w8 + 31) / 32;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const real* hb = sm + W::bBuf(bx);
  real* zb = sm + W::bBuf(bz);
  // ---- zbar_L (the top layer's comes with the seed); primal y_L from shared memory (y_0 = aug_1,
  // middle layers: their copies), tangent rows' y_L of the primal row and dual terms gathered
  if constexpr (L < W::NL - 1) {
    real y[RPW][CJ], yt[RPW][CJ], hbt[RPW][CJ];
    const real* ys = L == 0 ? sm + W::bAug(1) : sm + W::bYc(L);
    constexpr int ldy = L == 0 ? W::augld(1) : sld(d);
#pragma unroll
    for (int i = 0; i < RPW; ++i)
#pragma unroll
      for (int j = 0; j < CJ; ++j) {
        const int r = warp + NW * i, c = lane + 32 * j;
        y[i][j] = yt[i][j] = hbt[i][j] = 0.0;
        if (c < d && s_slot[r] >= 0) {
          y[i][j] = (tan || io.rmap) ? io.Yp[L][(size_t)s_prow[r] * d + c] : ys[r * ldy + c];
          const int tp = s_tpos[r];
          if (tp >= 0) {
            yt[i][j] = io.Yt[L][(size_t)tp * d + c];
            hbt[i][j] = io.Hbt[L][(size_t)tp * d + c];
          }
        }
      }
#pragma unroll
    for (int i = 0; i < RPW; ++i)
#pragma unroll
      for (int j = 0; j < CJ; ++j) {
        const int r = warp + NW * i, c = lane + 32 * j;
        if (c < w8) {
          real v = 0.0;
          if (c < d && s_slot[r] >= 0)
            v = (real(1) - y[i][j] * y[i][j]) * hb[r * BLD + c] - real(2) * y[i][j] * yt[i][j] * hbt[i][j];
          zb[r * BLD + c] = v;
        }
      }
    __syncthreads();
  }
  if (wantw) wgrad_layer<W, L>(acc, sm, bz);
  if constexpr (L > 0) {
    constexpr int din = W::din(L), n8 = pad8(din), skip = W::skip(L);
    real* hn = sm + W::bBuf(bn);
    real* Hbt = tan ? io.Hbt[L - 1] : nullptr;
    // hbar_{L-1} = zbar_L W_L^T + skip^T(hbar_L) straight from the accumulators
    cta_mma<true, T / 8, n8 / 8, pad4(d), BLD, sld(d), NW>(zb, sm + W::bW(L), [&](int r, int c, real v0, real v1) {
      real v[2] = {v0, v1};
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const int cc = c + q;
        if (cc < din) {
          if (skip == 1) v[q] += hb[r * BLD + cc];
          else if (skip == 2) v[q] += hb[r * BLD + cc] + hb[r * BLD + cc + din];
          if (Hbt && r0 + r < R) Hbt[(size_t)(r0 + r) * din + cc] = v[q];
        } else {
          v[q] = 0.0;
        }
      }
      *reinterpret_cast<real2*>(hn + r * BLD + c) = make_real2(v[0], v[1]);
    });
    __syncthreads();
  } else if (io.sbar) {
    // sbar = zbar_0 . W_0 (4 threads per row), then the row's dE/dd = (dR + sbar e_0) J, stored per slot;
    // the forces and virials are gathered from these in a fixed order (force_gather_kernel, nets.cu)
    const int t = threadIdx.x;
    if (t < T * 4) {
      const int r = t >> 2, part = t & 3;
      // (sbar is written per primal row)
      const real* w0 = sm + W::bW(0);
      real sb = 0.0;
#pragma unroll
      for (int cc = part; cc < d; cc += 4) sb = fma(zb[r * BLD + cc], w0[cc], sb);
      sb += __shfl_xor_sync(0xffffffffu, sb, 1);
      sb += __shfl_xor_sync(0xffffffffu, sb, 2);
      const int row = r0 + r;
      if (part == 0 && row < R) io.sbar[s_prow[r]] = sb;
      if (io.dR && part < 3 && row < R) {
        const int be = part, slot = s_slot[r];
        const real* J = io.jac + (size_t)slot * 12;
        io.frow[(size_t)slot * 3 + be] = (s_dr[r * 4] + sb) * J[be] + s_dr[r * 4 + 1] * J[3 + be] +
                                         s_dr[r * 4 + 2] * J[6 + be] + s_dr[r * 4 + 3] * J[9 + be];
      }
    }
  }
}

// h_L of a stored row from the stored y (h_0 = y_0, h_l = skip(h_{l-1}) + y_l), all loads independent
template <class W, int L>
__device__ __forceinline__ real hval(const EmbBwdIO& io, int row, int c) {
  real v = io.Y[L][(size_t)row * W::d(L) + c];
  if constexpr (L > 0) {
    if constexpr (W::skip(L) == 1) v += hval<W, L - 1>(io, row, c);
    else if constexpr (W::skip(L) == 2) v += hval<W, L - 1>(io, row, c % W::d(L - 1));
  }
  return v;
}

// aug_L = [h_{L-1} | one] for L = 1..NL-1 and the middle layers' y copies, one load phase per tile
template <class W, int L>
__device__ __forceinline__ void build_aug(real* sm, const EmbBwdIO& io, int r0, int R, real one) {
  constexpr int T = W::T, NW = EMB_BWD_WARPS, RPW = T / NW;
  constexpr int din = W::din(L), w8 = pad8(din + 1), CJ = (w8 + 31) / 32, ld = W::augld(L);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  real v[RPW][CJ];
#pragma unroll
  for (int i = 0; i < RPW; ++i)
#pragma unroll
    for (int j = 0; j < CJ; ++j) {
      const int r = warp + NW * i, c = lane + 32 * j;
      v[i][j] = (r0 + r < R && c < din) ? hval<W, L - 1>(io, r0 + r, c) : real(0);
    }
#pragma unroll
  for (int i = 0; i < RPW; ++i)
#pragma unroll
    for (int j = 0; j < CJ; ++j) {
      const int r = warp + NW * i, c = lane + 32 * j;
      if (c < w8) sm[W::bAug(L) + r * ld + c] = (c == din && r0 + r < R) ? one : v[i][j];
    }
  if constexpr (L >= 1 && L <= W::NL - 2) {  // y_L copy (primal rows' zbar_L reads it from here)
    constexpr int d = W::d(L), d8 = pad8(d), CJY = (d8 + 31) / 32, ldy = sld(d);
    real y[RPW][CJY];
#pragma unroll
    for (int i = 0; i < RPW; ++i)
#pragma unroll
      for (int j = 0; j < CJY; ++j) {
        const int r = warp + NW * i, c = lane + 32 * j;
        y[i][j] = (r0 + r < R && c < d) ? io.Y[L][(size_t)(r0 + r) * d + c] : real(0);
      }
#pragma unroll
    for (int i = 0; i < RPW; ++i)
#pragma unroll
      for (int j = 0; j < CJY; ++j) {
        const int r = warp + NW * i, c = lane + 32 * j;
        if (c < d8) sm[W::bYc(L) + r * ldy + c] = y[i][j];
      }
  }
  if constexpr (L + 1 < W::NL) build_aug<W, L + 1>(sm, io, r0, R, one);
}

// seed of the reverse chain for the tile's rows (warp w owns rows w, w + NW): hbar_{L-1} = Gbar, written
// per row by desc_bwd_seed_kernel (primal rows: Gbar; tangent rows: Gdotbar in hdotbar_{L-1}); forces: the
// per-row R~ adjoint dR
template <class W>
__device__ __forceinline__ void seed_rows(real* sm, const EmbBwdIO& io, int r0, int R, bool tan, real* s_dr,
                                          const int* s_prow, const int* s_tpos) {
  constexpr int T = W::T, NW = EMB_BWD_WARPS, RPW = T / NW, BLD = W::BLD, NL = W::NL, M = W::M;
  constexpr int w8 = pad8(M), CJ = (w8 + 31) / 32;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const real* src = tan ? io.Hbt[NL - 1] : io.Gbar;
  real* Hb = sm + W::bBuf(0);
  real* Zb = sm + W::bBuf(1);
  real v[RPW][CJ], y[RPW][CJ], yt[RPW][CJ], hbt[RPW][CJ];
#pragma unroll
  for (int i = 0; i < RPW; ++i)
#pragma unroll
    for (int j = 0; j < CJ; ++j) {
      const int r = warp + NW * i, c = lane + 32 * j;
      v[i][j] = y[i][j] = yt[i][j] = hbt[i][j] = 0.0;
      if (c < M && r0 + r < R) {
        v[i][j] = src[(size_t)(tan ? r0 + r : s_prow[r]) * M + c];
        y[i][j] = io.Yp[NL - 1][(size_t)s_prow[r] * M + c];
        const int tp = s_tpos[r];
        if (tp >= 0) {
          yt[i][j] = io.Yt[NL - 1][(size_t)tp * M + c];
          hbt[i][j] = io.Hbt[NL - 1][(size_t)tp * M + c];
        }
      }
    }
  // hbar_{L-1} = Gbar and, in the same pass, zbar_{L-1} = (1 - y^2) hbar [- 2 y ydot hdotbar]
#pragma unroll
  for (int i = 0; i < RPW; ++i)
#pragma unroll
    for (int j = 0; j < CJ; ++j) {
      const int r = warp + NW * i, c = lane + 32 * j;
      if (c < w8) {
        Hb[r * BLD + c] = v[i][j];
        Zb[r * BLD + c] = (real(1) - y[i][j] * y[i][j]) * v[i][j] - real(2) * y[i][j] * yt[i][j] * hbt[i][j];
      }
    }
  if (io.dR && threadIdx.x < T * 4) {
    const int r = threadIdx.x >> 2;
    s_dr[threadIdx.x] = r0 + r < R ? io.dR[(size_t)s_prow[r] * 4 + (threadIdx.x & 3)] : real(0);
  }
}

template <class W>
__global__ void __launch_bounds__(EMB_BWD_WARPS * 32, 1) emb_bwd_kernel(const real* __restrict__ wp, EmbBwdIO io) {
  extern __shared__ __align__(16) real sm[];
  constexpr int T = W::T, NL = W::NL;
  __shared__ int s_slot[T], s_prow[T], s_tpos[T];
  __shared__ real s_dr[T * 4];
  const int tid = threadIdx.x;
  const bool tan = io.tidx != nullptr;
  const bool wantw = io.ws != nullptr;
  const int R = min(io.Rmax, *io.Rdev);
  // ---- stage W (zero-padded [pad8(din)][sld(d)])
  for (int c = tid; c < pad8(W::d(0)); c += blockDim.x) sm[W::bW(0) + c] = c < W::d(0) ? wp[W::goff(0) + c] : real(0);
#pragma unroll
  for (int l = 1; l < NL; ++l) {
    const int din = W::din(l), d = W::d(l), ld = sld(d), n = pad8(din) * ld;
    for (int e = tid; e < n; e += blockDim.x) {
      const int k = e / ld, j = e % ld;
      sm[W::bW(l) + e] = (k < din && j < d) ? wp[W::goff(l) + k * d + j] : real(0);
    }
  }
  real acc[W::MAXB][2][2][2];
#pragma unroll
  for (int q = 0; q < W::MAXB; ++q)
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) acc[q][i][j][0] = acc[q][i][j][1] = 0.0;
  const real one = tan ? real(0) : real(1);
  const int ntiles = (R + T - 1) / T;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * T;
    __syncthreads();
    if (tid < T) {
      const int row = r0 + tid;
      int slot = -1, pr = 0, tp = -1;
      if (row < R) {
        pr = tan ? io.tidx[row] : (io.rmap ? io.rmap[row] : row);
        slot = io.row_idx[pr];
        if (io.tpos) tp = io.tpos[row];
      }
      s_slot[tid] = slot;
      s_prow[tid] = pr;
      s_tpos[tid] = tp;
    }
    __syncthreads();
    // the next tile's stored activations (contiguous rows) on their way to L2 while this one computes
    if (tid == 0 && !io.rmap) {
      const int rn = r0 + gridDim.x * T;
      if (rn + T <= io.Rmax) {
#pragma unroll
        for (int l = 0; l < NL; ++l) l2_prefetch(io.Y[l] + (size_t)rn * W::d(l), T * W::d(l) * sizeof(real));
        l2_prefetch((tan ? io.Hbt[NL - 1] : io.Gbar) + (size_t)rn * W::M, T * W::M * sizeof(real));
        if (io.dR) l2_prefetch(io.dR + (size_t)rn * 4, T * 4 * sizeof(real));
      }
    }
    // ---- [h_{l-1} | 1] for every layer (h recomputed from the stored y) and the middle layers' y
    if (wantw && tid < T * 8) {
      const int r = tid >> 3, cc = tid & 7;
      const int row = r0 + r;
      real v = 0.0;
      if (row < R) v = cc == 0 ? io.hin[row] : (cc == 1 ? one : real(0));
      sm[W::bAug(0) + r * W::augld(0) + cc] = v;
    }
    // (rmap rows take no weight gradient and gather their y from the primal rows)
    if constexpr (NL >= 2)
      if (!io.rmap) build_aug<W, 1>(sm, io, r0, R, one);
    // ---- seed: hbar_{L-1} = Gbar, zbar_{L-1} (and, for forces, the per-row R~ adjoint)
    seed_rows<W>(sm, io, r0, R, tan, s_dr, s_prow, s_tpos);
    __syncthreads();
    if constexpr (NL >= 4) bwd_layer<W, 3>(acc, sm, io, r0, R, tan, wantw, s_slot, s_prow, s_tpos, s_dr);
    if constexpr (NL >= 3) bwd_layer<W, 2>(acc, sm, io, r0, R, tan, wantw, s_slot, s_prow, s_tpos, s_dr);
    if constexpr (NL >= 2) bwd_layer<W, 1>(acc, sm, io, r0, R, tan, wantw, s_slot, s_prow, s_tpos, s_dr);
    bwd_layer<W, 0>(acc, sm, io, r0, R, tan, wantw, s_slot, s_prow, s_tpos, s_dr);
  }
  if (wantw) {
    real* out = io.ws + (size_t)blockIdx.x * W::GS;
    if constexpr (NL >= 4) write_partials<W, 3>(acc, out);
    if constexpr (NL >= 3) write_partials<W, 2>(acc, out);
    if constexpr (NL >= 2) write_partials<W, 1>(acc, out);
    write_partials<W, 0>(acc, out);
  }
}

// g[i] += sum over the partial sets in a fixed order
__global__ void emb_wgrad_reduce_kernel(const real* __restrict__ ws, int nsets, int gsize, double* __restrict__ g) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= gsize) return;
  real a = 0.0;
  for (int k = 0; k < nsets; ++k) a += ws[(size_t)k * gsize + i];
  g[i] += (double)a;
}

template <class W>
static fekf_status launch_bwd(const real* wp, const EmbBwdIO& io, long long Rmax, int max_grid, int sms,
                              int* grid_out, cudaStream_t s) {
  constexpr size_t smem = sizeof(real) * W::B_SMEM;
  static int occ = 0;
  if (!occ) {
    FEKF_CHECK_CUDA(cudaFuncSetAttribute(emb_bwd_kernel<W>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    FEKF_CHECK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, emb_bwd_kernel<W>, EMB_BWD_WARPS * 32, smem));
    if (occ < 1) { set_error("emb_bwd_kernel: does not fit on an SM"); return FEKF_EINVAL; }
  }
  const long long tiles = (Rmax + EMB_T - 1) / EMB_T;
  const int grid = (int)std::max<long long>(1, std::min<long long>({tiles, (long long)sms * occ, (long long)max_grid}));
  emb_bwd_kernel<W><<<grid, EMB_BWD_WARPS * 32, smem, s>>>(wp, io);
  FEKF_LAUNCH_CHECK();
  count_launch();
  *grid_out = grid;
  return FEKF_OK;
}

template <class W>
static fekf_status emb_backward_t(Ctx& c, int p, long long Rmax, int mode, double* g, cudaStream_t s) {
  PairNet& P = c.pairs[p];
  const bool sel = mode == MODE_FORCE_SEL;
  const bool dual = mode == MODE_FORCE_JAC, wantw = mode != MODE_FORCE && !sel;
  const real* wp = w_of(c) + P.L[0].W;
  EmbBwdIO io{};
  io.Rmax = (int)Rmax;
  io.row_idx = P.row_idx.as<int>();
  io.Gbar = P.Hb[W::NL - 1].template as<real>();
  for (int l = 0; l < W::NL; ++l) {
    io.Yp[l] = P.Y[l].as<real>();
    io.Yt[l] = P.Yt[l].as<real>();
    io.Hbt[l] = P.Hbt[l].as<real>();
  }
  int cap = (int)std::min<size_t>(1 << 20, c.splitk_elems / (2 * (size_t)W::GS));
  if (c.emb_grid_cap > 0) cap = std::min(cap, c.emb_grid_cap);
  const int sms = c.emb_sms > 0 ? c.emb_sms : num_sms();   // split P pass: the SMs it leaves free
  real* ws = c.splitk_ws.as<real>();
  int nsets = 0;
  if (dual) {
    EmbBwdIO t = io;
    t.Rdev = c.rowcnt.as<int>() + c.pairs.size() + p;
    t.tidx = P.tidx.as<int>();
    t.hin = P.hin_t.as<real>();
    for (int l = 0; l < W::NL; ++l) t.Y[l] = P.Yt[l].as<real>();
    t.ws = ws;
    int gt = 0;
    FEKF_TRY(launch_bwd<W>(wp, t, Rmax, cap, sms, &gt, s));
    nsets += gt;
  }
  io.Rdev = c.rowcnt.as<int>() + (sel ? c.pairs.size() + p : p);
  io.rmap = sel ? P.tidx.as<int>() : nullptr;
  io.tpos = dual ? P.tpos.as<int>() : nullptr;
  io.hin = P.hin.as<real>();
  for (int l = 0; l < W::NL; ++l) io.Y[l] = P.Y[l].as<real>();
  io.sbar = (mode == MODE_FORCE || sel) ? P.sbar.as<real>() : nullptr;
  if (mode == MODE_FORCE || sel) {
    io.dR = P.Zb[0].template as<real>();
    io.jac = jac_of(c);
    io.frow = c.frow.as<real>();
  }
  io.ws = wantw ? ws + (size_t)nsets * W::GS : nullptr;
  int gp = 0;
  FEKF_TRY(launch_bwd<W>(wp, io, Rmax, cap, sms, &gp, s));
  if (wantw) {
    nsets += gp;
    emb_wgrad_reduce_kernel<<<cdiv(W::GS, 256), 256, 0, s>>>(ws, nsets, W::GS, g + P.L[0].W);
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  return FEKF_OK;
}

// ---------------------------------------------------------------------------------------------
// width dispatch: the embedding nets of the configured models (fixtures/synth.py)
// ---------------------------------------------------------------------------------------------
using EmbC2 = EmbW<25, 50, 100, 0>;   // water-64, Cu-108 (C3a), CH4 (C3b)
using EmbC1 = EmbW<8, 16, 32, 0>;     // Cu-32
using EmbPCu = EmbW<25, 25, 25, 0>;   // the paper's Cu model (26 651 parameters)
using EmbT2 = EmbW<4, 8, 16, 0>;      // tiny test model

static int emb_kind(const Ctx& c) {
  const fekf_model_cfg& m = c.m;
  if (m.n_emb != 3) return -1;
  auto is = [&](int a, int b, int d) { return m.emb[0] == a && m.emb[1] == b && m.emb[2] == d; };
  if (is(25, 50, 100)) return 0;
  if (is(8, 16, 32)) return 1;
  if (is(25, 25, 25)) return 2;
  if (is(4, 8, 16)) return 3;
  return -1;
}

bool emb_fused_ok(const Ctx& c) { return emb_kind(c) >= 0; }

fekf_status emb_forward(Ctx& c, int p, long long Rmax, bool tangent, cudaStream_t s) {
  switch (emb_kind(c)) {
    case 0: return emb_forward_t<EmbC2>(c, p, Rmax, tangent, s);
    case 1: return emb_forward_t<EmbC1>(c, p, Rmax, tangent, s);
    case 2: return emb_forward_t<EmbPCu>(c, p, Rmax, tangent, s);
    case 3: return emb_forward_t<EmbT2>(c, p, Rmax, tangent, s);
  }
  set_error("emb_forward: no fused kernel for these embedding widths");
  return FEKF_EINVAL;
}

fekf_status emb_backward(Ctx& c, int p, long long Rmax, int mode, double* g, cudaStream_t s) {
  switch (emb_kind(c)) {
    case 0: return emb_backward_t<EmbC2>(c, p, Rmax, mode, g, s);
    case 1: return emb_backward_t<EmbC1>(c, p, Rmax, mode, g, s);
    case 2: return emb_backward_t<EmbPCu>(c, p, Rmax, mode, g, s);
    case 3: return emb_backward_t<EmbT2>(c, p, Rmax, mode, g, s);
  }
  set_error("emb_backward: no fused kernel for these embedding widths");
  return FEKF_EINVAL;
}

}  // namespace FEKF_NETNS
}  // namespace fekf
