// Fused embedding-net kernels (sm_100a; fp64 DMMA m8n8k4, fp32 the split-tf32 pair of real.cuh): every layer of the embedding net
// G = E_{L-1} o ... o E_0(s) (skip rule: reading Z12) runs in one kernel with the activations
// on chip, instead of one GEMM launch per layer with the activations round-tripping through HBM: the
// forward per warp on 16-row tiles (no CTA barrier), the backward per CTA on 32-row tiles (its weight
// gradients are split over the warps).  The kernels are compiled for the embedding widths of the
// configured models (all index math constant-folded); other widths take the per-layer GEMM path.
//
// Shared-memory layout (elements of the nets' type, real.cuh).  Every matrix uses a leading dimension ld = 16*ceil(w8/16) + 4
// (w8 = width rounded up to 8): ld = 4 (mod 16) makes both DMMA fragment patterns conflict-free,
//   row pattern        (m = lane/4, k = lane%4) at m*ld + k     (A of a forward / data-gradient GEMM)
//   transposed pattern (k = lane%4, n = lane/4) at k*ld + n     (B of a forward GEMM, A/B of a W-grad)
// because each half-warp then touches 16 distinct 8-byte bank pairs.
#pragma once
#include "model.cuh"
#include "real.cuh"

namespace fekf {
namespace FEKF_NETNS {

constexpr int EMB_T = 32;       // rows per CTA tile of the backward
constexpr int EMB_BWD_WARPS = 16;

__host__ __device__ constexpr int pad4(int x) { return (x + 3) & ~3; }
__host__ __device__ constexpr int pad8(int x) { return (x + 7) & ~7; }
__host__ __device__ constexpr int sld(int w) { return ((pad8(w) + 15) / 16) * 16 + 4; }

// Compile-time description of an embedding net (widths d_0..d_{NL-1}, input width 1) and the
// shared-memory layouts of its fused kernels.
template <int D0, int D1, int D2, int D3>
struct EmbW {
  static constexpr int T = EMB_T;
  static constexpr int NL = D3 ? 4 : (D2 ? 3 : (D1 ? 2 : 1));
  __host__ __device__ static constexpr int d(int l) { return l == 0 ? D0 : (l == 1 ? D1 : (l == 2 ? D2 : D3)); }
  __host__ __device__ static constexpr int din(int l) { return l == 0 ? 1 : d(l - 1); }
  __host__ __device__ static constexpr int skip(int l) {
    return l == 0 ? 0 : (d(l) == din(l) ? 1 : (d(l) == 2 * din(l) ? 2 : 0));
  }
  static constexpr int M = d(NL - 1);
  __host__ __device__ static constexpr int maxw(int parity) {  // parity -1: all layers
    int m = 1;
    for (int l = 0; l < NL; ++l)
      if (parity < 0 || (l & 1) == parity) m = d(l) > m ? d(l) : m;
    return m;
  }
  // ---- forward: W_0 [pad8(d0)] | W_l [pad4(din)][sld(d)] | b_l [pad8(d)] | per-warp activations
  __host__ __device__ static constexpr int fW(int l) {
    int o = pad8(D0);
    for (int k = 1; k < l; ++k) o += pad4(din(k)) * sld(d(k));
    return l == 0 ? 0 : o;
  }
  __host__ __device__ static constexpr int fB(int l) {
    int o = fW(NL);
    for (int k = 0; k < l; ++k) o += pad8(d(k));
    return o;
  }
  // ---- warp-tiled forward (emb_fwd_kernel): W_l and b_l as above ([0, fB(NL)) of the layout), then per
  // warp two activation buffers of RT rows (layer l's h in buffer l & 1, the last layer's never staged)
  static constexpr int RT = 8;                                    // rows per warp tile (one DMMA strip)
  __host__ __device__ static constexpr int wmaxw(int parity) {
    int m = 1;
    for (int l = 0; l + 1 < NL; ++l)
      if ((l & 1) == parity) m = d(l) > m ? d(l) : m;
    return m;
  }
  __host__ __device__ static constexpr int wALD(int q) { return sld(wmaxw(q)); }
  static constexpr int WS = fB(NL);                              // weights + biases (elements)
  static constexpr int WRP = RT * (wALD(0) + wALD(1));           // per-warp activations (elements)
  static constexpr int WNW_FIT = ((int)(227 * 1024 / sizeof(real)) - 32 - WS) / WRP;
  static constexpr int WNW = WNW_FIT > 24 ? 24 : WNW_FIT;        // warps per CTA (one CTA per SM)
  static constexpr int W_SMEM = WS + WNW * WRP;
  // ---- backward: W_0 | W_l [pad8(din)][sld(d)] | aug_l [T][sld(din+1)] | 3 x buf [T][BLD] | rr [T][8]
  __host__ __device__ static constexpr int bW(int l) {
    int o = pad8(D0);
    for (int k = 1; k < l; ++k) o += pad8(din(k)) * sld(d(k));
    return l == 0 ? 0 : o;
  }
  __host__ __device__ static constexpr int augld(int l) { return sld(din(l) + 1); }
  __host__ __device__ static constexpr int bAug(int l) {
    int o = bW(NL);
    for (int k = 0; k < l; ++k) o += T * augld(k);
    return o;
  }
  static constexpr int BLD = sld(maxw(-1));
  __host__ __device__ static constexpr int bBuf(int q) { return bAug(NL) + q * T * BLD; }
  // y_l of the middle layers 1..NL-2 (y_0 sits in aug_1, y_{NL-1} is consumed by the seed phase)
  __host__ __device__ static constexpr int bYc(int l) {
    int o = bBuf(3);
    for (int k = 1; k < l; ++k) o += T * sld(d(k));
    return o;
  }
  static constexpr int B_SMEM = bYc(NL > 2 ? NL - 1 : 1);
  // ---- weight-gradient blocks: 2x2 DMMA tiles of [din+1 x d] per layer, top layer first
  __host__ __device__ static constexpr int mblk(int l) { return (pad8(din(l) + 1) / 8 + 1) / 2; }
  __host__ __device__ static constexpr int nblk(int l) { return (pad8(d(l)) / 8 + 1) / 2; }
  __host__ __device__ static constexpr int blk_first(int l) {  // first block index of layer l
    int o = 0;
    for (int k = NL - 1; k > l; --k) o += mblk(k) * nblk(k);
    return o;
  }
  static constexpr int NBLK = blk_first(-1);
  __host__ __device__ static constexpr int goff(int l) {
    int o = 0;
    for (int k = 0; k < l; ++k) o += (din(k) + 1) * d(k);
    return o;
  }
  static constexpr int GS = goff(NL);
  static constexpr int MAXB = (NBLK + EMB_BWD_WARPS - 1) / EMB_BWD_WARPS;
};

// the nets' views of the context's fp64 inputs: fp32 copies for the fp32 nets (nets.cu prepare_geometry,
// model_forward), the fp64 buffers themselves otherwise
#ifdef FEKF_NETS32
inline real* em_of(const Ctx& c) { return c.em32.as<real>(); }
inline real* jac_of(const Ctx& c) { return c.jac32.as<real>(); }
inline real* rij_of(const Ctx& c) { return c.rij32.as<real>(); }
inline real* w_of(const Ctx& c) { return c.w32.as<real>(); }
#else
inline real* em_of(const Ctx& c) { return c.em.as<real>(); }
inline real* jac_of(const Ctx& c) { return c.jac.as<real>(); }
inline real* rij_of(const Ctx& c) { return c.rij.as<real>(); }
inline real* w_of(const Ctx& c) { return c.w.as<real>(); }
#endif

bool emb_fused_ok(const Ctx& c);
fekf_status emb_forward(Ctx& c, int p, long long Rmax, bool tangent, cudaStream_t s);
// Reverse pass of one pair's embedding net from the atoms' X-bar (mode: nets.cu Mode).  Adds the
// weight gradients (ENERGY_GRAD, FORCE_JAC) into g, or writes s-bar per row (FORCE).
fekf_status emb_backward(Ctx& c, int p, long long Rmax, int mode, double* g, cudaStream_t s);

}  // namespace FEKF_NETNS
}  // namespace fekf
