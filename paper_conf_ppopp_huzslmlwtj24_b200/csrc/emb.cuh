// Fused embedding-net kernels (sm_100a, fp64 DMMA m8n8k4): one CTA runs every layer of the
// embedding net G = E_{L-1} o ... o E_0(s) (skip rule: reading Z12) on a tile of rows with
// the activations resident in shared memory, instead of one GEMM launch per layer with the
// activations round-tripping through HBM.
//
// Shared-memory layout (doubles).  Every matrix uses a leading dimension ld = 16*ceil(w8/16) + 4
// (w8 = width rounded up to 8): ld = 4 (mod 16) makes both DMMA fragment patterns conflict-free,
//   row pattern        (m = lane/4, k = lane%4) at m*ld + k     (A of a forward / data-gradient GEMM)
//   transposed pattern (k = lane%4, n = lane/4) at k*ld + n     (B of a forward GEMM, A/B of a W-grad)
// because each half-warp then touches 16 distinct 8-byte bank pairs.
#pragma once
#include "model.cuh"

namespace fekf {

constexpr int EMB_MAXW = 128;   // widths handled by the fused kernels (else: per-layer GEMM path)
constexpr int EMB_T = 32;       // rows per CTA tile
constexpr int EMB_FWD_WARPS = 8;
constexpr int EMB_BWD_WARPS = 16;
constexpr int EMB_MAXB = 3;     // 2x2-tile weight-gradient blocks held per warp (C2: 38 blocks / 16 warps)

__host__ __device__ inline int pad4(int x) { return (x + 3) & ~3; }
__host__ __device__ inline int pad8(int x) { return (x + 7) & ~7; }
__host__ __device__ inline int sld(int w) { return ((pad8(w) + 15) / 16) * 16 + 4; }

struct EmbNetArgs {
  int nl;
  int din[FEKF_MAX_LAYERS], dout[FEKF_MAX_LAYERS], skip[FEKF_MAX_LAYERS];
  const double* W[FEKF_MAX_LAYERS];   // [din][dout] row-major (global, inside w)
  const double* b[FEKF_MAX_LAYERS];
  int wofs[FEKF_MAX_LAYERS];          // smem offset of W_l (l >= 1): [pad8(din)][sld(dout)]; W_0 (din 1): [dout]
  int bofs[FEKF_MAX_LAYERS];          // smem offset of b_l
  int aofs[2], ald[2];                // activation buffers: layer l output goes to buffer l & 1
  int smem_doubles;
};

struct EmbBwdArgs {
  int nl, M, Nm;
  int din[FEKF_MAX_LAYERS], dout[FEKF_MAX_LAYERS], skip[FEKF_MAX_LAYERS];
  const double* W[FEKF_MAX_LAYERS];
  int wofs[FEKF_MAX_LAYERS];          // W_l (l >= 1): [pad8(din)][sld(dout)]; W_0: [pad8(dout)]
  int augofs[FEKF_MAX_LAYERS];        // [h_{l-1} | 1] (h_{-1} = s): [T][augld]
  int augld[FEKF_MAX_LAYERS];
  int bofs[3], bld;                   // three rotating adjoint buffers [T][bld]
  int rofs;                           // per-row R~ and R~-dot [T][8]
  int smem_doubles;
  int nblk;                           // weight-gradient blocks, packed (l << 16) | (bm << 8) | bn
  int blk[EMB_BWD_WARPS * EMB_MAXB];
  int goff[FEKF_MAX_LAYERS];          // offset of [W_l ; b_l] in the pair's gradient segment
  int gsize;
};

bool emb_fused_ok(const Ctx& c);
bool emb_bwd_fused_ok(const Ctx& c);
fekf_status emb_forward(Ctx& c, int p, long long Rmax, bool tangent, cudaStream_t s);
// Reverse pass of one pair's embedding net from the atoms' X-bar (mode: nets.cu Mode).  Adds the
// weight gradients (ENERGY_GRAD, FORCE_JAC) into g, or writes s-bar per row (FORCE).
fekf_status emb_backward(Ctx& c, int p, long long Rmax, int mode, double* g, cudaStream_t s);

}  // namespace fekf
