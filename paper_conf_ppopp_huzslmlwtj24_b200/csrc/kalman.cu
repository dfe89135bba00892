// Blocked FEKF Kalman update (Algorithm 1 lines 8-13; RLEKF blocks P:L123).
//
// Storage: every block P_i (n_i x n_i, fp64) is padded to a multiple of T = 64 and stored as its
// upper-triangle tiles (diagonal tiles full), each tile 64x64 row-major and contiguous (32 KiB).
// Symmetrisation (Alg. 1 line 11) is therefore exact by construction.
//
// Deferred corrections (a generalisation of the paper's Pg caching): the stored "base"
// B and the covariance are related by P_t = sigma (B - sum_k beta_k u_k u_k^T), k over at most `defer`
// deferred rank-1 terms (u_k = P_k g_k, beta_k = A_k / sigma_k).  One update streams the local P once:
//   - read-only pass while fewer than `defer` corrections are pending:  u_B = B g, then
//     u_t = P_t g = sigma (u_B - sum_k beta_k (u_k . g) u_k) in vector form;
//   - read-write pass otherwise: B <- sigma (B - sum_k beta_k u_k u_k^T) tile by tile in SMEM, written
//     back, and u_B = B_new g in the same pass.
// With defer = 5 a minibatch (5 updates) costs 1 read-write + 4 read-only passes instead of 5
// read-write passes.  Tiles move HBM <-> SMEM with 1-D TMA bulk copies (cp.async.bulk + mbarrier), a
// producer warp keeps STAGES tiles in flight, 8 consumer warps work in SMEM, a bulk store writes back.
// Partial u's go to a workspace slot per (item row) / (tile column) and are summed in a fixed order
// (kf_reduce_u) — no floating-point atomics, bit-reproducible.
#include <algorithm>
#include <cstdlib>
#include <cmath>
#include <numeric>

#include "kalman.cuh"

namespace fekf {

// ------------------------------------------------------------------------------------------------
// host planner
// ------------------------------------------------------------------------------------------------
void KfPlan::build(const std::vector<int>& blocks, int world_, int rank_, int seg_tiles, int row_slots, int late) {
  rps = row_slots;
  late_blocks = late;
  n = blocks;
  L = (int)n.size();
  world = world_;
  rank = rank_;
  nt.resize(L);
  off.resize(L + 1);
  tc_off.resize(L + 1);
  off[0] = 0;
  tc_off[0] = 0;
  for (int i = 0; i < L; ++i) {
    nt[i] = (n[i] + KT - 1) / KT;
    off[i + 1] = off[i] + n[i];
    tc_off[i + 1] = tc_off[i] + nt[i];
  }
  N = off[L];
  n_tc = tc_off[L];
  Npad = n_tc * KT;
  tc_blk.resize(n_tc);
  tc_c.resize(n_tc);
  for (int i = 0; i < L; ++i)
    for (int c = 0; c < nt[i]; ++c) {
      tc_blk[tc_off[i] + c] = i;
      tc_c[tc_off[i] + c] = c;
    }
  // all items (tile-row segments) in canonical order
  struct It { int blk, I, J0, nJ; };
  std::vector<It> all;
  for (int i = 0; i < L; ++i)
    for (int I = 0; I < nt[i]; ++I)
      for (int J0 = I; J0 < nt[i]; J0 += seg_tiles) all.push_back({i, I, J0, std::min(seg_tiles, nt[i] - J0)});
  total_tiles = 0;
  for (auto& it : all) total_tiles += it.nJ;
  // LPT over ranks by tile count (largest first, ties -> canonical order, lowest rank)
  std::vector<int> order(all.size());
  std::iota(order.begin(), order.end(), 0);
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) { return all[a].nJ > all[b].nJ; });
  std::vector<int64_t> load(world, 0);
  owner.assign(all.size(), 0);
  for (int k : order) {
    int r = (int)(std::min_element(load.begin(), load.end()) - load.begin());
    owner[k] = r;
    load[r] += all[k].nJ;
  }
  // this rank's items, largest first (dynamic scheduling on the device picks them in this order); the
  // early blocks' items ahead of the late blocks' items
  std::stable_partition(order.begin(), order.end(), [&](int k) { return all[k].blk >= late_blocks; });
  items.clear();
  n_early = 0;
  int64_t tile_off = 0;
  for (int k : order) {
    if (owner[k] != rank) continue;
    if (all[k].blk >= late_blocks) ++n_early;
    ItemD d;
    d.blk = all[k].blk; d.I = all[k].I; d.J0 = all[k].J0; d.nJ = all[k].nJ;
    d.tile_off = tile_off;
    d.vbase = (long long)tc_off[d.blk] * KT;
    tile_off += d.nJ;
    items.push_back(d);
  }
  tiles_local = tile_off;
  const int64_t n_items = (int64_t)items.size();
  for (int64_t k = 0; k < n_items; ++k) {
    items[k].row_slot = (int)k;   // slots row_slot*rps .. +rps-1
    items[k].col_slot0 = (long long)(rps * n_items + items[k].tile_off);
  }
  ws_slots = rps * n_items + tiles_local;
  // per-tile owner in canonical packed order (for fekf_plan_shard)
  tile_owner.clear();
  tile_owner.reserve(total_tiles);
  for (size_t k = 0; k < all.size(); ++k)
    for (int t = 0; t < all[k].nJ; ++t) tile_owner.push_back(owner[k]);
  // CSR of workspace slots per tile column: row partials of strip c (by J0), then column partials
  // of tiles (I < c, c) (by I).  Fixed order => deterministic sums.
  std::vector<std::vector<std::pair<long long, long long>>> rows(n_tc), cols(n_tc);
  for (int64_t k = 0; k < n_items; ++k) {
    const ItemD& d = items[k];
    for (int g = 0; g < rps; ++g) rows[tc_off[d.blk] + d.I].push_back({(long long)d.J0 * rps + g, (long long)d.row_slot * rps + g});
    for (int t = 0; t < d.nJ; ++t) {
      int J = d.J0 + t;
      if (J == d.I) continue;
      cols[tc_off[d.blk] + J].push_back({d.I, d.col_slot0 + t});
    }
  }
  csr_ptr.assign(n_tc + 1, 0);
  csr_idx.clear();
  for (int64_t tc = 0; tc < n_tc; ++tc) {
    std::sort(rows[tc].begin(), rows[tc].end());
    std::sort(cols[tc].begin(), cols[tc].end());
    for (auto& e : rows[tc]) csr_idx.push_back(e.second);
    for (auto& e : cols[tc]) csr_idx.push_back(e.second);
    csr_ptr[tc + 1] = (long long)csr_idx.size();
  }
}

// ------------------------------------------------------------------------------------------------
// PTX helpers (mbarrier + 1-D TMA bulk copies)
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t addr = smem_u32(bar);
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(addr),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_1d(void* dst_smem, const void* src_gmem, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst_smem)),
      "l"(src_gmem), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_store_1d(void* dst_gmem, const void* src_smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst_gmem),
               "r"(smem_u32(src_smem)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void consumer_bar() { asm volatile("bar.sync 1, 256;" ::: "memory"); }

// ------------------------------------------------------------------------------------------------
// the P pass
// ------------------------------------------------------------------------------------------------
constexpr int MAX_STAGES = 12;
constexpr int TILE_ELEMS = KT * KT;
constexpr int VS = KT + 8;   // SMEM stride of the correction vectors: DMMA fragment loads at the 2-wavefront minimum

// Storage element of P: fp64 (default) or fp32 (the fp32 variant, reading Z22).  A lane handles two
// adjacent columns of a tile row; fp64 storage: every product and correction in fp64; fp32 storage: the
// deferred corrections in fp64 (elements widened, rounded back on store), the u = P g products in fp32 with
// sums up to one lane's share of an item in fp32 and every sum beyond it in fp64 (kf_pass_kernel).
__device__ __forceinline__ double2 ld2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ double2 ld2(const float* p) {
  const float2 v = *reinterpret_cast<const float2*>(p);
  return make_double2((double)v.x, (double)v.y);
}
__device__ __forceinline__ void st2(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
__device__ __forceinline__ void st2(float* p, double2 v) {
  *reinterpret_cast<float2*>(p) = make_float2(__double2float_rn(v.x), __double2float_rn(v.y));
}
constexpr int PASS_THREADS = 288;  // 8 consumer warps + 1 producer warp
constexpr size_t PASS_SMEM = 227 * 1024 - 256;  // + 128 B of static shared memory (deferred coefficients)
// [full | empty | meta] barriers and stage metadata, column-reduction buffers (8 KiB), then the stage
// ring; a stage is one tile plus, for a read-write pass, the 2K fp64 vector segments (u_k rows I, u_k
// columns J) it needs.
constexpr size_t PASS_HDR = 2 * MAX_STAGES * sizeof(uint64_t) + MAX_STAGES * sizeof(int4) + 2 * 8 * KT * sizeof(double);

// Deferred corrections of one tile on the FP64 tensor path: C = (beta o U_I) U_J^T, a [64 x K] x [K x 64]
// product (K <= 16, zero-padded to a multiple of 4) done as m8n8k4 DMMAs, each warp owning 8-row strips;
// then B <- sigma (B - C) in place in the stage.  A scalar k-loop issued ~10 shared loads per 16 FMAs and
// made a read-write pass with 15 pending corrections compute-bound (18 ms fp64 / 27 ms fp32 for
// water-64's 41 / 21 GB instead of the 12.3 / 6.3 ms of its traffic).
__device__ __forceinline__ void dmma884k(double& d0, double& d1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
               : "+d"(d0), "+d"(d1)
               : "d"(a), "d"(b));
}
// Warp tile of the correction: NSTRIP 8-row strips x NJ 8-column chunks.  fp64 (one group of 8 warps): 2 strips
// x 4 chunks (warp w: strips 2 (w >> 1) + {0, 1}, columns 32 (w & 1) + [0, 32)), so each u_k[J] fragment load
// feeds 2 DMMAs (8-row strips x all 8 chunks per warp loaded every fragment for a single DMMA: 14.99 -> 14.36 ms
// per read-write pass in the step; 4 strips x 2 chunks measured 14.46).  fp32 (groups of 4 warps): 2 strips x 8.
#ifndef CORR_STRIPS
#define CORR_STRIPS 2
#endif
template <typename PT, int NSTRIP, int NJ>
__device__ __forceinline__ void apply_corrections(PT* t, const double (&ai)[NSTRIP][KMAX / 4], const double* vJ, int K,
                                                  double sig, int strip0, int j0, int lane) {
  const int fr = lane >> 2, fk = lane & 3;
  // strips sharing each fragment load: all of them while their accumulators fit (fp64: 2 x 4 chunks), else
  // one at a time (fp32: 8 chunks per strip)
  constexpr int SG = NSTRIP * NJ <= 8 ? NSTRIP : 1;
  constexpr int X = sizeof(PT) == 8 ? 1 : 3;
  static_assert(NJ > X, "rotation stays inside the warp's chunks");
  const int rx = fr & X;
#pragma unroll
  for (int s0 = 0; s0 < NSTRIP; s0 += SG) {
    double c[SG][NJ][2];
#pragma unroll
    for (int sp = 0; sp < SG; ++sp)
#pragma unroll
      for (int j = 0; j < NJ; ++j) c[sp][j][0] = c[sp][j][1] = 0.0;
#pragma unroll
    for (int ks = 0; ks < KMAX / 4; ++ks) {
      const int k0 = 4 * ks;
      if (k0 >= K) break;
      const int k = k0 + fk;
      const bool kv = k < K;
      double b[NJ];
#pragma unroll
      for (int j = 0; j < NJ; ++j) b[j] = kv ? vJ[k * VS + 8 * (j0 + j) + fr] : 0.0;
#pragma unroll
      for (int sp = 0; sp < SG; ++sp) {
        const double a = ai[s0 + sp][ks];   // beta_k u_k[row] of this item (registers, loaded at item start)
#pragma unroll
        for (int j = 0; j < NJ; ++j) dmma884k(c[sp][j][0], c[sp][j][1], a, b[j]);
      }
    }
    // The fragment puts 4 lanes on each of 8 rows (lane = 4 fr + fk, columns 8j + 2fk, +1).  Rows are
    // 64 elements apart, so visiting the column chunks j in the same order on every row would land the
    // lanes of one shared-memory phase (8 lanes for 16-byte fp64 pairs, 16 for 8-byte fp32 pairs) on the
    // same banks.  Row fr visits chunk q ^ (fr & X) at step q instead (X = 1 fp64, 3 fp32): the rows of a
    // phase then cover disjoint banks.  The accumulator is picked with compile-time indices (selects).
#pragma unroll
    for (int sp = 0; sp < SG; ++sp) {
      PT* row = t + (8 * (strip0 + s0 + sp) + fr) * KT + 2 * fk + 8 * j0;
#pragma unroll
      for (int q = 0; q < NJ; ++q) {
        double a0 = c[sp][q][0], a1 = c[sp][q][1];
#pragma unroll
        for (int x = 1; x <= X; ++x)
          if (rx == x) { a0 = c[sp][q ^ x][0]; a1 = c[sp][q ^ x][1]; }
        const int j = q ^ rx;
        double2 v = ld2(row + 8 * j);
        v.x = sig * (v.x - a0);
        v.y = sig * (v.y - a1);
        st2(row + 8 * j, v);
      }
    }
  }
}

// rw = 0: read-only pass, u_B = B g.  rw = 1: B <- sigma (B - sum_{k<K} beta_k u_k u_k^T) written back,
// then u_B = B_new g.  Tile-row segments are pulled from an atomic counter by a producer warp that
// streams each tile (and its g_J segment, and for rw the 2K 512-byte vector segments it needs) with TMA
// bulk copies into a ring of `nst` stages (fp64: 6 for read-only passes, fewer when corrections ride
// along; fp32 tiles are 16 KiB, so twice as many).  `stage_bytes` = tile bytes + (2T + K*VS)*8: a stage carries
// the tile's column segments u_k[J] and, on a group's first tile of an item, the item's row segment g_I; the
// row segments u_k[I] are the same for every tile of an item and are loaded once per item into the
// consumers' registers (round 1 staged both per tile: 4 stages, now 5).
//
// The 8 consumer warps form NG independent groups of 8/NG warps (named barrier 1 + group); group g
// takes the stages s = g (mod NG), so NG tiles are in flight in the consumers at once.  fp64 uses one
// group (a 32 KiB tile leaves enough time per tile); fp32 uses two: with a 16 KiB tile the per-tile
// latency chain (stage wait, loads, conversions, FMA chains, barrier, column reduction) of a single group
// no longer fits in the tile's HBM time.  Row partials: NG slots per item (a group flushes its share at
// its last tile of the item; an item shorter than NG tiles zeroes the slots of the groups it skips).
template <typename PT, int NG>
__global__ void __launch_bounds__(PASS_THREADS, 1)
kf_pass_kernel(PT* __restrict__ P, const ItemD* __restrict__ items, int n_items, int* counter,
               const double* __restrict__ gpad, const double* __restrict__ ulist, long long npad, int rw, int K,
               int nst, int stage_bytes, const KfState* st, double* __restrict__ ws, const ItemD* __restrict__ items2,
               int n_items2, int* counter2) {
  constexpr uint32_t TILE_BYTES = TILE_ELEMS * sizeof(PT);
  constexpr int NGW = 8 / NG;            // warps per group
  constexpr int RPW = KT / NGW;          // rows per warp and tile
  constexpr int GT = NGW * 32;           // threads per group
  extern __shared__ __align__(128) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + MAX_STAGES;
  int4* meta = reinterpret_cast<int4*>(empty + MAX_STAGES);
  double* colred = reinterpret_cast<double*>(meta + MAX_STAGES);
  unsigned char* stages = reinterpret_cast<unsigned char*>(colred + 2 * 8 * KT);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (!rw) K = 0;

  if (tid == 0) {
    for (int s = 0; s < nst; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    fence_mbar_init();
  }
  __syncthreads();

  if (warp == 8) {
    // ------------------------------ producer ------------------------------
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      bool own = true;
      const uint32_t bytes = TILE_BYTES + (1u + (uint32_t)K) * KT * sizeof(double);   // bytes landed
      while (true) {
        // own list first, then (split pass, late launch) the early launch's unclaimed items
        int itx = -1, lst = 0;
        if (own) {
          itx = atomicAdd(counter, 1);
          if (itx >= n_items) own = false;
        }
        if (!own) {
          itx = n_items2 > 0 ? atomicAdd(counter2, 1) : n_items2;
          if (itx >= n_items2) break;
          lst = 1;
        }
        const ItemD it = (lst ? items2 : items)[itx];
        for (int t = 0; t < it.nJ; ++t) {
          mbar_wait(&empty[s], ph ^ 1);
          // flags: 1 first tile of the item for its group, 2 last one, 4 item shorter than NG tiles
          const bool gfirst = t < NG;   // the group's first tile of the item
          meta[s] = make_int4(itx, it.J0 + t, (gfirst ? 1 : 0) | (t >= it.nJ - NG ? 2 : 0) | (it.nJ < NG ? 4 : 0), lst);
          unsigned char* st_s = stages + (size_t)s * stage_bytes;
          double* st_g = reinterpret_cast<double*>(st_s + TILE_BYTES);
          double* st_v = st_g + KT;
          mbar_arrive_tx(&full[s], bytes + (gfirst ? KT * sizeof(double) : 0u));
          tma_load_1d(st_s, P + (size_t)(it.tile_off + t) * TILE_ELEMS, TILE_BYTES, &full[s]);
          // g_J rides with its tile: no dependent global load on the consumers' per-tile path
          tma_load_1d(st_g, gpad + it.vbase + (size_t)(it.J0 + t) * KT, KT * sizeof(double), &full[s]);
          // and g_I with the group's first tile of an item (the row segment its row sums and column
          // partials need for the whole item): the item start no longer waits on global loads
          if (gfirst)
            tma_load_1d(st_v + K * VS, gpad + it.vbase + (size_t)it.I * KT, KT * sizeof(double), &full[s]);
          for (int k = 0; k < K; ++k) {   // the column segments u_k[J] (the row segments u_k[I] of an item
                                            // sit in the consumers' registers)
            const double* uk = ulist + (size_t)k * npad + it.vbase;
            tma_load_1d(st_v + k * VS, uk + (size_t)(it.J0 + t) * KT, KT * sizeof(double), &full[s]);
          }
          if (++s == nst) { s = 0; ph ^= 1; }
        }
      }
      for (int g = 0; g < NG; ++g) {  // one end marker per consumer group
        mbar_wait(&empty[s], ph ^ 1);
        meta[s] = make_int4(-1, 0, 0, 0);
        mbar_arrive(&full[s]);
        if (++s == nst) { s = 0; ph ^= 1; }
      }
    }
    return;
  }

  // ------------------------------ consumers ------------------------------
  __shared__ double s_beta[KMAX];
  if (tid < KMAX) s_beta[tid] = tid < K ? st->beta[tid] : 0.0;
  asm volatile("bar.sync 1, 256;" ::: "memory");  // consumer warps only
  const int gi = warp / NGW, wg = warp % NGW, tg = tid - gi * GT;
  const double sig = st->sigma;
  const int c0 = 2 * lane;
  double gI[RPW], racc[RPW];
  float gIf[RPW], raccf[RPW];   // fp32 storage: g_I rounded once per item, the item's row sums in fp32
  // correction warp tile (apply_corrections): NSC strips x NJC chunks; fp64 (8 warps): 4 strips x 2 chunks
  // (column quarter wg & 3), fp32 (4 warps per group): 2 strips x 8 chunks
  constexpr int NSC = NGW == 8 ? CORR_STRIPS : 2, NJC = 64 / (NGW * NSC);
  const int cstrip0 = NSC * (wg / (8 / NJC)), cj0 = NJC * (wg % (8 / NJC));
  static_assert(NGW * NSC * NJC == 64, "correction tiles cover the 8 x 8 chunks of a tile");
  double ai[NSC][KMAX / 4];
#pragma unroll
  for (int k = 0; k < RPW; ++k) { gI[k] = 0.0; gIf[k] = 0.f; racc[k] = 0.0; raccf[k] = 0.f; }
  int s = gi, prev_s = -1;
  uint32_t ph = 0;
  uint32_t tcount = 0;
  double* colg = colred + gi * (2 * NGW * KT);
  while (true) {
    mbar_wait(&full[s], ph);
    const int4 mt = meta[s];
    if (mt.x < 0) break;
    const ItemD it = (mt.w ? items2 : items)[mt.x];
    const int J = mt.y;
    const bool first = mt.z & 1, last = mt.z & 2, diag = (J == it.I);
    if (first) {
      const double* vgi = reinterpret_cast<const double*>(stages + (size_t)s * stage_bytes + TILE_BYTES) + KT + K * VS;
#pragma unroll
      for (int k = 0; k < RPW; ++k) {
        gI[k] = vgi[wg + NGW * k];
        if constexpr (sizeof(PT) == 4) gIf[k] = __double2float_rn(gI[k]);
        racc[k] = 0.0;
        raccf[k] = 0.f;
      }
      if (rw) {   // beta_k u_k[row] of this warp's correction strips, fixed for the whole item
        const int fr = lane >> 2, fk = lane & 3;
#pragma unroll
        for (int sp = 0; sp < NSC; ++sp)
#pragma unroll
          for (int ks = 0; ks < KMAX / 4; ++ks) {
            const int k = 4 * ks + fk;
            const int row = 8 * (cstrip0 + sp) + fr;
            ai[sp][ks] = k < K ? s_beta[k] * __ldg(ulist + (size_t)k * npad + it.vbase + (long long)it.I * KT + row) : 0.0;
          }
      }
    }
    PT* t = reinterpret_cast<PT*>(stages + (size_t)s * stage_bytes);
    const double* vg = reinterpret_cast<const double*>(t + TILE_ELEMS);
    const double2 gJ = *reinterpret_cast<const double2*>(vg + c0);
    const double* vJ = vg + KT;
    // fp64: the column partials in 2 independent chains of RPW/2 DFMAs (early split launch 6.13 -> 6.08 ms in
    // ncu); fp32 keeps one chain (4 chains measured 5.39 -> 5.63 ms: its 16-row tiles are register-bound)
    constexpr int CA = sizeof(PT) == 8 ? 2 : 1;
    double ca0v[CA], ca1v[CA];
#pragma unroll
    for (int q = 0; q < CA; ++q) ca0v[q] = ca1v[q] = 0.0;
    if (rw) {
      // B <- sigma (B - C) on the tensor path, a 16 x 32 (fp64) or 16 x 64 (fp32) warp tile; then the group
      // re-reads the rewritten tile (u_B = B_new g with B_new as stored) in its own element layout
      apply_corrections<PT, NSC, NJC>(t, ai, vJ, K, sig, cstrip0, cj0, lane);
      asm volatile("bar.sync %0, %1;" ::"r"(1 + gi), "r"(GT) : "memory");
    }
    if constexpr (sizeof(PT) == 4) {
      // fp32 storage: the products in fp32 (the stored element is fp32 already; g_I, g_J rounded to fp32); a
      // lane's row sums over the item's tiles (<= 64 products) and a column's RPW products per tile summed in
      // fp32, every sum across lanes, warps, items and blocks in fp64.  Widening each element to fp64 first (2 F2F + 2 DFMA per element) made the fp32
      // pass's consumers the bound of its early split launch (48 GB/s per SM).
      const float gJx = (float)gJ.x, gJy = (float)gJ.y;
      float cf0 = 0.f, cf1 = 0.f;
#pragma unroll
      for (int h = 0; h < RPW / 8; ++h) {
        float2 v[8];
#pragma unroll
        for (int q = 0; q < 8; ++q)
          v[q] = *reinterpret_cast<const float2*>(t + (wg + NGW * (8 * h + q)) * KT + c0);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          raccf[8 * h + q] = fmaf(v[q].x, gJx, fmaf(v[q].y, gJy, raccf[8 * h + q]));
          cf0 = fmaf(v[q].x, gIf[8 * h + q], cf0);
          cf1 = fmaf(v[q].y, gIf[8 * h + q], cf1);
        }
      }
      ca0v[0] = cf0;
      ca1v[0] = cf1;
    } else {
#pragma unroll
      for (int h = 0; h < RPW / 8; ++h) {
        double2 v[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) v[q] = ld2(t + (wg + NGW * (8 * h + q)) * KT + c0);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          racc[8 * h + q] = fma(v[q].x, gJ.x, fma(v[q].y, gJ.y, racc[8 * h + q]));
          ca0v[q % CA] = fma(v[q].x, gI[8 * h + q], ca0v[q % CA]);
          ca1v[q % CA] = fma(v[q].y, gI[8 * h + q], ca1v[q % CA]);
        }
      }
    }
    double ca0 = ca0v[0], ca1 = ca1v[0];
#pragma unroll
    for (int q = 1; q < CA; ++q) { ca0 += ca0v[q]; ca1 += ca1v[q]; }
    double* cr = colg + (tcount & 1) * (NGW * KT);
    if (!diag) *reinterpret_cast<double2*>(cr + wg * KT + c0) = make_double2(ca0, ca1);
    asm volatile("bar.sync %0, %1;" ::"r"(1 + gi), "r"(GT) : "memory");
    if (tg == 0) {
      if (rw) {
        fence_proxy_async();
        tma_store_1d(P + (size_t)(it.tile_off + (J - it.J0)) * TILE_ELEMS, t, TILE_BYTES);
        bulk_commit();
        if (prev_s >= 0) {
          bulk_wait_read<1>();
          mbar_arrive(&empty[prev_s]);
        }
        prev_s = s;
      } else {
        mbar_arrive(&empty[s]);  // read-only: the stage is free once every consumer of the group passed
      }
    }
    if (!diag && tg < KT) {
      double a = 0.0;
#pragma unroll
      for (int w = 0; w < NGW; ++w) a += cr[w * KT + tg];
      ws[(size_t)(it.col_slot0 + (J - it.J0)) * KT + tg] = a;
    }
    if (last) {
      double* rs = ws + ((size_t)it.row_slot * NG + gi) * KT;
#pragma unroll
      for (int q = 0; q < RPW; ++q) {
        double v = sizeof(PT) == 4 ? (double)raccf[q] : racc[q];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0) rs[wg + NGW * q] = v;
      }
      if (NG > 1 && (mt.z & 4) && tg < KT) {   // the other groups never see this item
        for (int g = 0; g < NG; ++g)
          if (g != gi) ws[((size_t)it.row_slot * NG + g) * KT + tg] = 0.0;
      }
    }
    s += NG;
    if (s >= nst) { s -= nst; ph ^= 1; }
    ++tcount;
  }
  if (tg == 0) {
    if (prev_s >= 0) {
      bulk_wait_read<0>();
      mbar_arrive(&empty[prev_s]);
    }
    bulk_wait_all();
  }
}

// ------------------------------------------------------------------------------------------------
// small kernels
// ------------------------------------------------------------------------------------------------
// g (flat, n_i per block) -> padded vector (n_t*T per block, zero pad)
__global__ void kf_pad_kernel(const double* __restrict__ g, double* __restrict__ gpad, const int* tc_blk,
                              const int* tc_c, const long long* off, const int* nblk, long long p0, long long npad) {
  long long p = p0 + (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= npad) return;
  const long long tc = p / KT;
  const int b = tc_blk[tc];
  const int loc = tc_c[tc] * KT + (int)(p % KT);
  gpad[p] = loc < nblk[b] ? g[off[b] + loc] : 0.0;
}

// u_B[tc*T + t] = sum over the CSR entries of tile column tc (fixed order)
__global__ void kf_reduce_u_kernel(const double* __restrict__ ws, const long long* __restrict__ ptr,
                                   const long long* __restrict__ idx, long long n_tc, double* __restrict__ u) {
  const long long tc = (long long)blockIdx.x * (blockDim.x / KT) + threadIdx.x / KT;
  const int t = threadIdx.x % KT;
  if (tc >= n_tc) return;
  double a = 0.0;
  for (long long e = ptr[tc]; e < ptr[tc + 1]; ++e) a += ws[(size_t)idx[e] * KT + t];
  u[tc * KT + t] = a;
}

// per tile column: dotp[0][tc] = g . u_B, dotp[1+k][tc] = g . u_k (k < K deferred vectors)
__global__ void kf_dot_kernel(const double* __restrict__ gpad, const double* __restrict__ ub,
                              const double* __restrict__ ulist, long long npad, int K, long long n_tc,
                              double* __restrict__ dotp) {
  const long long tc = (long long)blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  const int lane = threadIdx.x & 31;
  if (tc >= n_tc) return;
  const double g0 = gpad[tc * KT + lane], g1 = gpad[tc * KT + 32 + lane];
  for (int k = -1; k < K; ++k) {
    const double* u = k < 0 ? ub : ulist + (size_t)k * npad;
    double a = g0 * u[tc * KT + lane] + g1 * u[tc * KT + 32 + lane];
    for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
    if (lane == 0) dotp[(size_t)(k + 1) * n_tc + tc] = a;
  }
}

// Per block i (P is block-diagonal; the deferred terms live inside each block):
//   P_t,i = sigma (B_i - sum_k beta_k u_k,i u_k,i^T)  =>  u_t,i = sigma (u_B,i - sum_k beta_k d_k,i u_k,i),
//   d_k,i = u_k,i . g_i, and g^T u_t = sigma sum_i (g_i . u_B,i - sum_k beta_k d_k,i^2).
// kf_block_dot_kernel: dblk[k][i] = sum of the tile-column partials of block i (fixed order).
__global__ void kf_block_dot_kernel(const double* __restrict__ dotp, long long n_tc, int K, int L,
                                    const long long* __restrict__ tcoff, double* __restrict__ dblk) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= (K + 1) * L) return;
  const int k = e / L, i = e % L;
  double a = 0.0;
  for (long long tc = tcoff[i]; tc < tcoff[i + 1]; ++tc) a += dotp[(size_t)k * n_tc + tc];
  dblk[e] = a;
}

// A = 1/(c + g^T u_t) (Alg. 1 line 8, c = L*lambda or lambda), K = A u_t (line 9),
// P_{t+1} = (P_t - A u_t u_t^T)/lambda blockwise (line 10)  =>  append beta = A/sigma, sigma <- sigma/lambda;
// lambda <- nu lambda + 1 - nu (line 12, Eq. 3); w += sqrt(bs) ABE K (line 13, Eq. 2).
// rw: the pass just rewrote B = P_t, so sigma = 1 and the deferred list is empty.
__global__ void kf_finish_kernel(const double* __restrict__ dblk, int L, int K, int rw, KfState* st,
                                 double* __restrict__ cub, const double* abe, double sqrt_bs) {
  __shared__ double red[256];
  double a = 0.0;
  for (int i = threadIdx.x; i < L; i += blockDim.x) {
    double v = dblk[i];
    for (int k = 0; k < K; ++k) {
      const double d = dblk[(size_t)(k + 1) * L + i];
      const double bd = st->beta[k] * d;
      cub[(size_t)k * L + i] = bd;
      v -= bd * d;
    }
    a += v;
  }
  red[threadIdx.x] = a;
  __syncthreads();
  if (threadIdx.x == 0) {
    const double lam = st->lambda;
    const double sig = rw ? 1.0 : st->sigma;
    double gtu = 0.0;
    for (int t = 0; t < (int)blockDim.x; ++t) gtu += red[t];
    gtu *= sig;
    const double A = 1.0 / (st->c_mult * lam + gtu);
    const double e = abe ? *abe : 0.0;
    const int slot = rw ? 0 : st->npend;
    // a non-finite A or ABE (a bad batch) makes the update a no-op apart from the latched flag: the
    // deferred slot holds a zero correction (kf_vec_kernel stores u = 0 there), w, sigma and lambda stay
    const bool bad = !isfinite(A) || !isfinite(e);
    st->skip = bad ? 1 : 0;
    st->sig_cur = sig;
    st->A_last = A;
    st->coef_w = bad ? 0.0 : sqrt_bs * e * A;
    st->slot = slot;
    st->beta[slot] = bad ? 0.0 : A / sig;
    st->npend = slot + 1;
    st->sigma = bad ? sig : sig / lam;
    if (!bad) st->lambda = lam * st->nu + 1.0 - st->nu;
    st->t += 1;
    if (bad) st->flags |= 2;
  }
}

// u_t = sigma (u_B - sum_k beta_k d_k,i u_k) -> deferred slot; w += sqrt(bs) ABE A u_t
__global__ void kf_vec_kernel(const double* __restrict__ ub, double* __restrict__ ulist, long long npad, int K, int L,
                              const double* __restrict__ cub, const KfState* st, double* __restrict__ w,
                              const int* tc_blk, const int* tc_c, const long long* off, const int* nblk) {
  const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= npad) return;
  const long long tc = p / KT;
  const int b = tc_blk[tc];
  if (st->skip) {   // non-finite update: zero correction, w untouched
    ulist[(size_t)st->slot * npad + p] = 0.0;
    return;
  }
  double v = ub[p];
  for (int k = 0; k < K; ++k) v -= cub[(size_t)k * L + b] * ulist[(size_t)k * npad + p];
  v *= st->sig_cur;
  ulist[(size_t)st->slot * npad + p] = v;
  const int loc = tc_c[tc] * KT + (int)(p % KT);
  if (loc < nblk[b]) w[off[b] + loc] += st->coef_w * v;
}

__device__ __forceinline__ double deferred_value(double b, const KfState* st, const double* ulist, long long npad,
                                                 long long pr, long long pc) {
  double c = 0.0;
  for (int k = 0; k < st->npend; ++k) c += st->beta[k] * ulist[(size_t)k * npad + pr] * ulist[(size_t)k * npad + pc];
  return st->sigma * (b - c);
}

// rewrite B = P_t (flush) — one CTA per item
template <typename PT>
__global__ void kf_apply_pending_kernel(PT* __restrict__ P, const ItemD* __restrict__ items,
                                        const double* __restrict__ ulist, long long npad, const KfState* st) {
  const ItemD it = items[blockIdx.x];
  for (int t = 0; t < it.nJ; ++t) {
    PT* tile = P + (size_t)(it.tile_off + t) * TILE_ELEMS;
    const int J = it.J0 + t;
    for (int e = threadIdx.x; e < TILE_ELEMS; e += blockDim.x) {
      const int r = e / KT, c = e % KT;
      tile[e] = (PT)deferred_value((double)tile[e], st, ulist, npad, it.vbase + (long long)it.I * KT + r,
                                   it.vbase + (long long)J * KT + c);
    }
  }
}
__global__ void kf_clear_pending_kernel(KfState* st) {
  st->npend = 0;
  st->sigma = 1.0;
}

// P = I on the valid part of every block, 0 on the padding
template <typename PT>
__global__ void kf_init_kernel(PT* __restrict__ P, const ItemD* __restrict__ items, const int* nblk) {
  const ItemD it = items[blockIdx.x];
  const int n = nblk[it.blk];
  for (int t = 0; t < it.nJ; ++t) {
    PT* tile = P + (size_t)(it.tile_off + t) * TILE_ELEMS;
    const int J = it.J0 + t;
    for (int e = threadIdx.x; e < TILE_ELEMS; e += blockDim.x) {
      const int r = e / KT, c = e % KT;
      const int gr = it.I * KT + r, gc = J * KT + c;
      tile[e] = (gr == gc && gr < n) ? (PT)1 : (PT)0;
    }
  }
}

// dense <-> packed for one block (tests / checkpoints); get applies the deferred corrections on the fly
template <typename PT>
__global__ void kf_get_block_kernel(const PT* __restrict__ P, const ItemD* __restrict__ items, int blk, int n,
                                    const double* __restrict__ ulist, long long npad, const KfState* st,
                                    double* __restrict__ dst) {
  const ItemD it = items[blockIdx.x];
  if (it.blk != blk) return;
  for (int t = 0; t < it.nJ; ++t) {
    const PT* tile = P + (size_t)(it.tile_off + t) * TILE_ELEMS;
    const int J = it.J0 + t;
    for (int e = threadIdx.x; e < TILE_ELEMS; e += blockDim.x) {
      const int r = e / KT, c = e % KT;
      const int gr = it.I * KT + r, gc = J * KT + c;
      if (gr >= n || gc >= n) continue;
      const double v = deferred_value((double)tile[e], st, ulist, npad, it.vbase + gr, it.vbase + gc);
      dst[(size_t)gr * n + gc] = v;
      if (J != it.I) dst[(size_t)gc * n + gr] = v;
    }
  }
}
template <typename PT>
__global__ void kf_set_block_kernel(PT* __restrict__ P, const ItemD* __restrict__ items, int blk, int n,
                                    const double* __restrict__ src) {
  const ItemD it = items[blockIdx.x];
  if (it.blk != blk) return;
  for (int t = 0; t < it.nJ; ++t) {
    PT* tile = P + (size_t)(it.tile_off + t) * TILE_ELEMS;
    const int J = it.J0 + t;
    for (int e = threadIdx.x; e < TILE_ELEMS; e += blockDim.x) {
      const int r = e / KT, c = e % KT;
      const int gr = it.I * KT + r, gc = J * KT + c;
      tile[e] = (PT)((gr < n && gc < n) ? src[(size_t)gr * n + gc] : 0.0);
    }
  }
}

// ------------------------------------------------------------------------------------------------
// host side of fekf_kf
// ------------------------------------------------------------------------------------------------
static int num_sms() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms;
}

fekf_status Kf::create(const std::vector<int>& blocks, const fekf_opt_cfg& o, fekf_comm* c, int world_o, int rank_o) {
  opt = o;
  comm = c;
  defer = std::max(1, std::min(KMAX, o.p_defer > 0 ? o.p_defer : 1));
  if (o.precision != 0 && o.precision != 32 && o.precision != 64) {
    set_error("kf_create: precision must be 32 or 64");
    return FEKF_EINVAL;
  }
  p32 = o.precision == 32;
  int world = 1, rank = 0;
  if (o.p_mode != 0 && o.p_mode != 1) {
    set_error("kf_create: p_mode must be 0 (sharded) or 1 (replicated)");
    return FEKF_EINVAL;
  }
  replicated = o.p_mode == 1;
  if (!replicated) {
    if (comm) { world = comm_world(comm); rank = comm_rank(comm); }
    else if (world_o > 0) { world = world_o; rank = rank_o; }
  }
  ng = p32 ? 2 : 1;   // fp64: one group (measured: a second group slows the read-write pass)
  if (const char* e = getenv("FEKF_FP64_NG")) if (!p32 && atoi(e) == 2) ng = 2;   // experiments
  plan.build(blocks, world, rank, SEG_TILES, ng, std::min<int>(late_blocks, (int)blocks.size()));
  const KfPlan& p = plan;
  FEKF_TRY(dalloc(P, (size_t)p.tiles_local * TILE_ELEMS * elem() + 16));
  FEKF_TRY(dalloc(items_d, std::max<size_t>(1, p.items.size()) * sizeof(ItemD)));
  FEKF_TRY(dalloc(ws, (size_t)std::max<int64_t>(1, p.ws_slots) * KT * sizeof(double)));
  FEKF_TRY(dalloc(gpad, p.Npad * sizeof(double)));
  FEKF_TRY(dalloc(ub, p.Npad * sizeof(double)));
  FEKF_TRY(dalloc(ulist, (size_t)KMAX * p.Npad * sizeof(double)));
  FEKF_TRY(dalloc(dotp, (size_t)(1 + KMAX) * p.n_tc * sizeof(double)));
  FEKF_TRY(dalloc(csr_ptr, (p.n_tc + 1) * sizeof(long long)));
  FEKF_TRY(dalloc(csr_idx, std::max<size_t>(1, p.csr_idx.size()) * sizeof(long long)));
  FEKF_TRY(dalloc(tc_blk, p.n_tc * sizeof(int)));
  FEKF_TRY(dalloc(tc_c, p.n_tc * sizeof(int)));
  FEKF_TRY(dalloc(off_d, (p.L + 1) * sizeof(long long)));
  FEKF_TRY(dalloc(n_d, p.L * sizeof(int)));
  FEKF_TRY(dalloc(state, sizeof(KfState)));
  FEKF_TRY(dalloc(counter, sizeof(int)));
  FEKF_TRY(dalloc(counter2, sizeof(int)));
  FEKF_TRY(dalloc(tcoff_d, (p.L + 1) * sizeof(long long)));
  FEKF_TRY(dalloc(dblk, (size_t)(1 + KMAX) * p.L * sizeof(double)));
  FEKF_TRY(dalloc(cub, (size_t)KMAX * p.L * sizeof(double)));
  FEKF_CHECK_CUDA(cudaMemcpy(tcoff_d.p, p.tc_off.data(), (p.L + 1) * sizeof(long long), cudaMemcpyHostToDevice));
  if (!p.items.empty())
    FEKF_CHECK_CUDA(cudaMemcpy(items_d.p, p.items.data(), p.items.size() * sizeof(ItemD), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(csr_ptr.p, p.csr_ptr.data(), (p.n_tc + 1) * sizeof(long long), cudaMemcpyHostToDevice));
  if (!p.csr_idx.empty())
    FEKF_CHECK_CUDA(cudaMemcpy(csr_idx.p, p.csr_idx.data(), p.csr_idx.size() * sizeof(long long), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(tc_blk.p, p.tc_blk.data(), p.n_tc * sizeof(int), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(tc_c.p, p.tc_c.data(), p.n_tc * sizeof(int), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(off_d.p, p.off.data(), (p.L + 1) * sizeof(long long), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(n_d.p, p.n.data(), p.L * sizeof(int), cudaMemcpyHostToDevice));
  KfState s{};
  s.lambda = o.lambda0;
  s.nu = o.nu;
  s.sigma = 1.0;
  s.c_mult = o.noise_mode == 0 ? (double)p.L : 1.0;
  FEKF_CHECK_CUDA(cudaMemcpy(state.p, &s, sizeof(KfState), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemset(ulist.p, 0, (size_t)KMAX * p.Npad * sizeof(double)));
  // the work counters are zeroed before every launch (stream-ordered memset, a graph node when captured);
  // zeroing them once here too keeps compute-sanitizer's initcheck, which does not see graph memset nodes,
  // free of false reports
  FEKF_CHECK_CUDA(cudaMemset(counter.p, 0, sizeof(int)));
  FEKF_CHECK_CUDA(cudaMemset(counter2.p, 0, sizeof(int)));
  FEKF_CHECK_CUDA(cudaFuncSetAttribute(kf_pass_kernel<double, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PASS_SMEM));
  FEKF_CHECK_CUDA(cudaFuncSetAttribute(kf_pass_kernel<float, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PASS_SMEM));
  FEKF_CHECK_CUDA(cudaFuncSetAttribute(kf_pass_kernel<double, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PASS_SMEM));
  if (!p.items.empty()) {
    if (p32) kf_init_kernel<<<(unsigned)p.items.size(), 256>>>(P.as<float>(), items_d.as<ItemD>(), n_d.as<int>());
    else kf_init_kernel<<<(unsigned)p.items.size(), 256>>>(P.as<double>(), items_d.as<ItemD>(), n_d.as<int>());
    FEKF_LAUNCH_CHECK();
  }
  if (split_sms > 0 && plan.n_early > 0) {
    // highest priority: the early pass's CTAs take SMs ahead of the reverse pass's queued CTAs
    int lo = 0, hi = 0;
    FEKF_CHECK_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    FEKF_CHECK_CUDA(cudaStreamCreateWithPriority(&side, cudaStreamNonBlocking, hi));
    FEKF_CHECK_CUDA(cudaEventCreateWithFlags(&ev_early, cudaEventDisableTiming));
    FEKF_CHECK_CUDA(cudaEventCreateWithFlags(&ev_ctr, cudaEventDisableTiming));
  } else {
    split_sms = 0;
  }
  FEKF_CHECK_CUDA(cudaDeviceSynchronize());
  npend = 0;
  return FEKF_OK;
}

fekf_status Kf::harvest(std::vector<EvPair>& pairs, size_t n) {
  // wall span of each pass: an unsplit pass's launch; a split pass from its early launch's start to the
  // later of the two launches' ends (the pairs of one pass are recorded consecutively: early, then late)
  long long pend = -1;
  float pend_ms = 0.f;
  for (size_t k = 0; k < n; ++k) {
    FEKF_CHECK_CUDA(cudaEventSynchronize(pairs[k].b));
    float ms = 0.f;
    FEKF_CHECK_CUDA(cudaEventElapsedTime(&ms, pairs[k].a, pairs[k].b));
    t_part[(int)pairs[k].part] += ms;
    if (pairs[k].part == 2) continue;
    t_ms += ms;
    if (!pairs[k].part) {
      t_n += 1;
      t_rw += pairs[k].rw;
      if (pend >= 0) t_span += pend_ms;
      pend = (long long)k;
      pend_ms = ms;
    } else if (pend >= 0) {
      float to_late = 0.f;
      FEKF_CHECK_CUDA(cudaEventElapsedTime(&to_late, pairs[pend].a, pairs[k].b));
      t_span += std::max(pend_ms, to_late);
      pend = -1;
    }
  }
  if (pend >= 0) t_span += pend_ms;
  return FEKF_OK;
}

fekf_status Kf::harvest_graph(GraphTiming* g) {
  if (!g->pending) return FEKF_OK;
  g->pending = false;
  pend_graphs.erase(std::remove(pend_graphs.begin(), pend_graphs.end(), g), pend_graphs.end());
  return harvest(g->ev, g->ev.size());
}

fekf_status Kf::timing_ctl(int mode, double* total_ms, int64_t* launches, int64_t* rw_launches) {
  if (mode == 1) {
    timing = true;
    ev_used = 0;
    for (GraphTiming* g : pend_graphs) g->pending = false;
    pend_graphs.clear();
    t_ms = 0.0;
    t_part[0] = t_part[1] = t_part[2] = 0.0;
    t_span = 0.0;
    t_n = t_rw = 0;
    return FEKF_OK;
  }
  FEKF_TRY(harvest(ev_pool, ev_used));
  ev_used = 0;
  while (!pend_graphs.empty()) FEKF_TRY(harvest_graph(pend_graphs.back()));
  timing = false;
  if (total_ms) *total_ms = t_ms;
  if (launches) *launches = t_n;
  if (rw_launches) *rw_launches = t_rw;
  return FEKF_OK;
}

Kf::~Kf() {
  if (side) { cudaStreamSynchronize(side); cudaStreamDestroy(side); }
  if (ev_early) cudaEventDestroy(ev_early);
  if (ev_ctr) cudaEventDestroy(ev_ctr);
  for (EvPair& e : ev_pool) { cudaEventDestroy(e.a); cudaEventDestroy(e.b); }
  for (DBuf* b : {&P, &items_d, &ws, &gpad, &ub, &ulist, &dotp, &csr_ptr, &csr_idx, &tc_blk, &tc_c, &off_d, &n_d,
                  &state, &counter, &counter2, &tcoff_d, &dblk, &cub, &nG, &nU, &nws, &ndot, &ncoef})
    dfree(*b);
}

// One launch of the P pass over items [i0, i0 + n) with its own work counter, bracketed by a timing
// event pair when timing or capturing.
fekf_status Kf::pass_launch(bool rw, int i0, int n, int* ctr, int grid, cudaStream_t s, int part, int i2, int n2,
                            int* ctr2, bool zero_ctr) {
  const KfPlan& p = plan;
  if (zero_ctr) FEKF_CHECK_CUDA(cudaMemsetAsync(ctr, 0, sizeof(int), s));
  EvPair* tp = nullptr;
  if (timing || capturing) {
    if (capturing) {
      rec->emplace_back();
      tp = &rec->back();
    } else {
      if (ev_pool.size() <= ev_used) ev_pool.emplace_back();
      tp = &ev_pool[ev_used++];
    }
    if (!tp->a) {
      FEKF_CHECK_CUDA(cudaEventCreate(&tp->a));
      FEKF_CHECK_CUDA(cudaEventCreate(&tp->b));
    }
    tp->rw = rw ? 1 : 0;
    tp->part = (char)part;
    FEKF_CHECK_CUDA(cudaEventRecordWithFlags(tp->a, s, capturing ? cudaEventRecordExternal : cudaEventRecordDefault));
  }
  const int K = rw ? npend : 0;
  const int stage_bytes = (int)(TILE_ELEMS * elem() + (2 * KT + K * VS) * sizeof(double));   // + g_J, u_k[J], g_I
  int nst = (int)std::min<size_t>(MAX_STAGES, (PASS_SMEM - PASS_HDR) / stage_bytes);
  if (ng == 2) nst &= ~1;   // two consumer groups alternate stages
  const ItemD* it = items_d.as<ItemD>() + i0;
  const ItemD* it2 = items_d.as<ItemD>() + i2;
  if (p32)
    kf_pass_kernel<float, 2><<<grid, PASS_THREADS, PASS_SMEM, s>>>(
        P.as<float>(), it, n, ctr, gpad.as<double>(), ulist.as<double>(), p.Npad, rw ? 1 : 0, K, nst, stage_bytes,
        state.as<KfState>(), ws.as<double>(), it2, n2, ctr2);
  else if (ng == 2)
    kf_pass_kernel<double, 2><<<grid, PASS_THREADS, PASS_SMEM, s>>>(
        P.as<double>(), it, n, ctr, gpad.as<double>(), ulist.as<double>(), p.Npad, rw ? 1 : 0, K, nst, stage_bytes,
        state.as<KfState>(), ws.as<double>(), it2, n2, ctr2);
  else
    kf_pass_kernel<double, 1><<<grid, PASS_THREADS, PASS_SMEM, s>>>(
        P.as<double>(), it, n, ctr, gpad.as<double>(), ulist.as<double>(), p.Npad, rw ? 1 : 0, K, nst, stage_bytes,
        state.as<KfState>(), ws.as<double>(), it2, n2, ctr2);
  FEKF_LAUNCH_CHECK();
  count_launch();
  if (tp) FEKF_CHECK_CUDA(cudaEventRecordWithFlags(tp->b, s, capturing ? cudaEventRecordExternal : cudaEventRecordDefault));
  return FEKF_OK;
}

fekf_status Kf::pass(const double* g, bool rw, cudaStream_t s, cudaEvent_t ready, double* ar_g) {
  FEKF_TRY(idle_check("kf_pass"));
  const KfPlan& p = plan;
  if (ar_g && !comm) ar_g = nullptr;
  const int tb = 256;
  const int n_items = (int)p.items.size();
  const bool split = ready && side && split_sms > 0 && p.n_early > 0;
  if (split) {
    // early blocks: pad + pass on the side stream as soon as their gradient is final
    const long long p0 = p.tc_off[p.late_blocks] * KT;
    FEKF_CHECK_CUDA(cudaStreamWaitEvent(side, ready, 0));
    // the early blocks' gradient segment and the error sum g[N] are final: their all-reduce goes first
    if (ar_g) FEKF_TRY(comm_allreduce(comm, ar_g + p.off[p.late_blocks], p.N + 1 - p.off[p.late_blocks], side));
    // diagnostic pair (timing only): early pass start on the side stream -> the producing stream is done
    // with the reverse pass (index, not pointer: the pair lists grow below)
    std::vector<EvPair>* dl = nullptr;
    size_t di = 0;
    if (timing || capturing) {
      dl = capturing ? rec : &ev_pool;
      if (capturing) {
        rec->emplace_back();
        di = rec->size() - 1;
      } else {
        if (ev_pool.size() <= ev_used) ev_pool.emplace_back();
        di = ev_used++;
      }
      EvPair& d = (*dl)[di];
      if (!d.a) {
        FEKF_CHECK_CUDA(cudaEventCreate(&d.a));
        FEKF_CHECK_CUDA(cudaEventCreate(&d.b));
      }
      d.part = 2;
      FEKF_CHECK_CUDA(cudaEventRecordWithFlags(d.a, side, capturing ? cudaEventRecordExternal : cudaEventRecordDefault));
    }
    kf_pad_kernel<<<cdiv(p.Npad - p0, tb), tb, 0, side>>>(g, gpad.as<double>(), tc_blk.as<int>(), tc_c.as<int>(),
                                                           off_d.as<long long>(), n_d.as<int>(), p0, p.Npad);
    FEKF_LAUNCH_CHECK();
    count_launch();
    FEKF_CHECK_CUDA(cudaMemsetAsync(counter2.p, 0, sizeof(int), side));
    FEKF_CHECK_CUDA(cudaEventRecord(ev_ctr, side));   // the late launch below shares counter2
    FEKF_TRY(pass_launch(rw, 0, p.n_early, counter2.as<int>(), std::min(p.n_early, split_sms), side, 0, 0, 0, nullptr,
                         false));
    FEKF_CHECK_CUDA(cudaEventRecord(ev_early, side));
    if (dl)
      FEKF_CHECK_CUDA(cudaEventRecordWithFlags((*dl)[di].b, s, capturing ? cudaEventRecordExternal : cudaEventRecordDefault));
    // late blocks on the producing stream
    if (ar_g && p.off[p.late_blocks] > 0) FEKF_TRY(comm_allreduce(comm, ar_g, p.off[p.late_blocks], s));
    if (p0 > 0) {
      kf_pad_kernel<<<cdiv(p0, tb), tb, 0, s>>>(g, gpad.as<double>(), tc_blk.as<int>(), tc_c.as<int>(),
                                                off_d.as<long long>(), n_d.as<int>(), 0, p0);
      FEKF_LAUNCH_CHECK();
      count_launch();
    }
    FEKF_CHECK_CUDA(cudaStreamWaitEvent(s, ev_ctr, 0));
    // the late launch takes the late items, then helps finish the early launch's unclaimed items on the
    // SMs the reverse pass has released (shared counter; every item's partials go to its fixed slots)
    FEKF_TRY(pass_launch(rw, p.n_early, n_items - p.n_early, counter.as<int>(), num_sms(), s, 1, 0, p.n_early,
                         counter2.as<int>()));
    FEKF_CHECK_CUDA(cudaStreamWaitEvent(s, ev_early, 0));
  } else {
    if (ar_g) FEKF_TRY(comm_allreduce(comm, ar_g, p.N + 1, s));
    kf_pad_kernel<<<cdiv(p.Npad, tb), tb, 0, s>>>(g, gpad.as<double>(), tc_blk.as<int>(), tc_c.as<int>(),
                                                   off_d.as<long long>(), n_d.as<int>(), 0, p.Npad);
    FEKF_LAUNCH_CHECK();
    count_launch();
    static const int cap = [] { const char* e = getenv("FEKF_PASS_SMS"); return e ? atoi(e) : 0; }();   // experiments
    if (n_items > 0)
      FEKF_TRY(pass_launch(rw, 0, n_items, counter.as<int>(), std::min(n_items, cap > 0 ? cap : num_sms()), s));
  }
  if (n_items > 0) {
    if (rw) ++rw_passes; else ++r_passes;
  }
  kf_reduce_u_kernel<<<cdiv(p.n_tc, 4), 256, 0, s>>>(ws.as<double>(), csr_ptr.as<long long>(),
                                                      csr_idx.as<long long>(), p.n_tc, ub.as<double>());
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// One update (Alg. 1 lines 8-13).  The stored P is rewritten only when `defer` corrections are
// pending; otherwise the pass is read-only and the corrections are applied to u in vector form.
fekf_status Kf::update(const double* g, const double* abe, double sqrt_bs, double* w, cudaStream_t s,
                       cudaEvent_t ready) {
  FEKF_TRY(update_begin(g, s, ready));
  if (comm && !replicated) FEKF_TRY(comm_allreduce(comm, ub.as<double>(), plan.Npad, s));
  return update_end(abe, sqrt_bs, w, s);
}

fekf_status Kf::update_begin(const double* g, cudaStream_t s, cudaEvent_t ready, double* ar_g) {
  if (in_update || naive_n > 0) { set_error("kf update_begin: previous update not ended"); return FEKF_ESTATE; }
  cur_rw = npend >= defer;
  FEKF_TRY(pass(g, cur_rw, s, ready, ar_g));
  in_update = true;
  return FEKF_OK;
}

fekf_status Kf::update_end(const double* abe, double sqrt_bs, double* w, cudaStream_t s) {
  if (!in_update) { set_error("kf update_end: no update begun"); return FEKF_ESTATE; }
  in_update = false;
  const KfPlan& p = plan;
  const bool rw = cur_rw;
  const int K = rw ? 0 : npend;
  kf_dot_kernel<<<cdiv(p.n_tc, 8), 256, 0, s>>>(gpad.as<double>(), ub.as<double>(), ulist.as<double>(), p.Npad, K,
                                                p.n_tc, dotp.as<double>());
  FEKF_LAUNCH_CHECK();
  kf_block_dot_kernel<<<cdiv((K + 1) * p.L, 128), 128, 0, s>>>(dotp.as<double>(), p.n_tc, K, p.L,
                                                                 tcoff_d.as<long long>(), dblk.as<double>());
  FEKF_LAUNCH_CHECK();
  kf_finish_kernel<<<1, 256, 0, s>>>(dblk.as<double>(), p.L, K, rw ? 1 : 0, state.as<KfState>(), cub.as<double>(), abe,
                                     sqrt_bs);
  FEKF_LAUNCH_CHECK();
  kf_vec_kernel<<<cdiv(p.Npad, 256), 256, 0, s>>>(ub.as<double>(), ulist.as<double>(), p.Npad, K, p.L, cub.as<double>(),
                                                   state.as<KfState>(), w, tc_blk.as<int>(), tc_c.as<int>(),
                                                   off_d.as<long long>(), n_d.as<int>());
  FEKF_LAUNCH_CHECK();
  count_launch(4);
  npend = (rw ? 0 : npend) + 1;
  return FEKF_OK;
}

fekf_status Kf::idle_check(const char* what) const {
  if (in_update || naive_n > 0) {
    set_error(std::string(what) + ": not allowed between an update's begin and end");
    return FEKF_ESTATE;
  }
  return FEKF_OK;
}

fekf_status Kf::flush(cudaStream_t s) {
  FEKF_TRY(idle_check("kf_flush"));
  if (!plan.items.empty() && npend > 0) {
    if (p32)
      kf_apply_pending_kernel<<<(unsigned)plan.items.size(), 256, 0, s>>>(P.as<float>(), items_d.as<ItemD>(),
                                                                           ulist.as<double>(), plan.Npad,
                                                                           state.as<KfState>());
    else
      kf_apply_pending_kernel<<<(unsigned)plan.items.size(), 256, 0, s>>>(P.as<double>(), items_d.as<ItemD>(),
                                                                           ulist.as<double>(), plan.Npad,
                                                                           state.as<KfState>());
    FEKF_LAUNCH_CHECK();
  }
  kf_clear_pending_kernel<<<1, 1, 0, s>>>(state.as<KfState>());
  FEKF_LAUNCH_CHECK();
  npend = 0;
  return FEKF_OK;
}

fekf_status Kf::get_block(int b, double* dst, cudaStream_t s) {
  if (b < 0 || b >= plan.L) { set_error("get_block: bad block"); return FEKF_EINVAL; }
  FEKF_TRY(idle_check("kf_get_block"));
  if (plan.items.empty()) return FEKF_OK;
  const unsigned nit = (unsigned)plan.items.size();
  if (p32)
    kf_get_block_kernel<<<nit, 256, 0, s>>>(P.as<float>(), items_d.as<ItemD>(), b, plan.n[b], ulist.as<double>(),
                                            plan.Npad, state.as<KfState>(), dst);
  else
    kf_get_block_kernel<<<nit, 256, 0, s>>>(P.as<double>(), items_d.as<ItemD>(), b, plan.n[b], ulist.as<double>(),
                                            plan.Npad, state.as<KfState>(), dst);
  FEKF_LAUNCH_CHECK();
  return FEKF_OK;
}

fekf_status Kf::set_block(int b, const double* src, cudaStream_t s) {
  if (b < 0 || b >= plan.L) { set_error("set_block: bad block"); return FEKF_EINVAL; }
  FEKF_TRY(flush(s));
  if (plan.items.empty()) return FEKF_OK;
  const unsigned nit = (unsigned)plan.items.size();
  if (p32) kf_set_block_kernel<<<nit, 256, 0, s>>>(P.as<float>(), items_d.as<ItemD>(), b, plan.n[b], src);
  else kf_set_block_kernel<<<nit, 256, 0, s>>>(P.as<double>(), items_d.as<ItemD>(), b, plan.n[b], src);
  FEKF_LAUNCH_CHECK();
  return FEKF_OK;
}

fekf_status Kf::get_state(double* lambda, double* A_last, int* flags) {
  KfState s;
  FEKF_CHECK_CUDA(cudaDeviceSynchronize());
  FEKF_CHECK_CUDA(cudaMemcpy(&s, state.p, sizeof(KfState), cudaMemcpyDeviceToHost));
  if (lambda) *lambda = s.lambda;
  if (A_last) *A_last = s.A_last;
  if (flags) *flags = s.flags;
  return FEKF_OK;
}

}  // namespace fekf
