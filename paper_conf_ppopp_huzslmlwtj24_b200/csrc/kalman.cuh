// Blocked Kalman filter state (see kalman.cu for the algorithm and its citations).
#pragma once
#include <vector>

#include "common.cuh"

namespace fekf {

constexpr int KT = FEKF_TILE;    // tile edge (64 fp64 = 32 KiB per tile)
constexpr int SEG_TILES = 32;    // max tiles per work item (tile-row segment)
constexpr int KMAX = 16;         // max deferred rank-1 corrections held before P is rewritten
constexpr int NAIVE_NMAX = 32;   // max samples of one Naive-EKF update (naive.cu)

// One P-pass work item: tiles (I, J0..J0+nJ-1) of block `blk`, stored contiguously at tile_off.
struct ItemD {
  int blk, I, J0, nJ;
  long long tile_off;   // in tiles, into this rank's P buffer
  long long vbase;      // offset of the block in the padded vectors
  long long col_slot0;  // workspace slot of the first tile's column partial
  int row_slot;         // workspace slot of the item's row partial
  int pad_;
};

// Device-resident optimizer scalars.  The stored P (the "base" B) and the current covariance are
// related by P_t = sigma (B - sum_k beta_k u_k u_k^T) over the npend deferred corrections.
struct KfState {
  double lambda, nu, sigma, c_mult;
  double A_last, coef_w;       // last A and sqrt(bs) * ABE * A
  double sig_cur;              // sigma used to form the current u
  double beta[KMAX];           // deferred coefficients
  long long t;
  int npend, flags, slot, skip;   // skip: the last update saw a non-finite A / ABE (no-op)
};

struct KfPlan {
  int L = 0, world = 1, rank = 0;
  std::vector<int> n, nt;
  std::vector<long long> off, tc_off;
  long long N = 0, n_tc = 0, Npad = 0;
  std::vector<int> tc_blk, tc_c;
  std::vector<ItemD> items;           // this rank's items (largest first)
  long long tiles_local = 0, total_tiles = 0, ws_slots = 0;
  std::vector<int> owner;             // owner rank of every canonical item
  std::vector<int> tile_owner;        // owner rank of every tile, canonical packed order
  std::vector<long long> csr_ptr, csr_idx;
  int rps = 1;                        // row-partial slots per item (consumer groups of the P pass)
  // blocks [0, late_blocks) are "late" (their gradient is the last one the reverse pass finishes): this
  // rank's items of the other ("early") blocks come first, n_early of them, so a pass can be split in two
  int late_blocks = 0, n_early = 0;
  void build(const std::vector<int>& blocks, int world, int rank, int seg_tiles, int row_slots = 1, int late = 0);
};

// communicator helpers (comm.cu)
int comm_world(fekf_comm* c);
int comm_rank(fekf_comm* c);
bool comm_is_loopback(fekf_comm* c);
fekf_status comm_allreduce(fekf_comm* c, double* buf, long long n, cudaStream_t s);

struct EvPair {
  cudaEvent_t a = nullptr, b = nullptr;
  char rw = 0;
  char part = 0;   // 1: second launch of a split pass (its time adds to the pass; not counted as a pass);
                   // 2: diagnostic pair (early pass start -> producer stream done with the reverse pass)
};

// Event pairs recorded inside one captured step graph; harvested before the graph is replayed again
// (by then its previous replay has finished) and when timing stops.
struct GraphTiming {
  std::vector<EvPair> ev;
  bool pending = false;
};

struct Kf {
  fekf_opt_cfg opt{};
  fekf_comm* comm = nullptr;
  KfPlan plan;
  int defer = 1;                 // corrections deferred before P is rewritten (1 = rewrite every update)
  int npend = 0;                 // host mirror of the device npend
  bool p32 = false;              // P stored fp32 (opt.precision == 32, reading Z22)
  bool replicated = false;       // opt.p_mode == 1: every rank holds all of P, no u exchange
  int ng = 1;                    // consumer groups of the P pass
  size_t elem() const { return p32 ? sizeof(float) : sizeof(double); }
  DBuf P, items_d, ws, gpad, ub, ulist, dotp, csr_ptr, csr_idx, tc_blk, tc_c, off_d, n_d, state, counter;
  DBuf tcoff_d, dblk, cub;       // block -> tile-column offsets, per-block dots, per-block coefficients
  // Live timing of the P pass: a [start, stop] event pair recorded on the launching stream around every
  // pass launch.  Eager launches draw pairs from `ev_pool`; while a step graph is being captured the pairs
  // go to that graph's own list (`rec`, external event-record nodes) and are harvested after each replay.
  bool timing = false;
  bool capturing = false;
  std::vector<EvPair> ev_pool;
  size_t ev_used = 0;
  std::vector<EvPair>* rec = nullptr;   // non-null while capturing with timing on
  double t_ms = 0.0;
  double t_part[3] = {0.0, 0.0, 0.0};   // split passes: early launch, late launch, early start -> tail done
  double t_span = 0.0;                  // summed wall span of the timed passes (split: early start -> last end)
  int64_t t_n = 0, t_rw = 0;
  long long rw_passes = 0, r_passes = 0;
  fekf_status timing_ctl(int mode, double* total_ms, int64_t* launches, int64_t* rw_launches);
  std::vector<GraphTiming*> pend_graphs;  // replayed graphs whose pairs are not harvested yet
  fekf_status harvest(std::vector<EvPair>& pairs, size_t n);   // add the elapsed times of n recorded pairs
  fekf_status harvest_graph(GraphTiming* g);
  // world/rank > 0 without a communicator: shard plan of that rank, exchange of u left to the caller
  fekf_status create(const std::vector<int>& blocks, const fekf_opt_cfg& o, fekf_comm* c, int world = 0, int rank = 0);
  ~Kf();
  // Split pass: with `ready` (an event recorded on the producing stream once the early blocks' gradient is
  // final) the early items stream on `split_sms` SMs from a side stream while the producer finishes the late
  // blocks' gradient; the late items follow on `s`.  With a communicator the gradient's all-reduce is split
  // the same way (pass(ar_g)), so the overlap survives at N > 1.
  int late_blocks = 0, split_sms = 0;
  cudaStream_t side = nullptr;
  cudaEvent_t ev_early = nullptr, ev_ctr = nullptr;
  DBuf counter2;
  // ar_g (with a communicator): g is not yet all-reduced over the ranks; the pass all-reduces it in place, in
  // two segments with the split (the early blocks' segment and the error sum at g[N] on the side stream as
  // soon as `ready` fires, the late blocks' segment on `s`), else in one piece on `s` (the early reduction,
  // P:L170)
  fekf_status pass(const double* g, bool rw, cudaStream_t s, cudaEvent_t ready = nullptr, double* ar_g = nullptr);
  fekf_status pass_launch(bool rw, int i0, int n, int* ctr, int grid, cudaStream_t s, int part = 0, int i2 = 0,
                          int n2 = 0, int* ctr2 = nullptr, bool zero_ctr = true);
  fekf_status update(const double* g, const double* abe, double sqrt_bs, double* w, cudaStream_t s,
                     cudaEvent_t ready = nullptr);
  // update = begin (P pass: this rank's partial u) + all-reduce of u over ranks + end (A, K, w, lambda)
  bool in_update = false, cur_rw = false;
  fekf_status update_begin(const double* g, cudaStream_t s, cudaEvent_t ready = nullptr, double* ar_g = nullptr);
  fekf_status update_end(const double* abe, double sqrt_bs, double* w, cudaStream_t s);
  fekf_status flush(cudaStream_t s);
  fekf_status idle_check(const char* what) const;   // FEKF_ESTATE between an update's begin and end
  fekf_status get_block(int b, double* dst, cudaStream_t s);
  fekf_status set_block(int b, const double* src, cudaStream_t s);
  fekf_status get_state(double* lambda, double* A_last, int* flags);
  // Naive-EKF (naive.cu): n per-sample gradients G [n][ldg], per-sample ABE [n]; rank-n update of P
  DBuf nG, nU, nws, ndot, ncoef;
  int naive_np = 0;
  int naive_n = 0;               // > 0 between update_naive_begin and update_naive_end
  fekf_status update_naive(const double* G, long long ldg, const double* abe, int n, double* w, double* A_out,
                           cudaStream_t s);
  fekf_status update_naive_begin(const double* G, long long ldg, int n, cudaStream_t s);
  fekf_status update_naive_end(const double* abe, double* w, double* A_out, cudaStream_t s);
  long long naive_u_len() const;
};

}  // namespace fekf

struct fekf_kf {
  fekf::Kf kf;
};
