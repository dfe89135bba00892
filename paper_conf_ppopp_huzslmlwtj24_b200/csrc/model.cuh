// DeePMD se_a model context: parameter layout, work buffers and the kernel launchers of the
// forward / backward / Jacobian passes.  See nets.cu for the math and citations.
#pragma once
#include <map>
#include <memory>
#include <vector>

#include "kalman.cuh"

namespace fekf {

struct Layer {
  int din, dout;
  long long W, b, dt;  // offsets into the flat parameter vector (dt = -1: none)
  int skip;            // 0 none, 1 identity (d_l == d_{l-1}), 2 concat [h, h] (d_l == 2 d_{l-1})
};

struct PairNet {       // embedding net of the type pair (ti, tj)
  int ti, tj;
  long long R;         // max rows = B * n_ti * sel_tj; the live count (valid slots only) is on the device
  std::vector<Layer> L;
  DBuf row_idx;        // [R]  global slot index (b*Na + i)*Nm + slot of every compacted row
  DBuf row_start;      // [B*n_ti + 1] first row of atom (b, k)
  DBuf tidx, tpos;     // [R]  tangent row -> primal row, primal row -> tangent row or -1
  DBuf hin, hin_t;     // [R]  s (primal rows), s-dot (active tangent rows)
  std::vector<DBuf> Y, H, Hb, Zb;       // primal   [R x d_l]
  std::vector<DBuf> Yt, Ht, Hbt, Zbt;   // tangent  [R x d_l] (only the first T rows are live)
  DBuf sbar;           // [R] adjoint of s (forces)
};

struct FitNet {        // fitting net of type t
  int t;
  long long F;         // rows = B * n_t
  std::vector<Layer> L;
  long long Wout, bout;
  DBuf D, Db;          // [2F x M*M2]
  std::vector<DBuf> Y, H, Hb, Zb;
  DBuf eout, ebar;     // [2F]
};

// One captured minibatch step (a10: "one CUDA graph").  The launch sequence of a step depends on the
// host state only through the number of pending Kalman corrections at entry (which passes rewrite P),
// so graphs are cached by that count and a step-parity bit (two graphs alternate, so the P-pass event
// pairs of a graph's previous replay can be read back for live timing without stalling the stream).
struct StepGraph {
  cudaGraphExec_t exec = nullptr;
  int npend_after = 0;
  int64_t launches = 0;
  GraphTiming tm;
};

struct Ctx {
  fekf_model_cfg m{};
  fekf_opt_cfg o{};
  int Na = 0, B = 0, Bg = 0, nt = 0, Nm = 0, M = 0, M2 = 0;
  int sec[FEKF_MAX_TYPES + 1]{};
  std::vector<int> types, tindex;                 // type of atom, index within its type
  std::vector<std::vector<int>> atoms_of;         // atoms of each type
  long long Np = 0;
  std::vector<int> blocks;
  std::vector<PairNet> pairs;                     // nt*nt, index ti*nt + tj
  std::vector<FitNet> fits;                       // nt
  fekf_comm* comm = nullptr;
  std::unique_ptr<::fekf_kf> kfo;                 // owns the Kalman filter
  Kf* kf = nullptr;
  // device
  DBuf types_d, tindex_d, atoms_d, atoms_off_d, sel_d, sec_d, err_d;
  DBuf env_stats;                                 // [2][nt][4]: avg | std of the R~ rows (reading Z11)
  DBuf w, gbuf;                                   // [Np], [Np + 1] (g || error sum, the allreduce payload)
  DBuf nl_j, nl_s, overflow, em, jac, rij, rdot, vdir;
  // fp32 nets (net_prec 32): fp32 copies of R~, its Jacobian, d and the weights (nets.cu prepare_geometry /
  // model_forward); every other nets buffer holds elements of the nets' type
  int net_prec = 64;
  DBuf em32, jac32, rij32, w32;
  // atomics-free force scatter (reverse neighbour map, built once per geometry): frow [slot][3] = dE/dd of
  // every valid slot, rev_off [B*Na + 1] / rev_idx [slots] = for every atom j the slots whose neighbour is
  // j, in slot order; rev_cnt [B][Na][Na] scratch of the deterministic fill
  DBuf frow, rev_cnt, rev_off, rev_idx;
  const int* sel_atoms = nullptr;                 // MODE_FORCE_SEL: the force group's atoms (mark_selected)
  int n_sel_atoms = 0;
  DBuf X, Xb;                                     // [2 * B*Na*4*M] (primal | tangent)
  DBuf eatom, etot, force, virial, vatom;
  DBuf splitk_ws, colsum_ws;
  DBuf rowcnt;                                    // [2 * npairs] live primal / tangent rows per pair
  DBuf chunks;                                    // [npairs * max_chunks] tangent-row scan workspace
  int max_chunks = 1;
  DBuf abe, metrics_tmp, abs_sum;
  DBuf naive_G, naive_es, naive_abe;              // Naive-EKF step: [B][Np] per-image g, [B] error sums, [B] ABE
  size_t splitk_elems = 0, colsum_elems = 0;
  int64_t last_launches = 0;
  // step graphs: inputs are staged into ctx-owned buffers so the captured pointers stay fixed
  bool use_graph = true;
  bool graphs_ready = false;   // every (pending-correction count, parity) variant captured
  bool trows_ready = false;                       // tangent-active rows already built for this force update
  std::map<int, StepGraph> graphs;
  cudaStream_t gstream = nullptr;
  // Split P pass (kalman.cu Kf::pass): model_backward records ev_fit once the fitting nets' weight
  // gradients are final (split_armed, set by the step around a gradient pass that feeds an update) and
  // caps the embedding backward at emb_sms SMs while the early P pass streams on the others.
  cudaEvent_t ev_fit = nullptr;
  bool split_armed = false;
  int emb_sms = 0;
  // per-pair concurrency of the embedding launches on the step's critical path (primal / tangent forward,
  // the force-only reverse): one stream per type pair, each launch's persistent grid capped at its share of
  // the SMs (emb_grid_cap, 0 = no cap) so the pairs run side by side instead of back to back
  std::vector<cudaStream_t> pstreams;
  std::vector<cudaEvent_t> pev;      // [0] fork, [1 + p] join of pair p
  int emb_grid_cap = 0;
  cudaEvent_t gev_in = nullptr, gev_out = nullptr;
  DBuf st_coord, st_box, st_e, st_f, st_fidx, st_met;
  int64_t nsteps = 0;
  void drop_graphs();

  fekf_status init(const fekf_model_cfg& m, const fekf_opt_cfg& o, int natoms, const int32_t* types_host, int B,
                   int Bg, fekf_comm* comm);
  ~Ctx();
};

// geom.cu
fekf_status launch_nlist(Ctx& c, const double* coord, const double* box, int nb, int* nl_j, int* nl_s, int* overflow,
                         cudaStream_t s);
fekf_status launch_envmat(Ctx& c, const double* coord, const double* box, const int* nl_j, const int* nl_s, int nb,
                          double* em, double* jac, double* rij, cudaStream_t s);

// nets.cu (compiled twice, real.cuh: n64 = fp64 nets, n32 = fp32 nets)
// MODE_FORCE_SEL: forces on the selected atoms only (a force update needs F_pred on S_k):
// the embedding reverse runs over the rows that touch S_k (the tangent-active rows, built beforehand by
// mark_selected) instead of every row; forces of other atoms are left partial.
enum Mode { MODE_ENERGY_GRAD = 0, MODE_FORCE = 1, MODE_FORCE_JAC = 2, MODE_FORCE_SEL = 3 };
#define FEKF_NETS_API                                                                                       \
  fekf_status prepare_geometry(Ctx& c, int nb, cudaStream_t s);                                             \
  fekf_status model_forward(Ctx& c, int nb, bool tangent, cudaStream_t s);                                  \
  fekf_status mark_selected(Ctx& c, int nb, const int* atom_idx, int n_sel, cudaStream_t s);                \
  fekf_status model_backward(Ctx& c, int nb, Mode mode, double* g, cudaStream_t s);                         \
  fekf_status energy_outputs(Ctx& c, int nb, cudaStream_t s);                                               \
  fekf_status energy_error(Ctx& c, int nb, const double* e_label, double* abs_sum, cudaStream_t s);         \
  fekf_status force_error(Ctx& c, int nb, const double* f_label, const int* atom_idx, int n_sel,            \
                          double* abs_sum, cudaStream_t s);                                                 \
  fekf_status tangent_env(Ctx& c, int nb, cudaStream_t s);                                                  \
  fekf_status build_rows(Ctx& c, int nb, cudaStream_t s);                                                   \
  fekf_status build_reverse(Ctx& c, int nb, cudaStream_t s);                                                \
  fekf_status seed_force(Ctx& c, int nb, cudaStream_t s);
namespace n64 { FEKF_NETS_API }
namespace n32 { FEKF_NETS_API }
#undef FEKF_NETS_API
// the nets' precision of a context (fekf_opt_cfg::net_precision; 0 follows `precision`)
inline bool nets32(const Ctx& c) { return c.net_prec == 32; }
#define FEKF_NETS_CALL(f) return nets32(c) ? n32::f : n64::f
inline fekf_status prepare_geometry(Ctx& c, int nb, cudaStream_t s) { FEKF_NETS_CALL(prepare_geometry(c, nb, s)); }
inline fekf_status model_forward(Ctx& c, int nb, bool t, cudaStream_t s) { FEKF_NETS_CALL(model_forward(c, nb, t, s)); }
inline fekf_status mark_selected(Ctx& c, int nb, const int* a, int n, cudaStream_t s) {
  FEKF_NETS_CALL(mark_selected(c, nb, a, n, s));
}
inline fekf_status model_backward(Ctx& c, int nb, Mode m, double* g, cudaStream_t s) {
  FEKF_NETS_CALL(model_backward(c, nb, m, g, s));
}
inline fekf_status energy_outputs(Ctx& c, int nb, cudaStream_t s) { FEKF_NETS_CALL(energy_outputs(c, nb, s)); }
inline fekf_status energy_error(Ctx& c, int nb, const double* e, double* a, cudaStream_t s) {
  FEKF_NETS_CALL(energy_error(c, nb, e, a, s));
}
inline fekf_status force_error(Ctx& c, int nb, const double* f, const int* idx, int n, double* a, cudaStream_t s) {
  FEKF_NETS_CALL(force_error(c, nb, f, idx, n, a, s));
}
inline fekf_status tangent_env(Ctx& c, int nb, cudaStream_t s) { FEKF_NETS_CALL(tangent_env(c, nb, s)); }
inline fekf_status build_rows(Ctx& c, int nb, cudaStream_t s) { FEKF_NETS_CALL(build_rows(c, nb, s)); }
inline fekf_status build_reverse(Ctx& c, int nb, cudaStream_t s) { FEKF_NETS_CALL(build_reverse(c, nb, s)); }
inline fekf_status seed_force(Ctx& c, int nb, cudaStream_t s) { FEKF_NETS_CALL(seed_force(c, nb, s)); }
#undef FEKF_NETS_CALL

}  // namespace fekf

struct fekf_ctx {
  fekf::Ctx c;
};
