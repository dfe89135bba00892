// C ABI of libfekf.so (include/fekf.h): context setup, parameter layout, step orchestration.
//
// The training step follows the paper's update schedule: per minibatch one energy update
// and `force_groups` force updates, each: forward with the current weights -> sign flip + error
// (Alg. 1 lines 3-6) -> summed gradient (line 7) -> early reduction over ranks ->
// blocked Kalman update (lines 8-13).
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <string>

#include "model.cuh"

namespace fekf {

static thread_local std::string g_err;
thread_local int64_t g_launches = 0;

void set_error(const std::string& msg) { g_err = msg; }

fekf_status dalloc(DBuf& b, size_t bytes) {
  if (bytes == 0) bytes = 16;
  cudaError_t e = cudaMalloc(&b.p, bytes);
  if (e != cudaSuccess) {
    b.p = nullptr;
    set_error(std::string("cudaMalloc(") + std::to_string(bytes) + "): " + cudaGetErrorString(e));
    return e == cudaErrorMemoryAllocation ? FEKF_ENOMEM : FEKF_ECUDA;
  }
  b.bytes = bytes;
  return FEKF_OK;
}
void dfree(DBuf& b) {
  if (b.p) cudaFree(b.p);
  b.p = nullptr;
  b.bytes = 0;
}

// ---------------------------------------------------------------------------------------------
// layout (must agree with the oracle's param_tensors — checked by the tests)
// ---------------------------------------------------------------------------------------------
struct TensorSpec {
  int kind;  // 0 emb, 1 fit
  long long size;
};

static fekf_status check_model(const fekf_model_cfg& m) {
  if (m.ntypes < 1 || m.ntypes > FEKF_MAX_TYPES) { set_error("ntypes out of range"); return FEKF_EINVAL; }
  if (m.n_emb < 1 || m.n_emb > FEKF_MAX_LAYERS || m.n_fit < 1 || m.n_fit > FEKF_MAX_LAYERS) {
    set_error("layer count out of range");
    return FEKF_EINVAL;
  }
  for (int l = 0; l < m.n_emb; ++l)
    if (m.emb[l] < 1 || m.emb[l] > 1024) { set_error("embedding width out of range"); return FEKF_EINVAL; }
  for (int l = 0; l < m.n_fit; ++l)
    if (m.fit[l] < 1 || m.fit[l] > 4096) { set_error("fitting width out of range"); return FEKF_EINVAL; }
  if (m.m2 < 1 || m.m2 > m.emb[m.n_emb - 1]) { set_error("m2 must be in [1, M]"); return FEKF_EINVAL; }
  int nm = 0;
  for (int t = 0; t < m.ntypes; ++t) {
    if (m.sel[t] < 0 || m.sel[t] > 4096) { set_error("sel out of range"); return FEKF_EINVAL; }
    nm += m.sel[t];
  }
  if (nm < 1) { set_error("sum(sel) must be positive"); return FEKF_EINVAL; }
  if (!(m.rcut > 0) || !(m.rcut_smth >= 0) || !(m.rcut_smth < m.rcut)) { set_error("need 0 <= rcut_smth < rcut"); return FEKF_EINVAL; }
  if (m.switch_kind != 0 && m.switch_kind != 1) { set_error("switch_kind must be 0 (quintic) or 1 (cosine)"); return FEKF_EINVAL; }
  if (m.type_one_side != 0 && m.type_one_side != 1) { set_error("type_one_side must be 0 or 1"); return FEKF_EINVAL; }
  return FEKF_OK;
}

static int skip_rule(int din, int dout) { return dout == din ? 1 : (dout == 2 * din ? 2 : 0); }

// Builds layer descriptors with parameter offsets; returns total count and per-tensor sizes.
static long long build_layout(const fekf_model_cfg& m, std::vector<long long>* sizes,
                              std::vector<std::vector<Layer>>* emb, std::vector<std::vector<Layer>>* fit,
                              std::vector<long long>* wout, std::vector<long long>* bout) {
  long long off = 0;
  auto push = [&](long long n) {
    long long o = off;
    off += n;
    if (sizes) sizes->push_back(n);
    return o;
  };
  for (int ti = 0; ti < m.ntypes; ++ti)
    for (int tj = 0; tj < m.ntypes; ++tj) {
      if (m.type_one_side && ti > 0) {   // one net per neighbour type t_j (reading Z15 flag): shared
        if (emb) emb->push_back((*emb)[tj]);
        continue;
      }
      std::vector<Layer> Ls;
      int din = 1;
      for (int l = 0; l < m.n_emb; ++l) {
        Layer L;
        L.din = din;
        L.dout = m.emb[l];
        L.W = push((long long)din * m.emb[l]);
        L.b = push(m.emb[l]);
        L.dt = -1;
        L.skip = l == 0 ? 0 : skip_rule(din, m.emb[l]);
        Ls.push_back(L);
        din = m.emb[l];
      }
      if (emb) emb->push_back(Ls);
    }
  const int M = m.emb[m.n_emb - 1];
  for (int ti = 0; ti < m.ntypes; ++ti) {
    std::vector<Layer> Ls;
    int din = M * m.m2;
    for (int l = 0; l < m.n_fit; ++l) {
      Layer L;
      L.din = din;
      L.dout = m.fit[l];
      L.W = push((long long)din * m.fit[l]);
      L.b = push(m.fit[l]);
      const bool res = l > 0 && m.fit[l] == din;
      L.dt = (res && m.fit_resnet_dt) ? push(m.fit[l]) : -1;
      L.skip = res ? 1 : 0;
      Ls.push_back(L);
      din = m.fit[l];
    }
    if (fit) fit->push_back(Ls);
    long long wo = push(din);
    long long bo = push(1);
    if (wout) wout->push_back(wo);
    if (bout) bout->push_back(bo);
  }
  return off;
}

// RLEKF gather/split
static std::vector<int> block_split(const std::vector<long long>& sizes, long long nb) {
  std::vector<int> out;
  long long cur = 0;
  for (long long n : sizes) {
    if (cur + n > nb) {
      if (cur > 0) out.push_back((int)cur);
      if (n >= nb) {
        long long q = n / nb, r = n % nb;
        for (long long k = 0; k < q; ++k) out.push_back((int)nb);
        if (r) out.push_back((int)r);
        cur = 0;
      } else {
        cur = n;
      }
    } else {
      cur += n;
    }
  }
  if (cur > 0) out.push_back((int)cur);
  return out;
}

// ---------------------------------------------------------------------------------------------
// context
// ---------------------------------------------------------------------------------------------
fekf_status Ctx::init(const fekf_model_cfg& mm, const fekf_opt_cfg& oo, int natoms, const int32_t* types_host, int Bl,
                      int Bglob, fekf_comm* cm) {
  FEKF_TRY(check_model(mm));
  if (natoms < 1 || !types_host || Bl < 1 || Bglob < Bl) { set_error("create: bad natoms/types/batch"); return FEKF_EINVAL; }
  if (oo.block_size < 1 || oo.force_groups < 0 || oo.atoms_per_group < 1 || !(oo.nu > 0 && oo.nu <= 1)) {
    set_error("create: bad optimizer config");
    return FEKF_EINVAL;
  }
  m = mm;
  o = oo;
  if (o.net_precision != 0 && o.net_precision != 32 && o.net_precision != 64) {
    set_error("create: net_precision must be 0 (follow precision), 32 or 64");
    return FEKF_EINVAL;
  }
  net_prec = o.net_precision ? o.net_precision : (o.precision == 32 ? 32 : 64);
  Na = natoms;
  B = Bl;
  Bg = Bglob;
  nt = m.ntypes;
  M = m.emb[m.n_emb - 1];
  M2 = m.m2;
  comm = cm;
  sec[0] = 0;
  for (int t = 0; t < nt; ++t) sec[t + 1] = sec[t] + m.sel[t];
  Nm = sec[nt];
  types.assign(types_host, types_host + natoms);
  atoms_of.assign(nt, {});
  tindex.assign(natoms, 0);
  for (int i = 0; i < natoms; ++i) {
    if (types[i] < 0 || types[i] >= nt) { set_error("atom type out of range"); return FEKF_EINVAL; }
    tindex[i] = (int)atoms_of[types[i]].size();
    atoms_of[types[i]].push_back(i);
  }
  std::vector<long long> sizes, wout, bout;
  std::vector<std::vector<Layer>> emb, fit;
  Np = build_layout(m, &sizes, &emb, &fit, &wout, &bout);
  blocks = block_split(sizes, o.block_size);

  // device tables
  std::vector<int> atoms_cat, atoms_off(nt + 1, 0);
  for (int t = 0; t < nt; ++t) {
    atoms_off[t + 1] = atoms_off[t] + (int)atoms_of[t].size();
    atoms_cat.insert(atoms_cat.end(), atoms_of[t].begin(), atoms_of[t].end());
  }
  FEKF_TRY(dalloc(types_d, sizeof(int) * Na));
  FEKF_TRY(dalloc(tindex_d, sizeof(int) * Na));
  FEKF_TRY(dalloc(atoms_d, sizeof(int) * Na));
  FEKF_TRY(dalloc(atoms_off_d, sizeof(int) * (nt + 1)));
  FEKF_TRY(dalloc(sel_d, sizeof(int) * FEKF_MAX_TYPES));
  FEKF_TRY(dalloc(sec_d, sizeof(int) * (FEKF_MAX_TYPES + 1)));
  FEKF_TRY(dalloc(err_d, sizeof(int) * 4));
  FEKF_TRY(dalloc(env_stats, sizeof(double) * 2 * nt * 4));
  {
    std::vector<double> st(2 * nt * 4, 0.0);
    for (int q = nt * 4; q < 2 * nt * 4; ++q) st[q] = 1.0;   // avg 0, std 1: no normalisation
    FEKF_CHECK_CUDA(cudaMemcpy(env_stats.p, st.data(), sizeof(double) * st.size(), cudaMemcpyHostToDevice));
  }
  FEKF_CHECK_CUDA(cudaMemcpy(types_d.p, types.data(), sizeof(int) * Na, cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(tindex_d.p, tindex.data(), sizeof(int) * Na, cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(atoms_d.p, atoms_cat.data(), sizeof(int) * Na, cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(atoms_off_d.p, atoms_off.data(), sizeof(int) * (nt + 1), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(sel_d.p, m.sel, sizeof(int) * FEKF_MAX_TYPES, cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemcpy(sec_d.p, sec, sizeof(int) * (FEKF_MAX_TYPES + 1), cudaMemcpyHostToDevice));
  FEKF_CHECK_CUDA(cudaMemset(err_d.p, 0, sizeof(int) * 4));

  const long long nslots = (long long)B * Na * Nm;
  FEKF_TRY(dalloc(w, sizeof(double) * Np));
  FEKF_TRY(dalloc(gbuf, sizeof(double) * (Np + 1)));
  FEKF_TRY(dalloc(nl_j, sizeof(int) * nslots));
  FEKF_TRY(dalloc(nl_s, sizeof(int) * nslots));
  FEKF_TRY(dalloc(overflow, sizeof(int) * B));
  FEKF_TRY(dalloc(em, sizeof(double) * nslots * 4));
  FEKF_TRY(dalloc(jac, sizeof(double) * nslots * 12));
  FEKF_TRY(dalloc(rij, sizeof(double) * nslots * 3));
  FEKF_TRY(dalloc(rdot, sizeof(double) * nslots * 4));
  if (net_prec == 32) {   // the fp32 nets' copies of the fp64 geometry and weights (nets.cu)
    FEKF_TRY(dalloc(em32, sizeof(float) * nslots * 4));
    FEKF_TRY(dalloc(jac32, sizeof(float) * nslots * 12));
    FEKF_TRY(dalloc(rij32, sizeof(float) * nslots * 3));
    FEKF_TRY(dalloc(w32, sizeof(float) * Np));
  }
  FEKF_TRY(dalloc(vdir, sizeof(double) * B * Na * 3));
  FEKF_TRY(dalloc(frow, sizeof(double) * nslots * 3));
  FEKF_TRY(dalloc(rev_cnt, sizeof(int) * (size_t)B * Na * Na));
  FEKF_TRY(dalloc(rev_off, sizeof(int) * ((size_t)B * Na + 1)));
  FEKF_TRY(dalloc(rev_idx, sizeof(int) * nslots));
  FEKF_CHECK_CUDA(cudaMemset(frow.p, 0, sizeof(double) * nslots * 3));
  FEKF_TRY(dalloc(X, sizeof(double) * 2 * B * Na * 4 * M));
  FEKF_TRY(dalloc(Xb, sizeof(double) * 2 * B * Na * 4 * M));
  FEKF_TRY(dalloc(eatom, sizeof(double) * B * Na));
  FEKF_TRY(dalloc(etot, sizeof(double) * B));
  FEKF_TRY(dalloc(force, sizeof(double) * B * Na * 3));
  FEKF_TRY(dalloc(virial, sizeof(double) * B * 9));
  FEKF_TRY(dalloc(vatom, sizeof(double) * B * Na * 9));
  FEKF_TRY(dalloc(abe, sizeof(double) * 2));
  FEKF_TRY(dalloc(abs_sum, sizeof(double) * 2));
  FEKF_TRY(dalloc(metrics_tmp, sizeof(double) * 64));
  FEKF_CHECK_CUDA(cudaMemset(rdot.p, 0, sizeof(double) * nslots * 4));
  FEKF_CHECK_CUDA(cudaMemset(X.p, 0, sizeof(double) * 2 * B * Na * 4 * M));
  splitk_elems = (size_t)16 << 20;
  FEKF_TRY(dalloc(splitk_ws, sizeof(double) * splitk_elems));
  int maxh = 1;
  for (int l = 0; l < m.n_fit; ++l) maxh = std::max(maxh, m.fit[l]);
  colsum_elems = (size_t)(2 * 148 + 2) * maxh;   // act_bwd_dt: at most 2 x 148 row chunks
  FEKF_TRY(dalloc(colsum_ws, sizeof(double) * colsum_elems * nt));   // one region per atom type

  pairs.clear();
  for (int ti = 0; ti < nt; ++ti)
    for (int tj = 0; tj < nt; ++tj) {
      PairNet P;
      P.ti = ti;
      P.tj = tj;
      P.R = (long long)B * atoms_of[ti].size() * m.sel[tj];
      P.L = emb[ti * nt + tj];
      pairs.push_back(std::move(P));
    }
  FEKF_TRY(dalloc(rowcnt, sizeof(int) * 2 * pairs.size()));
  for (auto& P : pairs) max_chunks = std::max(max_chunks, cdiv(std::max<long long>(P.R, 1), 1024));
  FEKF_TRY(dalloc(chunks, sizeof(int) * pairs.size() * max_chunks));
  FEKF_CHECK_CUDA(cudaMemset(rowcnt.p, 0, sizeof(int) * 2 * pairs.size()));
  for (auto& P : pairs) {
    const long long R1 = std::max<long long>(P.R, 1);
    FEKF_TRY(dalloc(P.row_idx, sizeof(int) * R1));
    FEKF_TRY(dalloc(P.row_start, sizeof(int) * (B * atoms_of[P.ti].size() + 1)));
    FEKF_TRY(dalloc(P.tidx, sizeof(int) * R1));
    FEKF_TRY(dalloc(P.tpos, sizeof(int) * R1));
    FEKF_TRY(dalloc(P.hin, sizeof(double) * R1));
    FEKF_TRY(dalloc(P.hin_t, sizeof(double) * R1));
    FEKF_TRY(dalloc(P.sbar, sizeof(double) * R1));
    const size_t nl = P.L.size();
    for (auto* v : {&P.Y, &P.H, &P.Hb, &P.Zb, &P.Yt, &P.Ht, &P.Hbt, &P.Zbt}) v->resize(nl);
    for (size_t l = 0; l < nl; ++l) {
      const size_t n = sizeof(double) * R1 * P.L[l].dout;
      for (auto* v : {&P.Y, &P.H, &P.Hb, &P.Zb, &P.Yt, &P.Ht, &P.Hbt, &P.Zbt}) FEKF_TRY(dalloc((*v)[l], n));
    }
  }
  fits.clear();
  for (int t = 0; t < nt; ++t) {
    FitNet F;
    F.t = t;
    F.F = (long long)B * atoms_of[t].size();
    F.L = fit[t];
    F.Wout = wout[t];
    F.bout = bout[t];
    fits.push_back(std::move(F));
  }
  for (auto& F : fits) {
    const long long F2 = 2 * std::max<long long>(F.F, 1);
    FEKF_TRY(dalloc(F.D, sizeof(double) * F2 * M * M2));
    FEKF_TRY(dalloc(F.Db, sizeof(double) * F2 * M * M2));
    FEKF_TRY(dalloc(F.eout, sizeof(double) * F2));
    FEKF_TRY(dalloc(F.ebar, sizeof(double) * F2));
    F.Y.resize(F.L.size()); F.H.resize(F.L.size()); F.Hb.resize(F.L.size()); F.Zb.resize(F.L.size());
    for (size_t l = 0; l < F.L.size(); ++l) {
      const size_t n = sizeof(double) * F2 * F.L[l].dout;
      FEKF_TRY(dalloc(F.Y[l], n)); FEKF_TRY(dalloc(F.H[l], n)); FEKF_TRY(dalloc(F.Hb[l], n)); FEKF_TRY(dalloc(F.Zb[l], n));
    }
  }
  kfo.reset(new fekf_kf());
  kf = &kfo->kf;
  {
    // blocks holding any embedding parameter (they come first in the layout) get their gradient last
    long long acc = 0;
    int late = 0;
    const long long emb_end = fits.empty() ? Np : fits[0].L[0].W;
    while (late < (int)blocks.size() && acc < emb_end) acc += blocks[late++];
    kf->late_blocks = late;
    const char* e = getenv("FEKF_SPLIT_SMS");
    kf->split_sms = e ? atoi(e) : (o.precision == 32 ? 80 : 96);   // measured defaults
  }
  FEKF_TRY(kf->create(blocks, o, comm));
  if (kf->split_sms > 0 && !getenv("FEKF_SPLIT_SMS") && kf->plan.total_tiles > 0) {
    // P sharded over the ranks (p_mode 0, world > 1): this rank streams a fraction f of P while its reverse
    // pass does the work of N = 1 (weak scaling: B images per rank), so the early pass needs fewer SMs.  With
    // S1 of the Ns SMs balancing the pass against the reverse pass at f = 1 (the measured defaults above),
    // pass time ~ f / S and reverse time ~ 1 / (Ns - S) balance at S(f) = Ns f / (f + (Ns - S1) / S1):
    // 96 -> 71 / 46 / 28 early SMs at 2 / 4 / 8 ranks (fp64).  Not measured on real multi-GPU runs.
    const double f = (double)kf->plan.tiles_local / (double)kf->plan.total_tiles;
    if (f < 0.999) {
      int cdev = 0, nsm = 148;
      FEKF_CHECK_CUDA(cudaGetDevice(&cdev));
      FEKF_CHECK_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, cdev));
      const double S1 = std::min<double>(kf->split_sms, nsm - 1), r = (nsm - S1) / S1;
      kf->split_sms = std::max(8, (int)std::lround(nsm * f / (f + r)));
    }
  }
  if (kf->split_sms > 0) FEKF_CHECK_CUDA(cudaEventCreateWithFlags(&ev_fit, cudaEventDisableTiming));
  int dev = 0;
  FEKF_CHECK_CUDA(cudaGetDevice(&dev));
  int maxsm = 0;
  FEKF_CHECK_CUDA(cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  const size_t need = (16 * (size_t)M + 2 * (size_t)M * (M2 + 1) + 8 * (size_t)Nm) * sizeof(double);
  if (need > (size_t)maxsm) { set_error("M*M2 too large for the descriptor kernels' shared memory"); return FEKF_EINVAL; }
  // step-graph staging buffers and the capture stream
  FEKF_TRY(dalloc(st_coord, sizeof(double) * B * Na * 3));
  FEKF_TRY(dalloc(st_box, sizeof(double) * B * 9));
  FEKF_TRY(dalloc(st_e, sizeof(double) * B));
  FEKF_TRY(dalloc(st_f, sizeof(double) * B * Na * 3));
  FEKF_TRY(dalloc(st_fidx, sizeof(int) * std::max(1, o.force_groups * o.atoms_per_group)));
  FEKF_TRY(dalloc(st_met, sizeof(double) * 8));
  FEKF_CHECK_CUDA(cudaStreamCreateWithFlags(&gstream, cudaStreamNonBlocking));
  {
    const char* v = getenv("FEKF_PAIR_STREAMS");   // measured default: on
    if (pairs.size() > 1 && !(v && atoi(v) == 0)) {
      pstreams.resize(pairs.size());
      pev.resize(pairs.size() + 1);
      for (auto& st : pstreams) FEKF_CHECK_CUDA(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
      for (auto& ev : pev) FEKF_CHECK_CUDA(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    }
  }
  FEKF_CHECK_CUDA(cudaEventCreateWithFlags(&gev_in, cudaEventDisableTiming));
  FEKF_CHECK_CUDA(cudaEventCreateWithFlags(&gev_out, cudaEventDisableTiming));
  FEKF_CHECK_CUDA(cudaDeviceSynchronize());
  return FEKF_OK;
}

void Ctx::drop_graphs() {
  for (auto& kv : graphs) {
    if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
    if (kf) {
      kf->pend_graphs.erase(std::remove(kf->pend_graphs.begin(), kf->pend_graphs.end(), &kv.second.tm),
                            kf->pend_graphs.end());
    }
    for (EvPair& e : kv.second.tm.ev) { cudaEventDestroy(e.a); cudaEventDestroy(e.b); }
  }
  graphs.clear();
  graphs_ready = false;
}

Ctx::~Ctx() {
  if (gstream) cudaStreamSynchronize(gstream);
  drop_graphs();
  if (gstream) cudaStreamDestroy(gstream);
  if (gev_in) cudaEventDestroy(gev_in);
  if (gev_out) cudaEventDestroy(gev_out);
  if (ev_fit) cudaEventDestroy(ev_fit);
  for (auto& st : pstreams) { cudaStreamSynchronize(st); cudaStreamDestroy(st); }
  for (auto& ev : pev) cudaEventDestroy(ev);
  for (DBuf* b : {&st_coord, &st_box, &st_e, &st_f, &st_fidx, &st_met, &naive_G, &naive_es, &naive_abe}) dfree(*b);
  kfo.reset();
  kf = nullptr;
  for (DBuf* b : {&types_d, &tindex_d, &atoms_d, &atoms_off_d, &sel_d, &sec_d, &err_d, &env_stats, &w, &gbuf, &nl_j, &nl_s,
                  &overflow, &em, &jac, &rij, &rdot, &em32, &jac32, &rij32, &w32, &vdir, &frow, &rev_cnt, &rev_off, &rev_idx, &X, &Xb, &eatom, &etot, &force, &virial, &vatom, &splitk_ws,
                  &colsum_ws, &abe, &metrics_tmp, &abs_sum, &rowcnt, &chunks})
    dfree(*b);
  for (auto& P : pairs) {
    for (DBuf* b : {&P.row_idx, &P.row_start, &P.tidx, &P.tpos, &P.hin, &P.hin_t, &P.sbar}) dfree(*b);
    for (auto* v : {&P.Y, &P.H, &P.Hb, &P.Zb, &P.Yt, &P.Ht, &P.Hbt, &P.Zbt}) for (auto& b : *v) dfree(b);
  }
  for (auto& F : fits) {
    dfree(F.D); dfree(F.Db); dfree(F.eout); dfree(F.ebar);
    for (auto* v : {&F.Y, &F.H, &F.Hb, &F.Zb}) for (auto& b : *v) dfree(b);
  }
}

// ABE from the reduced error sum: abe = sum * scale (Alg. 1 line 6; normalisations reading Z4)
__global__ void abe_kernel(const double* sum, double scale, double* abe, double* metric) {
  const double v = *sum * scale;
  *abe = v;
  if (metric) *metric = v;
}
__global__ void metrics_kernel(const KfState* st, const int* err, const int* overflow, int nb, double* metrics) {
  int ov = 0;
  for (int b = 0; b < nb; ++b) ov += overflow[b];
  int flags = st->flags | (err[0] ? 4 : 0) | (ov > 0 ? 1 : 0);
  metrics[5] = st->A_last;
  metrics[6] = st->lambda;
  metrics[7] = (double)flags;
}

static fekf_status geometry(Ctx& c, const double* coord, const double* box, int nb, cudaStream_t s) {
  FEKF_TRY(launch_nlist(c, coord, box, nb, c.nl_j.as<int>(), c.nl_s.as<int>(), c.overflow.as<int>(), s));
  FEKF_TRY(launch_envmat(c, coord, box, c.nl_j.as<int>(), c.nl_s.as<int>(), nb, c.em.as<double>(), c.jac.as<double>(),
                         c.rij.as<double>(), s));
  FEKF_TRY(prepare_geometry(c, nb, s));   // fp32 nets: fp32 copies of R~, J, d
  FEKF_TRY(build_rows(c, nb, s));
  FEKF_TRY(build_reverse(c, nb, s));
  return FEKF_OK;
}

static fekf_status energy_grad_pass(Ctx& c, int nb, const double* e_label, double* g, double* abs_sum, cudaStream_t s) {
  FEKF_TRY(model_forward(c, nb, false, s));
  FEKF_TRY(energy_outputs(c, nb, s));
  FEKF_TRY(energy_error(c, nb, e_label, abs_sum, s));
  FEKF_CHECK_CUDA(cudaMemsetAsync(g, 0, sizeof(double) * c.Np, s));
  FEKF_TRY(model_backward(c, nb, MODE_ENERGY_GRAD, g, s));
  return FEKF_OK;
}

static fekf_status force_grad_pass(Ctx& c, int nb, const double* f_label, const int* atom_idx, int n_sel, double* g,
                                   double* abs_sum, cudaStream_t s) {
  FEKF_TRY(model_forward(c, nb, false, s));
  FEKF_TRY(seed_force(c, nb, s));
  FEKF_TRY(mark_selected(c, nb, atom_idx, n_sel, s));   // rows touching S_k (tangent-active rows)
  FEKF_TRY(model_backward(c, nb, MODE_FORCE_SEL, nullptr, s));
  FEKF_TRY(force_error(c, nb, f_label, atom_idx, n_sel, abs_sum, s));
  FEKF_TRY(tangent_env(c, nb, s));
  FEKF_TRY(model_forward(c, nb, true, s));
  FEKF_CHECK_CUDA(cudaMemsetAsync(g, 0, sizeof(double) * c.Np, s));
  FEKF_TRY(model_backward(c, nb, MODE_FORCE_JAC, g, s));
  return FEKF_OK;
}

// One minibatch: geometry, 1 energy update, force_groups force updates, metrics.
static fekf_status step_body(Ctx& c, const double* coord, const double* box, const double* e_label,
                             const double* f_label, const int32_t* force_idx, double* metrics, cudaStream_t s) {
  const int nb = c.B;
  const double sqrt_bs = std::sqrt((double)c.Bg);
  double* g = c.gbuf.as<double>();
  double* esum = g + c.Np;
  FEKF_CHECK_CUDA(cudaMemsetAsync(metrics, 0, sizeof(double) * 8, s));
  FEKF_TRY(geometry(c, coord, box, nb, s));
  // Every update's P pass starts on the fitting blocks as soon as their gradient is final and overlaps
  // the tail of the reverse pass (split pass, Kf::pass); with a communicator the early reduction of
  // [g || error sum] is split the same way (Kf::pass ar_g), so the overlap holds at N > 1 too.
  const bool split = c.ev_fit != nullptr;
  // measured: round 1 kept the energy update unsplit (its reverse-pass tail was too short
  // to cover the slower 96-SM pass); with round 2's nets 1 wins (593 / 591 vs 586 / 585 images/s)
  static const int split_e = [] { const char* e = getenv("FEKF_SPLIT_E"); return e ? atoi(e) : 1; }();
  auto kalman = [&](double scale, double* metric) -> fekf_status {
    if (c.split_armed && c.comm) {
      FEKF_TRY(c.kf->update_begin(g, s, c.ev_fit, g));
      abe_kernel<<<1, 1, 0, s>>>(esum, scale, c.abe.as<double>(), metric);
      FEKF_LAUNCH_CHECK();
      count_launch();
      if (!c.kf->replicated) FEKF_TRY(comm_allreduce(c.comm, c.kf->ub.as<double>(), c.kf->plan.Npad, s));
      return c.kf->update_end(c.abe.as<double>(), sqrt_bs, c.w.as<double>(), s);
    }
    FEKF_TRY(comm_allreduce(c.comm, g, c.Np + 1, s));
    abe_kernel<<<1, 1, 0, s>>>(esum, scale, c.abe.as<double>(), metric);
    FEKF_LAUNCH_CHECK();
    count_launch();
    return c.kf->update(g, c.abe.as<double>(), sqrt_bs, c.w.as<double>(), s, c.split_armed ? c.ev_fit : nullptr);
  };
  // energy update (1 per minibatch)
  c.split_armed = split && split_e;
  FEKF_TRY(energy_grad_pass(c, nb, e_label, g, esum, s));
  FEKF_TRY(kalman(1.0 / c.Bg, metrics + 0));
  c.split_armed = split;
  // force updates
  const int apg = c.o.atoms_per_group;
  for (int k = 0; k < c.o.force_groups; ++k) {
    FEKF_TRY(force_grad_pass(c, nb, f_label, force_idx + (size_t)k * apg, apg, g, esum, s));
    FEKF_TRY(kalman(1.0 / ((double)c.Bg * apg * 3) / c.Na, k < 4 ? metrics + 1 + k : nullptr));
  }
  c.split_armed = false;
  metrics_kernel<<<1, 1, 0, s>>>(c.kf->state.as<KfState>(), c.err_d.as<int>(), c.overflow.as<int>(), nb, metrics);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// Naive-EKF minibatch: per-image gradients and errors into the rank-n update (naive.cu).
__global__ void naive_abe_kernel(const double* esum, int n, double scale, double* abe, double* metric) {
  double m = 0.0;
  for (int b = 0; b < n; ++b) {
    abe[b] = esum[b] * scale;
    m += abe[b];
  }
  if (metric) *metric = m / n;
}

static fekf_status naive_step_body(Ctx& c, const double* coord, const double* box, const double* e_label,
                                   const double* f_label, const int32_t* force_idx, double* metrics, cudaStream_t s) {
  const int nb = c.B;
  const size_t na3 = (size_t)c.Na * 3;
  if (!c.naive_G.p) {
    FEKF_TRY(dalloc(c.naive_G, sizeof(double) * (size_t)nb * c.Np));
    FEKF_TRY(dalloc(c.naive_es, sizeof(double) * nb));
    FEKF_TRY(dalloc(c.naive_abe, sizeof(double) * nb));
  }
  double* G = c.naive_G.as<double>();
  double* es = c.naive_es.as<double>();
  double* ab = c.naive_abe.as<double>();
  FEKF_CHECK_CUDA(cudaMemsetAsync(metrics, 0, sizeof(double) * 8, s));
  // energy update: g_b, |e_b| / N_a of image b alone
  for (int b = 0; b < nb; ++b) {
    FEKF_TRY(geometry(c, coord + b * na3, box + (size_t)b * 9, 1, s));
    FEKF_TRY(energy_grad_pass(c, 1, e_label + b, G + (size_t)b * c.Np, es + b, s));
  }
  naive_abe_kernel<<<1, 1, 0, s>>>(es, nb, 1.0, ab, metrics + 0);
  FEKF_LAUNCH_CHECK();
  count_launch();
  FEKF_TRY(c.kf->update_naive(G, c.Np, ab, nb, c.w.as<double>(), nullptr, s));
  // force updates
  const int apg = c.o.atoms_per_group;
  for (int k = 0; k < c.o.force_groups; ++k) {
    for (int b = 0; b < nb; ++b) {
      FEKF_TRY(geometry(c, coord + b * na3, box + (size_t)b * 9, 1, s));
      FEKF_TRY(force_grad_pass(c, 1, f_label + b * na3, force_idx + (size_t)k * apg, apg, G + (size_t)b * c.Np,
                               es + b, s));
    }
    naive_abe_kernel<<<1, 1, 0, s>>>(es, nb, 1.0 / ((double)apg * 3) / c.Na, ab, k < 4 ? metrics + 1 + k : nullptr);
    FEKF_LAUNCH_CHECK();
    count_launch();
    FEKF_TRY(c.kf->update_naive(G, c.Np, ab, nb, c.w.as<double>(), nullptr, s));
  }
  // neighbour-list overflow of every image (the per-image passes above reuse slot 0)
  FEKF_TRY(launch_nlist(c, coord, box, nb, c.nl_j.as<int>(), c.nl_s.as<int>(), c.overflow.as<int>(), s));
  metrics_kernel<<<1, 1, 0, s>>>(c.kf->state.as<KfState>(), c.err_d.as<int>(), c.overflow.as<int>(), nb, metrics);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

// Capture the step for the current host state (pending-correction count) unless cached.
static fekf_status step_graph(Ctx& c, StepGraph** out) {
  Kf& k = *c.kf;
  // every graph records a P-pass event pair (a negligible node) whether or not timing is on, so timing
  // never forces a re-capture; two graphs per count alternate by step parity
  const int key = k.npend * 2 + (int)(c.nsteps & 1);
  StepGraph& G = c.graphs[key];
  if (!G.exec) {
    const int npend0 = k.npend;
    const int64_t l0 = g_launches;
    const long long rwp = k.rw_passes, rp = k.r_passes;
    k.capturing = true;
    k.rec = &G.tm.ev;
    FEKF_CHECK_CUDA(cudaStreamBeginCapture(c.gstream, cudaStreamCaptureModeRelaxed));
    fekf_status st = step_body(c, c.st_coord.as<double>(), c.st_box.as<double>(), c.st_e.as<double>(),
                               c.st_f.as<double>(), c.st_fidx.as<int32_t>(), c.st_met.as<double>(), c.gstream);
    cudaGraph_t graph = nullptr;
    cudaError_t e = cudaStreamEndCapture(c.gstream, &graph);
    k.capturing = false;
    k.rec = nullptr;
    G.npend_after = k.npend;
    G.launches = g_launches - l0;
    k.npend = npend0;
    k.rw_passes = rwp;
    k.r_passes = rp;
    g_launches = l0;
    if (st != FEKF_OK || e != cudaSuccess) {
      if (graph) cudaGraphDestroy(graph);
      c.graphs.erase(key);
      if (st != FEKF_OK) return st;
      FEKF_CHECK_CUDA(e);
    }
    // FEKF_GRAPH_PRIO=1 honours the captured per-node priorities (the split pass's side stream is the
    // highest-priority stream): the early pass then starts while the last data-gradient GEMM still runs, which
    // stretches that GEMM over the remaining SMs; measured 594.8 vs 597.0 images/s, off
    static const unsigned long long gflags = [] {
      const char* v = getenv("FEKF_GRAPH_PRIO");
      return (v && atoi(v) == 1) ? (unsigned long long)cudaGraphInstantiateFlagUseNodePriority : 0ULL;
    }();
    e = cudaGraphInstantiateWithFlags(&G.exec, graph, gflags);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) {
      c.graphs.erase(key);
      FEKF_CHECK_CUDA(e);
    }
    // upload now (setup), not at the graph's first launch inside the step loop
    FEKF_CHECK_CUDA(cudaGraphUpload(G.exec, c.gstream));
  }
  *out = &G;
  return FEKF_OK;
}

}  // namespace fekf

using namespace fekf;

// =================================================================================================
extern "C" {

const char* fekf_last_error(void) { return g_err.c_str(); }
int fekf_version(void) { return 2; }

fekf_status fekf_plan_layout(const fekf_model_cfg* m, int block_size, int64_t* n_params, int32_t* blocks_host, int cap,
                             int* nblocks) {
  if (!m || block_size < 1) { set_error("plan_layout: bad args"); return FEKF_EINVAL; }
  FEKF_TRY(check_model(*m));
  std::vector<long long> sizes;
  long long n = build_layout(*m, &sizes, nullptr, nullptr, nullptr, nullptr);
  std::vector<int> bl = block_split(sizes, block_size);
  if (n_params) *n_params = n;
  if (nblocks) *nblocks = (int)bl.size();
  if (blocks_host) {
    if (cap < (int)bl.size()) { set_error("plan_layout: cap too small"); return FEKF_EINVAL; }
    std::copy(bl.begin(), bl.end(), blocks_host);
  }
  return FEKF_OK;
}

fekf_status fekf_opt_defaults(int global_batch, fekf_opt_cfg* o) {
  if (!o || global_batch < 1) { set_error("opt_defaults: bad args"); return FEKF_EINVAL; }
  *o = fekf_opt_cfg{};
  const bool large = global_batch > 1024;
  o->lambda0 = large ? 0.90 : 0.98;
  o->nu = large ? 0.996 : 0.9987;
  o->block_size = 10240;
  o->noise_mode = 0;
  o->grad_reduce = 0;
  o->force_groups = 4;
  o->atoms_per_group = 6;
  o->p_defer = 15;
  o->precision = 64;
  o->net_precision = 0;
  return FEKF_OK;
}

fekf_status fekf_plan_shard(const int32_t* blocks_host, int nblocks, int world, int rank, int64_t* tiles_local,
                            int64_t* bytes_local, int32_t* tile_owner_host) {
  if (!blocks_host || nblocks < 1 || world < 1 || rank < 0 || rank >= world) { set_error("plan_shard: bad args"); return FEKF_EINVAL; }
  KfPlan p;
  p.build(std::vector<int>(blocks_host, blocks_host + nblocks), world, rank, SEG_TILES);
  if (tiles_local) *tiles_local = p.tiles_local;
  if (bytes_local) *bytes_local = p.tiles_local * (int64_t)KT * KT * (int64_t)sizeof(double);
  if (tile_owner_host) std::copy(p.tile_owner.begin(), p.tile_owner.end(), tile_owner_host);
  return FEKF_OK;
}

// ---- Kalman filter ----
fekf_status fekf_kf_create(const int32_t* block_sizes_host, int nblocks, const fekf_opt_cfg* opt, fekf_comm* comm,
                           fekf_kf** out) {
  if (!block_sizes_host || nblocks < 1 || !opt || !out) { set_error("kf_create: bad args"); return FEKF_EINVAL; }
  for (int i = 0; i < nblocks; ++i)
    if (block_sizes_host[i] < 1) { set_error("kf_create: block size < 1"); return FEKF_EINVAL; }
  fekf_kf* k = new fekf_kf();
  fekf_status st = k->kf.create(std::vector<int>(block_sizes_host, block_sizes_host + nblocks), *opt, comm);
  if (st != FEKF_OK) { delete k; return st; }
  *out = k;
  return FEKF_OK;
}
fekf_status fekf_kf_create_shard(const int32_t* block_sizes_host, int nblocks, const fekf_opt_cfg* opt, int world,
                                 int rank, fekf_kf** out) {
  if (!block_sizes_host || nblocks < 1 || !opt || !out || world < 1 || rank < 0 || rank >= world) {
    set_error("kf_create_shard: bad args");
    return FEKF_EINVAL;
  }
  for (int i = 0; i < nblocks; ++i)
    if (block_sizes_host[i] < 1) { set_error("kf_create_shard: block size < 1"); return FEKF_EINVAL; }
  fekf_kf* k = new fekf_kf();
  fekf_status st = k->kf.create(std::vector<int>(block_sizes_host, block_sizes_host + nblocks), *opt, nullptr, world, rank);
  if (st != FEKF_OK) { delete k; return st; }
  *out = k;
  return FEKF_OK;
}
fekf_status fekf_kf_update_begin(fekf_kf* k, const double* g, cudaStream_t s) {
  if (!k || !g) { set_error("kf_update_begin: null"); return FEKF_EINVAL; }
  return k->kf.update_begin(g, s);
}
fekf_status fekf_kf_partial_u(fekf_kf* k, double** u, int64_t* n) {
  if (!k || !u || !n) { set_error("kf_partial_u: null"); return FEKF_EINVAL; }
  *u = k->kf.ub.as<double>();
  *n = k->kf.plan.Npad;
  return FEKF_OK;
}
fekf_status fekf_kf_update_end(fekf_kf* k, const double* abe, double sqrt_bs, double* w, cudaStream_t s) {
  if (!k || !abe || !w) { set_error("kf_update_end: null"); return FEKF_EINVAL; }
  return k->kf.update_end(abe, sqrt_bs, w, s);
}
fekf_status fekf_kf_destroy(fekf_kf* k) { delete k; return FEKF_OK; }
fekf_status fekf_kf_update(fekf_kf* k, const double* g, const double* abe, double sqrt_bs, double* w, cudaStream_t s) {
  if (!k || !g || !abe || !w) { set_error("kf_update: null"); return FEKF_EINVAL; }
  return k->kf.update(g, abe, sqrt_bs, w, s);
}
fekf_status fekf_kf_flush(fekf_kf* k, cudaStream_t s) { if (!k) return FEKF_EINVAL; return k->kf.flush(s); }
fekf_status fekf_kf_get_block(fekf_kf* k, int b, double* dst, cudaStream_t s) {
  if (!k || !dst) { set_error("kf_get_block: null"); return FEKF_EINVAL; }
  return k->kf.get_block(b, dst, s);
}
fekf_status fekf_kf_set_block(fekf_kf* k, int b, const double* src, cudaStream_t s) {
  if (!k || !src) { set_error("kf_set_block: null"); return FEKF_EINVAL; }
  return k->kf.set_block(b, src, s);
}
fekf_status fekf_kf_get_state(fekf_kf* k, double* lambda, double* A_last, int* flags) {
  if (!k) return FEKF_EINVAL;
  return k->kf.get_state(lambda, A_last, flags);
}
fekf_status fekf_kf_info(const fekf_kf* k, int64_t* pb, int64_t* tl, int64_t* npad, int64_t* items) {
  if (!k) return FEKF_EINVAL;
  const KfPlan& p = k->kf.plan;
  if (pb) *pb = p.tiles_local * (int64_t)KT * KT * (int64_t)k->kf.elem();
  if (tl) *tl = p.tiles_local;
  if (npad) *npad = p.Npad;
  if (items) *items = (int64_t)p.items.size();
  return FEKF_OK;
}
fekf_status fekf_kf_pass(fekf_kf* k, const double* g, cudaStream_t s) {
  if (!k || !g) { set_error("kf_pass: null"); return FEKF_EINVAL; }
  return k->kf.pass(g, false, s);
}
fekf_status fekf_kf_timing_parts(const fekf_kf* k, double* ms3) {
  if (!k || !ms3) { set_error("kf_timing_parts: null"); return FEKF_EINVAL; }
  for (int i = 0; i < 3; ++i) ms3[i] = k->kf.t_part[i];
  return FEKF_OK;
}
fekf_status fekf_kf_timing_span(const fekf_kf* k, double* span_ms) {
  if (!k || !span_ms) { set_error("kf_timing_span: null"); return FEKF_EINVAL; }
  *span_ms = k->kf.t_span;
  return FEKF_OK;
}
fekf_status fekf_kf_timing(fekf_kf* k, int mode, double* total_ms, int64_t* launches, int64_t* rw_launches) {
  if (!k || (mode != 0 && mode != 1)) { set_error("kf_timing: bad args"); return FEKF_EINVAL; }
  return k->kf.timing_ctl(mode, total_ms, launches, rw_launches);
}

// ---- context ----
fekf_status fekf_create(const fekf_model_cfg* m, const fekf_opt_cfg* opt, int natoms, const int32_t* types_host,
                        int local_batch, int global_batch, fekf_comm* comm, fekf_ctx** out) {
  if (!m || !opt || !out) { set_error("create: null"); return FEKF_EINVAL; }
  fekf_ctx* c = new fekf_ctx();
  fekf_status st = c->c.init(*m, *opt, natoms, types_host, local_batch, global_batch, comm);
  if (st != FEKF_OK) { delete c; return st; }
  *out = c;
  return FEKF_OK;
}
fekf_status fekf_destroy(fekf_ctx* c) { delete c; return FEKF_OK; }
fekf_status fekf_param_count(const fekf_ctx* c, int64_t* n) {
  if (!c || !n) return FEKF_EINVAL;
  *n = c->c.Np;
  return FEKF_OK;
}
fekf_status fekf_get_kf(fekf_ctx* c, fekf_kf** kf) {
  if (!c || !kf) return FEKF_EINVAL;
  *kf = c->c.kfo.get();
  return FEKF_OK;
}
fekf_status fekf_set_params(fekf_ctx* c, const double* w, cudaStream_t s) {
  if (!c || !w) { set_error("set_params: null"); return FEKF_EINVAL; }
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c->c.w.p, w, sizeof(double) * c->c.Np, cudaMemcpyDeviceToDevice, s));
  return FEKF_OK;
}
fekf_status fekf_get_params(const fekf_ctx* c, double* w, cudaStream_t s) {
  if (!c || !w) { set_error("get_params: null"); return FEKF_EINVAL; }
  FEKF_CHECK_CUDA(cudaMemcpyAsync(w, c->c.w.p, sizeof(double) * c->c.Np, cudaMemcpyDeviceToDevice, s));
  return FEKF_OK;
}

fekf_status fekf_set_env_stats(fekf_ctx* ctx, const double* avg, const double* sd) {
  if (!ctx) { set_error("set_env_stats: null"); return FEKF_EINVAL; }
  Ctx& c = ctx->c;
  std::vector<double> st(2 * c.nt * 4);
  for (int q = 0; q < c.nt * 4; ++q) {
    st[q] = avg ? avg[q] : 0.0;
    st[c.nt * 4 + q] = sd ? sd[q] : 1.0;
    if (!std::isfinite(st[q]) || !std::isfinite(st[c.nt * 4 + q]) || !(st[c.nt * 4 + q] > 0)) {
      set_error("set_env_stats: avg must be finite, std finite and > 0");
      return FEKF_EINVAL;
    }
  }
  if (c.gstream) FEKF_CHECK_CUDA(cudaStreamSynchronize(c.gstream));   // replays in flight read the table
  FEKF_CHECK_CUDA(cudaDeviceSynchronize());
  FEKF_CHECK_CUDA(cudaMemcpy(c.env_stats.p, st.data(), sizeof(double) * st.size(), cudaMemcpyHostToDevice));
  return FEKF_OK;
}

static fekf_status check_nb(const Ctx& c, int nb) {
  if (nb < 1 || nb > c.B) { set_error("nb must be in [1, local_batch]"); return FEKF_EINVAL; }
  return FEKF_OK;
}

fekf_status fekf_build_nlist(fekf_ctx* ctx, const double* coord, const double* box, int nb, int32_t* nlist_j,
                             int32_t* nlist_shift, int32_t* overflow, cudaStream_t s) {
  if (!ctx || !coord || !box || !nlist_j || !nlist_shift || !overflow) { set_error("build_nlist: null"); return FEKF_EINVAL; }
  FEKF_TRY(check_nb(ctx->c, nb));
  return launch_nlist(ctx->c, coord, box, nb, nlist_j, nlist_shift, overflow, s);
}

fekf_status fekf_env_mat(fekf_ctx* ctx, const double* coord, const double* box, const int32_t* nlist_j,
                         const int32_t* nlist_shift, int nb, double* em, double* em_deriv, double* rij, cudaStream_t s) {
  if (!ctx || !coord || !box || !nlist_j || !nlist_shift || !em || !em_deriv || !rij) { set_error("env_mat: null"); return FEKF_EINVAL; }
  FEKF_TRY(check_nb(ctx->c, nb));
  return launch_envmat(ctx->c, coord, box, nlist_j, nlist_shift, nb, em, em_deriv, rij, s);
}

fekf_status fekf_forward(fekf_ctx* ctx, const double* coord, const double* box, int nb, double* e_atom, double* e,
                         double* force, double* virial, cudaStream_t s) {
  if (!ctx || !coord || !box || !e_atom || !e) { set_error("forward: null"); return FEKF_EINVAL; }
  Ctx& c = ctx->c;
  FEKF_TRY(check_nb(c, nb));
  FEKF_TRY(geometry(c, coord, box, nb, s));
  FEKF_TRY(model_forward(c, nb, false, s));
  FEKF_TRY(energy_outputs(c, nb, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(e_atom, c.eatom.p, sizeof(double) * nb * c.Na, cudaMemcpyDeviceToDevice, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(e, c.etot.p, sizeof(double) * nb, cudaMemcpyDeviceToDevice, s));
  if (force || virial) {
    FEKF_TRY(seed_force(c, nb, s));
    FEKF_TRY(model_backward(c, nb, MODE_FORCE, nullptr, s));
    if (force) FEKF_CHECK_CUDA(cudaMemcpyAsync(force, c.force.p, sizeof(double) * nb * c.Na * 3, cudaMemcpyDeviceToDevice, s));
    if (virial) FEKF_CHECK_CUDA(cudaMemcpyAsync(virial, c.virial.p, sizeof(double) * nb * 9, cudaMemcpyDeviceToDevice, s));
  }
  return FEKF_OK;
}

fekf_status fekf_energy_jacobian(fekf_ctx* ctx, const double* coord, const double* box, const double* e_label, int nb,
                                 double* g_local, double* abs_err_sum, cudaStream_t s) {
  if (!ctx || !coord || !box || !e_label || !g_local || !abs_err_sum) { set_error("energy_jacobian: null"); return FEKF_EINVAL; }
  Ctx& c = ctx->c;
  FEKF_TRY(check_nb(c, nb));
  FEKF_TRY(geometry(c, coord, box, nb, s));
  return energy_grad_pass(c, nb, e_label, g_local, abs_err_sum, s);
}

fekf_status fekf_force_jacobian(fekf_ctx* ctx, const double* coord, const double* box, const double* f_label,
                                const int32_t* atom_idx, int n_sel, int nb, double* g_local, double* abs_err_sum,
                                cudaStream_t s) {
  if (!ctx || !coord || !box || !f_label || !atom_idx || !g_local || !abs_err_sum || n_sel < 1) {
    set_error("force_jacobian: bad args");
    return FEKF_EINVAL;
  }
  Ctx& c = ctx->c;
  FEKF_TRY(check_nb(c, nb));
  FEKF_TRY(geometry(c, coord, box, nb, s));
  return force_grad_pass(c, nb, f_label, atom_idx, n_sel, g_local, abs_err_sum, s);
}

fekf_status fekf_kalman_update(fekf_ctx* ctx, const double* g_global, const double* abs_sum, int kind, int n_sel,
                               cudaStream_t s) {
  if (!ctx || !g_global || !abs_sum || (kind != 0 && kind != 1) || (kind == 1 && n_sel < 1)) {
    set_error("kalman_update: bad args");
    return FEKF_EINVAL;
  }
  Ctx& c = ctx->c;
  const double scale = kind == 0 ? 1.0 / c.Bg : 1.0 / ((double)c.Bg * n_sel * 3) / c.Na;
  abe_kernel<<<1, 1, 0, s>>>(abs_sum, scale, c.abe.as<double>(), nullptr);
  FEKF_LAUNCH_CHECK();
  return c.kf->update(g_global, c.abe.as<double>(), std::sqrt((double)c.Bg), c.w.as<double>(), s);
}

fekf_status fekf_train_step(fekf_ctx* ctx, const double* coord, const double* box, const double* e_label,
                            const double* f_label, const int32_t* force_idx, double* metrics, cudaStream_t s) {
  if (!ctx || !coord || !box || !e_label || !f_label || !metrics || (!force_idx && ctx->c.o.force_groups > 0)) {
    set_error("train_step: null");
    return FEKF_EINVAL;
  }
  Ctx& c = ctx->c;
  if (!c.use_graph || comm_is_loopback(c.comm)) {   // loopback collectives are host barriers: eager only
    const int64_t l0 = g_launches;
    FEKF_TRY(step_body(c, coord, box, e_label, f_label, force_idx, metrics, s));
    c.last_launches = g_launches - l0;
    ++c.nsteps;
    return FEKF_OK;
  }
  // stage the step's inputs into the captured buffers (stream order on s), then replay on gstream
  const size_t na3 = sizeof(double) * (size_t)c.B * c.Na * 3;
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_coord.p, coord, na3, cudaMemcpyDeviceToDevice, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_box.p, box, sizeof(double) * c.B * 9, cudaMemcpyDeviceToDevice, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_e.p, e_label, sizeof(double) * c.B, cudaMemcpyDeviceToDevice, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_f.p, f_label, na3, cudaMemcpyDeviceToDevice, s));
  if (c.o.force_groups > 0)
    FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_fidx.p, force_idx, sizeof(int32_t) * c.o.force_groups * c.o.atoms_per_group,
                                    cudaMemcpyDeviceToDevice, s));
  StepGraph* G = nullptr;
  if (!c.graphs_ready) {
    // Capture every variant the step can take (pending-correction count at entry 0..p_defer, step parity)
    // once, here, instead of the first time each count comes round: a capture + instantiate of the ~540
    // nodes costs a few ms, and the count cycles through all p_defer + 1 values only every 16 steps.
    Kf& k = *c.kf;
    const int np0 = k.npend;
    const int64_t ns0 = c.nsteps;
    for (int np = 0; np <= k.defer; ++np)
      for (int par = 0; par < 2; ++par) {
        k.npend = np;
        c.nsteps = par;
        fekf_status st = step_graph(c, &G);
        if (st != FEKF_OK) {
          k.npend = np0;
          c.nsteps = ns0;
          return st;
        }
      }
    k.npend = np0;
    c.nsteps = ns0;
    c.graphs_ready = true;
  }
  FEKF_TRY(step_graph(c, &G));
  if (G->tm.pending) FEKF_TRY(c.kf->harvest_graph(&G->tm));
  FEKF_CHECK_CUDA(cudaEventRecord(c.gev_in, s));
  FEKF_CHECK_CUDA(cudaStreamWaitEvent(c.gstream, c.gev_in, 0));
  FEKF_CHECK_CUDA(cudaGraphLaunch(G->exec, c.gstream));
  FEKF_CHECK_CUDA(cudaEventRecord(c.gev_out, c.gstream));
  FEKF_CHECK_CUDA(cudaStreamWaitEvent(s, c.gev_out, 0));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(metrics, c.st_met.p, sizeof(double) * 8, cudaMemcpyDeviceToDevice, s));
  if (c.kf->timing && !G->tm.ev.empty()) {
    G->tm.pending = true;
    c.kf->pend_graphs.push_back(&G->tm);
  }
  c.kf->npend = G->npend_after;
  g_launches += G->launches;
  c.last_launches = G->launches;
  ++c.nsteps;
  return FEKF_OK;
}

// One captured graph of the Naive-EKF minibatch per pending-FEKF-correction count at entry (after the
// first naive update the count is 0, so one graph serves every later step).
static fekf_status naive_graph(Ctx& c, StepGraph** out) {
  Kf& k = *c.kf;
  const int key = (1 << 20) | k.npend;
  StepGraph& G = c.graphs[key];
  if (!G.exec) {
    const int npend0 = k.npend;
    const int64_t l0 = g_launches;
    FEKF_CHECK_CUDA(cudaStreamBeginCapture(c.gstream, cudaStreamCaptureModeRelaxed));
    fekf_status st = naive_step_body(c, c.st_coord.as<double>(), c.st_box.as<double>(), c.st_e.as<double>(),
                                     c.st_f.as<double>(), c.st_fidx.as<int32_t>(), c.st_met.as<double>(), c.gstream);
    cudaGraph_t graph = nullptr;
    cudaError_t e = cudaStreamEndCapture(c.gstream, &graph);
    G.npend_after = k.npend;
    G.launches = g_launches - l0;
    k.npend = npend0;
    g_launches = l0;
    if (st != FEKF_OK || e != cudaSuccess) {
      if (graph) cudaGraphDestroy(graph);
      c.graphs.erase(key);
      if (st != FEKF_OK) return st;
      FEKF_CHECK_CUDA(e);
    }
    e = cudaGraphInstantiate(&G.exec, graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) {
      c.graphs.erase(key);
      FEKF_CHECK_CUDA(e);
    }
    FEKF_CHECK_CUDA(cudaGraphUpload(G.exec, c.gstream));
  }
  *out = &G;
  return FEKF_OK;
}

fekf_status fekf_naive_train_step(fekf_ctx* ctx, const double* coord, const double* box, const double* e_label,
                                  const double* f_label, const int32_t* force_idx, double* metrics, cudaStream_t s) {
  if (!ctx || !coord || !box || !e_label || !f_label || !metrics || (!force_idx && ctx->c.o.force_groups > 0)) {
    set_error("naive_train_step: null");
    return FEKF_EINVAL;
  }
  Ctx& c = ctx->c;
  if (c.B != c.Bg || c.B > NAIVE_NMAX || c.comm) {
    set_error("naive_train_step: single rank with local_batch <= 32 only");
    return FEKF_EINVAL;
  }
  // eager on the first call (it allocates the per-image gradient and Naive-EKF workspaces), then one
  // captured graph per step like fekf_train_step
  const int np_needed = c.B <= 8 ? 8 : (c.B <= 16 ? 16 : 32);   // naive.cu's vector-set width for B samples
  if (!c.use_graph || !c.gstream || !c.naive_G.p || c.kf->naive_np < np_needed) {
    if (c.gstream) FEKF_CHECK_CUDA(cudaStreamSynchronize(c.gstream));   // earlier graph replays
    const int64_t l0 = g_launches;
    FEKF_TRY(naive_step_body(c, coord, box, e_label, f_label, force_idx, metrics, s));
    c.last_launches = g_launches - l0;
    ++c.nsteps;
    return FEKF_OK;
  }
  const size_t na3 = sizeof(double) * (size_t)c.B * c.Na * 3;
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_coord.p, coord, na3, cudaMemcpyDeviceToDevice, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_box.p, box, sizeof(double) * c.B * 9, cudaMemcpyDeviceToDevice, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_e.p, e_label, sizeof(double) * c.B, cudaMemcpyDeviceToDevice, s));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_f.p, f_label, na3, cudaMemcpyDeviceToDevice, s));
  if (c.o.force_groups > 0)
    FEKF_CHECK_CUDA(cudaMemcpyAsync(c.st_fidx.p, force_idx, sizeof(int32_t) * c.o.force_groups * c.o.atoms_per_group,
                                    cudaMemcpyDeviceToDevice, s));
  StepGraph* G = nullptr;
  FEKF_TRY(naive_graph(c, &G));
  FEKF_CHECK_CUDA(cudaEventRecord(c.gev_in, s));
  FEKF_CHECK_CUDA(cudaStreamWaitEvent(c.gstream, c.gev_in, 0));
  FEKF_CHECK_CUDA(cudaGraphLaunch(G->exec, c.gstream));
  FEKF_CHECK_CUDA(cudaEventRecord(c.gev_out, c.gstream));
  FEKF_CHECK_CUDA(cudaStreamWaitEvent(s, c.gev_out, 0));
  FEKF_CHECK_CUDA(cudaMemcpyAsync(metrics, c.st_met.p, sizeof(double) * 8, cudaMemcpyDeviceToDevice, s));
  c.kf->npend = G->npend_after;
  g_launches += G->launches;
  c.last_launches = G->launches;
  ++c.nsteps;
  return FEKF_OK;
}

fekf_status fekf_kf_update_naive_begin(fekf_kf* k, const double* G, int64_t ldg, int n, cudaStream_t s) {
  if (!k || !G) { set_error("kf_update_naive_begin: null"); return FEKF_EINVAL; }
  return k->kf.update_naive_begin(G, ldg, n, s);
}
fekf_status fekf_kf_naive_partial_u(fekf_kf* k, double** U, int64_t* len) {
  if (!k || !U || !len) { set_error("kf_naive_partial_u: null"); return FEKF_EINVAL; }
  if (k->kf.naive_n <= 0) { set_error("kf_naive_partial_u: no naive update begun"); return FEKF_ESTATE; }
  *U = k->kf.nU.as<double>();
  *len = k->kf.naive_u_len();
  return FEKF_OK;
}
fekf_status fekf_kf_update_naive_end(fekf_kf* k, const double* abe, double* w, double* A_out, cudaStream_t s) {
  if (!k || !abe || !w) { set_error("kf_update_naive_end: null"); return FEKF_EINVAL; }
  return k->kf.update_naive_end(abe, w, A_out, s);
}
fekf_status fekf_kf_update_naive(fekf_kf* k, const double* G, int64_t ldg, const double* abe, int n, double* w,
                                 double* A_out, cudaStream_t s) {
  if (!k || !G || !abe || !w) { set_error("kf_update_naive: null"); return FEKF_EINVAL; }
  return k->kf.update_naive(G, ldg, abe, n, w, A_out, s);
}

fekf_status fekf_set_graph_mode(fekf_ctx* ctx, int enable) {
  if (!ctx || (enable != 0 && enable != 1)) { set_error("set_graph_mode: bad args"); return FEKF_EINVAL; }
  Ctx& c = ctx->c;
  if (c.gstream) FEKF_CHECK_CUDA(cudaStreamSynchronize(c.gstream));
  if (!enable) c.drop_graphs();
  c.use_graph = enable != 0;
  return FEKF_OK;
}

fekf_status fekf_last_launch_count(const fekf_ctx* ctx, int64_t* n) {
  if (!ctx || !n) return FEKF_EINVAL;
  *n = ctx->c.last_launches;
  return FEKF_OK;
}

}  // extern "C"
