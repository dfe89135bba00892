// Library-owned NCCL communicator: the early reduction of [g || error sum]
// and, with sharded P, the reduction of the partial u = P g.  One process per GPU; NVLink/NVSwitch.
//
// Loopback backend: `world` logical ranks in ONE process on one GPU, one host thread per
// rank.  A collective is a host barrier plus device work ordered by events: every rank sums all ranks'
// buffers in rank order 0..world-1 into its own scratch (same bits on every rank), and overwrites its
// buffer only after every rank has finished reading it.  This runs the sharded / data-parallel step
// (local_batch < global_batch, P sharded over contexts, both exchanges) on a single GPU.
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstring>
#include <memory>
#include <mutex>

#include "kalman.cuh"

namespace fekf {

struct LoopGroup {
  int world = 1;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  long long gen = 0;
  std::vector<double*> bufs;
  std::vector<cudaEvent_t> ready, done;
  std::vector<DBuf> scratch;
  int refs = 0;
  // generation barrier; false after `timeout_s` without every rank (a peer failed or never called)
  bool barrier(double timeout_s = 120.0) {
    std::unique_lock<std::mutex> lk(mu);
    const long long g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
      return true;
    }
    const bool ok = cv.wait_for(lk, std::chrono::duration<double>(timeout_s), [&] { return gen != g; });
    if (!ok) --arrived;
    return ok;
  }
};

}  // namespace fekf

struct fekf_comm {
  ncclComm_t nc = nullptr;
  int rank = 0, world = 1;
  std::shared_ptr<fekf::LoopGroup> loop;   // loopback backend (no NCCL)
};

namespace fekf {

int comm_world(fekf_comm* c) { return c ? c->world : 1; }
int comm_rank(fekf_comm* c) { return c ? c->rank : 0; }
bool comm_is_loopback(fekf_comm* c) { return c && c->loop; }

__global__ void loop_sum_kernel(const double* const* __restrict__ bufs, int world, long long n,
                                double* __restrict__ out) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double a = bufs[0][i];
  for (int r = 1; r < world; ++r) a += bufs[r][i];
  out[i] = a;
}

static fekf_status loop_allreduce(fekf_comm* c, double* buf, long long n, cudaStream_t s) {
  LoopGroup& G = *c->loop;
  const int r = c->rank;
  DBuf& sc = G.scratch[r];
  // per-rank scratch: the summed vector, and (after it) the table of the ranks' buffer pointers
  const size_t need = sizeof(double) * (size_t)n + sizeof(double*) * G.world;
  if (sc.bytes < need) {
    FEKF_CHECK_CUDA(cudaStreamSynchronize(s));
    dfree(sc);
    FEKF_TRY(dalloc(sc, need));
  }
  G.bufs[r] = buf;
  FEKF_CHECK_CUDA(cudaEventRecord(G.ready[r], s));
  if (!G.barrier()) { set_error("loopback allreduce: a peer rank did not arrive"); return FEKF_ESTATE; }
  for (int q = 0; q < G.world; ++q)
    if (q != r) FEKF_CHECK_CUDA(cudaStreamWaitEvent(s, G.ready[q], 0));
  double* sum = sc.as<double>();
  double** tab = reinterpret_cast<double**>(sum + n);
  FEKF_CHECK_CUDA(cudaMemcpyAsync(tab, G.bufs.data(), sizeof(double*) * G.world, cudaMemcpyHostToDevice, s));
  if (n > 0) {
    loop_sum_kernel<<<cdiv(n, 256), 256, 0, s>>>(tab, G.world, n, sum);
    FEKF_LAUNCH_CHECK();
    count_launch();
  }
  FEKF_CHECK_CUDA(cudaEventRecord(G.done[r], s));
  // the pointer table was staged from G.bufs: make the copy complete before a peer reuses the slot
  FEKF_CHECK_CUDA(cudaStreamSynchronize(s));
  if (!G.barrier()) { set_error("loopback allreduce: a peer rank did not arrive"); return FEKF_ESTATE; }
  for (int q = 0; q < G.world; ++q)
    if (q != r) FEKF_CHECK_CUDA(cudaStreamWaitEvent(s, G.done[q], 0));
  if (n > 0) FEKF_CHECK_CUDA(cudaMemcpyAsync(buf, sum, sizeof(double) * n, cudaMemcpyDeviceToDevice, s));
  return FEKF_OK;
}

fekf_status comm_allreduce(fekf_comm* c, double* buf, long long n, cudaStream_t s) {
  if (c && c->loop) return loop_allreduce(c, buf, n, s);
  if (!c || !c->nc) return FEKF_OK;
  ncclResult_t r = ncclAllReduce(buf, buf, (size_t)n, ncclDouble, ncclSum, c->nc, s);
  if (r != ncclSuccess) {
    set_error(std::string("ncclAllReduce: ") + ncclGetErrorString(r));
    return FEKF_ENCCL;
  }
  count_launch();
  return FEKF_OK;
}

}  // namespace fekf

extern "C" {

fekf_status fekf_get_unique_id(unsigned char id_host[128]) {
  if (!id_host) { fekf::set_error("null id"); return FEKF_EINVAL; }
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) { fekf::set_error(std::string("ncclGetUniqueId: ") + ncclGetErrorString(r)); return FEKF_ENCCL; }
  static_assert(sizeof(ncclUniqueId) == 128, "nccl id size");
  std::memcpy(id_host, &id, 128);
  return FEKF_OK;
}

fekf_status fekf_comm_init(int rank, int world, const unsigned char id_host[128], fekf_comm** out) {
  if (!out || !id_host || world < 1 || rank < 0 || rank >= world) { fekf::set_error("comm_init: bad args"); return FEKF_EINVAL; }
  fekf_comm* c = new fekf_comm();
  c->rank = rank;
  c->world = world;
  {  // a single-rank communicator is a real NCCL communicator too (exercises the same path on one GPU)
    ncclUniqueId id;
    std::memcpy(&id, id_host, 128);
    ncclResult_t r = ncclCommInitRank(&c->nc, world, id, rank);
    if (r != ncclSuccess) {
      fekf::set_error(std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
      delete c;
      return FEKF_ENCCL;
    }
  }
  *out = c;
  return FEKF_OK;
}

fekf_status fekf_comm_init_loopback(int world, fekf_comm** out) {
  if (!out || world < 1 || world > 64) { fekf::set_error("comm_init_loopback: bad args"); return FEKF_EINVAL; }
  auto G = std::make_shared<fekf::LoopGroup>();
  G->world = world;
  G->bufs.assign(world, nullptr);
  G->ready.assign(world, nullptr);
  G->done.assign(world, nullptr);
  G->scratch.resize(world);
  for (int r = 0; r < world; ++r) {
    if (cudaEventCreateWithFlags(&G->ready[r], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&G->done[r], cudaEventDisableTiming) != cudaSuccess) {
      fekf::set_error("comm_init_loopback: cudaEventCreate failed");
      return FEKF_ECUDA;
    }
  }
  for (int r = 0; r < world; ++r) {
    fekf_comm* c = new fekf_comm();
    c->rank = r;
    c->world = world;
    c->loop = G;
    out[r] = c;
  }
  return FEKF_OK;
}

fekf_status fekf_comm_destroy(fekf_comm* c) {
  if (!c) return FEKF_OK;
  if (c->nc) ncclCommDestroy(c->nc);
  if (c->loop && c->loop.use_count() == 1) {   // last rank of the group: release the shared resources
    cudaDeviceSynchronize();
    for (auto& e : c->loop->ready) if (e) cudaEventDestroy(e);
    for (auto& e : c->loop->done) if (e) cudaEventDestroy(e);
    for (auto& b : c->loop->scratch) fekf::dfree(b);
  }
  delete c;
  return FEKF_OK;
}

fekf_status fekf_comm_allreduce_sum(fekf_comm* c, double* buf, int64_t n, cudaStream_t s) {
  if (!buf || n < 0) { fekf::set_error("allreduce: bad args"); return FEKF_EINVAL; }
  return fekf::comm_allreduce(c, buf, n, s);
}

}  // extern "C"
