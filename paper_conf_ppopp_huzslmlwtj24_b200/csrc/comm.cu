// Library-owned NCCL communicator: the early reduction of [g || error sum]
// and, with sharded P, the reduction of the partial u = P g.  One process per GPU; NVLink/NVSwitch.
#include <nccl.h>

#include <cstring>

#include "kalman.cuh"

struct fekf_comm {
  ncclComm_t nc = nullptr;
  int rank = 0, world = 1;
};

namespace fekf {

int comm_world(fekf_comm* c) { return c ? c->world : 1; }
int comm_rank(fekf_comm* c) { return c ? c->rank : 0; }

fekf_status comm_allreduce(fekf_comm* c, double* buf, long long n, cudaStream_t s) {
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

fekf_status fekf_comm_destroy(fekf_comm* c) {
  if (!c) return FEKF_OK;
  if (c->nc) ncclCommDestroy(c->nc);
  delete c;
  return FEKF_OK;
}

fekf_status fekf_comm_allreduce_sum(fekf_comm* c, double* buf, int64_t n, cudaStream_t s) {
  if (!buf || n < 0) { fekf::set_error("allreduce: bad args"); return FEKF_EINVAL; }
  return fekf::comm_allreduce(c, buf, n, s);
}

}  // extern "C"
