// NCCL plumbing for the row-block-sharded FW: one communicator per rank
// (one process per GPU), created from a unique id the caller distributes (torch.distributed).
// The only data-path collectives are the per-round pivot-row broadcast and the final all-gather of D.
#include <nccl.h>

#include "common.cuh"

namespace ear {

#define EAR_NCCL_TRY(expr)                                                                     \
  do {                                                                                         \
    ncclResult_t _r = (expr);                                                                  \
    if (_r != ncclSuccess) {                                                                   \
      ::ear::set_error("%s:%d %s: %s", __FILE__, __LINE__, #expr, ncclGetErrorString(_r));     \
      return EAR_ENCCL;                                                                        \
    }                                                                                          \
  } while (0)

ear_status_t comm_bcast(ear_comm_s *comm, int32_t *buf, int64_t count, int32_t root, cudaStream_t st) {
  EAR_NCCL_TRY(ncclBroadcast(buf, buf, (size_t)count, ncclInt32, root, (ncclComm_t)comm->nccl, st));
  return EAR_OK;
}

ear_status_t comm_allreduce_min(ear_comm_s *comm, int32_t *buf, int64_t count, cudaStream_t st) {
  EAR_NCCL_TRY(ncclAllReduce(buf, buf, (size_t)count, ncclInt32, ncclMin, (ncclComm_t)comm->nccl, st));
  return EAR_OK;
}

ear_status_t comm_allgather(ear_comm_s *comm, const int32_t *send, int32_t *recv, int64_t count,
                            cudaStream_t st) {
  EAR_NCCL_TRY(ncclAllGather(send, recv, (size_t)count, ncclInt32, (ncclComm_t)comm->nccl, st));
  return EAR_OK;
}

}  // namespace ear

extern "C" {

ear_status_t ear_comm_unique_id(uint8_t id[128]) {
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  ncclUniqueId u;
  EAR_NCCL_TRY(ncclGetUniqueId(&u));
  memcpy(id, &u, 128);
  return EAR_OK;
}

ear_status_t ear_comm_init(const uint8_t id[128], int32_t nranks, int32_t rank, ear_comm_t *out) {
  if (!id || !out || nranks < 1 || rank < 0 || rank >= nranks) {
    ear::set_error("ear_comm_init: bad arguments");
    return EAR_EINVAL;
  }
  ncclUniqueId u;
  memcpy(&u, id, 128);
  ncclComm_t c;
  EAR_NCCL_TRY(ncclCommInitRank(&c, nranks, u, rank));
  ear_comm_s *cm = new ear_comm_s;
  cm->nccl = c;
  cm->nranks = nranks;
  cm->rank = rank;
  cudaGetDevice(&cm->device);
  *out = cm;
  return EAR_OK;
}

ear_status_t ear_comm_info(ear_comm_t comm, int32_t *nranks, int32_t *rank) {
  if (!comm) {
    if (nranks) *nranks = 1;
    if (rank) *rank = 0;
    return EAR_OK;
  }
  if (nranks) *nranks = comm->nranks;
  if (rank) *rank = comm->rank;
  return EAR_OK;
}

void ear_comm_destroy(ear_comm_t comm) {
  if (!comm) return;
  if (comm->nccl) ncclCommDestroy((ncclComm_t)comm->nccl);
  delete comm;
}

}  // extern "C"
