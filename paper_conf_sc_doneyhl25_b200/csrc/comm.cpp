// comm.cpp -- NCCL communicator of a multi-GPU context (one process per GPU).
// Only the per-round exchange of newly sampled RRR sets crosses NVLink:
// an all-gather of the per-rank member counts and one broadcast per rank of
// its share (grouped), see imm.cpp.
#include <nccl.h>

#include <cstring>
#include <string>

#include "eim_internal.h"

namespace eim {

struct Comm {
  ncclComm_t c;
  int rank, world;
};

static void nccl_check(ncclResult_t r, const char* what) {
  if (r != ncclSuccess) fail(EIM_E_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

void comm_get_id(void* out) {
  static_assert(sizeof(ncclUniqueId) == EIM_NCCL_ID_BYTES, "NCCL unique id size");
  ncclUniqueId id;
  nccl_check(ncclGetUniqueId(&id), "ncclGetUniqueId");
  std::memcpy(out, &id, sizeof(id));
}

Comm* comm_create(int rank, int world, const void* id_bytes) {
  ncclUniqueId id;
  std::memcpy(&id, id_bytes, sizeof(id));
  Comm* c = new Comm{nullptr, rank, world};
  ncclResult_t r = ncclCommInitRank(&c->c, world, id, rank);
  if (r != ncclSuccess) {
    delete c;
    nccl_check(r, "ncclCommInitRank");
  }
  return c;
}

void comm_destroy(Comm* c) {
  if (!c) return;
  ncclCommDestroy(c->c);
  delete c;
}

void comm_allgather_u64(Comm* c, const uint64_t* d_send, uint64_t* d_recv, cudaStream_t st) {
  nccl_check(ncclAllGather(d_send, d_recv, 1, ncclUint64, c->c, st), "ncclAllGather");
}

void comm_broadcast(Comm* c, void* d_buf, size_t bytes, int root, cudaStream_t st) {
  nccl_check(ncclBroadcast(d_buf, d_buf, bytes, ncclUint8, root, c->c, st), "ncclBroadcast");
}

void comm_group_start() { nccl_check(ncclGroupStart(), "ncclGroupStart"); }
void comm_group_end() { nccl_check(ncclGroupEnd(), "ncclGroupEnd"); }

}  // namespace eim
