// comm.cpp -- the communicator of a multi-rank context.  Only the per-round
// exchange of newly sampled RRR sets crosses ranks: an all-gather of one
// 64-bit count per rank and one broadcast per rank of its share (imm.cpp).
//
// Two backends behind one interface:
//   NcclComm   one process per GPU, NCCL over NVLink/NVSwitch (eim_create
//              with an NCCL unique id);
//   LocalComm  several ranks in ONE process (eim_create_group), each driven
//              by its own host thread; the collectives are host rendezvous
//              plus stream-ordered device copies (cudaMemcpyAsync with UVA,
//              so the ranks may share one GPU -- "virtual ranks" -- or sit on
//              different GPUs).  The IMM driver's multi-rank code (sharding,
//              compaction, rank-order append, histogram) is the same for both.
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "eim_internal.h"

namespace eim {

Comm::~Comm() = default;

// ------------------------------------------------------------------ NCCL
namespace {

void nccl_check(ncclResult_t r, const char* what) {
  if (r != ncclSuccess) fail(EIM_E_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

struct NcclComm final : Comm {
  ncclComm_t c = nullptr;
  ~NcclComm() override {
    if (c) ncclCommDestroy(c);
  }
  void allgather_u64(const uint64_t* d_send, uint64_t* d_recv, cudaStream_t st) override {
    nccl_check(ncclAllGather(d_send, d_recv, 1, ncclUint64, c, st), "ncclAllGather");
  }
  void broadcast(void* d_buf, size_t bytes, int root, cudaStream_t st) override {
    nccl_check(ncclBroadcast(d_buf, d_buf, bytes, ncclUint8, root, c, st), "ncclBroadcast");
  }
  void group_start() override { nccl_check(ncclGroupStart(), "ncclGroupStart"); }
  void group_end() override { nccl_check(ncclGroupEnd(), "ncclGroupEnd"); }
  const char* kind() const override { return "nccl"; }
};

}  // namespace

void comm_get_id(void* out) {
  static_assert(sizeof(ncclUniqueId) == EIM_NCCL_ID_BYTES, "NCCL unique id size");
  ncclUniqueId id;
  nccl_check(ncclGetUniqueId(&id), "ncclGetUniqueId");
  std::memcpy(out, &id, sizeof(id));
}

Comm* comm_create(int rank, int world, const void* id_bytes) {
  ncclUniqueId id;
  std::memcpy(&id, id_bytes, sizeof(id));
  NcclComm* c = new NcclComm();
  c->rank = rank;
  c->world = world;
  ncclResult_t r = ncclCommInitRank(&c->c, world, id, rank);
  if (r != ncclSuccess) {
    c->c = nullptr;
    delete c;
    nccl_check(r, "ncclCommInitRank");
  }
  return c;
}

void comm_destroy(Comm* c) { delete c; }

// ------------------------------------------------------------------ local
// Shared state of the ranks of one eim_create_group.  A collective is two
// rendezvous: (1) every rank has finished the device work its operand
// depends on (stream synchronised) and has published its pointer; each
// rank then pulls what it needs with copies on its own stream and waits for
// them; (2) nobody leaves before every rank has pulled, so no operand is
// reused early.  A rank that fails aborts the group: the others stop
// waiting and fail too (no hang), as does every later collective.
struct LocalGroup {
  int world = 0;
  int refs = 0;
  std::mutex mu;
  std::condition_variable cv;
  uint64_t gen = 0;
  int arrived = 0;
  bool aborted = false;
  std::vector<const void*> ptr;

  void rendezvous() {
    std::unique_lock<std::mutex> lk(mu);
    if (aborted) fail(EIM_E_NCCL, "a rank of the local group failed");
    const uint64_t g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
      return;
    }
    // generous bound: a peer that never arrives is a bug, not a slow kernel
    const bool ok = cv.wait_for(lk, std::chrono::seconds(1800), [&] { return gen != g || aborted; });
    if (aborted) fail(EIM_E_NCCL, "a rank of the local group failed");
    if (!ok) {
      aborted = true;
      cv.notify_all();
      fail(EIM_E_NCCL, "local group rendezvous timed out");
    }
  }
  void abort() {
    std::lock_guard<std::mutex> lk(mu);
    aborted = true;
    cv.notify_all();
  }
};

namespace {

struct LocalComm final : Comm {
  LocalGroup* grp = nullptr;
  ~LocalComm() override {
    bool last = false;
    {
      std::lock_guard<std::mutex> lk(grp->mu);
      last = --grp->refs == 0;
    }
    if (last) delete grp;
  }
  void publish(const void* p, cudaStream_t st) {
    EIM_CUDA(cudaStreamSynchronize(st));
    {
      std::lock_guard<std::mutex> lk(grp->mu);
      grp->ptr[rank] = p;
    }
    grp->rendezvous();
  }
  void allgather_u64(const uint64_t* d_send, uint64_t* d_recv, cudaStream_t st) override {
    publish(d_send, st);
    for (int q = 0; q < world; ++q)
      EIM_CUDA(cudaMemcpyAsync(d_recv + q, grp->ptr[q], sizeof(uint64_t), cudaMemcpyDefault, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    grp->rendezvous();
  }
  void broadcast(void* d_buf, size_t bytes, int root, cudaStream_t st) override {
    publish(d_buf, st);
    if (rank != root && bytes) EIM_CUDA(cudaMemcpyAsync(d_buf, grp->ptr[root], bytes, cudaMemcpyDefault, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    grp->rendezvous();
  }
  void abort() override { grp->abort(); }
  const char* kind() const override { return "local"; }
};

}  // namespace

LocalGroup* local_group_new(int world) {
  LocalGroup* g = new LocalGroup();
  g->world = world;
  g->ptr.assign((size_t)world, nullptr);
  return g;
}

void delete_local_group(LocalGroup* grp) { delete grp; }

Comm* comm_create_local(LocalGroup* grp, int rank) {
  LocalComm* c = new LocalComm();
  c->rank = rank;
  c->world = grp->world;
  c->grp = grp;
  std::lock_guard<std::mutex> lk(grp->mu);
  grp->refs++;
  return c;
}

}  // namespace eim
