// eim_internal.h -- shared declarations of the CUDA path (never of the oracle).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "eim.h"

namespace eim {

// Thrown inside the library only; converted to eim_status at the ABI.
struct Error {
  eim_status code;
  std::string msg;
};

[[noreturn]] void fail(eim_status code, const std::string& msg);
void cuda_check(cudaError_t e, const char* what, const char* file, int line);
#define EIM_CUDA(x) ::eim::cuda_check((x), #x, __FILE__, __LINE__)

// Device buffer with geometric growth (contents optionally preserved).
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  void reserve(size_t need, bool keep, cudaStream_t st);
  void release();
  template <class T> T* as() const { return static_cast<T*>(p); }
};

// Device-resident reverse CSR.
struct GraphView {
  uint32_t n;
  uint64_t m;
  const uint64_t* off;   // n+1
  const uint32_t* nbr;   // m
  const uint32_t* thr;   // n: IC threshold floor((2^32-1)/d), 0 if d == 0
};

// Log-encoded reverse CSR (NEXT-2; layout R24): offsets and
// in-neighbours bit-packed with n_b = bit_width(max) bits each, in 32-bit
// containers (two zero words of padding so a decode may read 3 words).  No
// threshold array: T_v = floor((2^32-1)/d) is recomputed from the decoded
// degree once per expanded vertex.
struct PackedGraphView {
  uint32_t n;
  uint64_t m;
  const uint32_t* offw;  // n+1 values of boff bits
  const uint32_t* nbrw;  // m values of bnbr bits
  uint32_t boff, bnbr;
};

// Reverse CSR with general edge probabilities (NEXT-3, R25): in-edge e has
// p_e = (x_e + 1) / 2^32.  IC: live iff draw <= x_e.  LT: cum_e = (sum of
// w_i = x_i + 1 over the row up to and including e) - 1, so the choice is the
// first e of the row with cum_e >= tau (none if tau > the row's last cum).
// x is padded with zeros to a multiple of 4 entries (quad loads).
struct WeightedGraphView {
  uint32_t n;
  uint64_t m;
  const uint64_t* off;
  const uint32_t* nbr;
  const uint32_t* x;    // m (padded to 4): IC thresholds
  const uint32_t* cum;  // m: LT inclusive cumulative weights - 1 (valid when the graph's lt_ok)
};

// Log-encoded reverse CSR with general edge probabilities (NEXT-2 x NEXT-3):
// offsets and in-neighbours packed as in PackedGraphView ("applied to
// both the network data and the RRR sets"); the per-edge probabilities x
// and LT cumulative weights cum stay 32-bit (they are not small integers).
struct PackedWeightedGraphView {
  uint32_t n;
  uint64_t m;
  PackedGraphView p;
  const uint32_t* x;
  const uint32_t* cum;
};

// Per-launch control block (device memory).  The counters that every group
// polls or bumps sit on separate 128-byte lines.
struct SampleCtl {
  unsigned long long ticket, pad0[15];          // next sample id (s_local)
  unsigned long long thead, ttail, pad1[14];    // tasks claimed / pushed over all queues (a hint for idle groups)
  unsigned long long ptail, pad2[15];           // task seed pool: reserved
  unsigned long long outstanding, pad3[15];     // samples + tasks taken or queued, not finished
  unsigned long long edges;                     // examined in-edges / walk steps (finalize)
  unsigned long long arena_fail;                // table or task pool full: redo the round larger
  unsigned long long spilled;                   // samples that split off tasks
  unsigned long long tasks_pushed;              // tasks split off
  unsigned long long t_first, t_last_id, t_end;  // %globaltimer: first id taken, last id taken, last group exit (timeline)
  unsigned long long consumed;                   // source elimination: ids up to the last kept set
  unsigned long long ntickets;                   // IC: ids that need a traversal (the root pre-pass list)
  unsigned long long pad4[7];
};

// Communicator of a multi-rank context (comm.cpp): NCCL across processes,
// or an in-process group of ranks (eim_create_group).  Collectives are
// stream-ordered on `st`; every rank calls them in the same order.
struct Comm {
  int rank = 0, world = 1;
  virtual ~Comm();
  // d_recv[q] = rank q's *d_send (one u64 per rank)
  virtual void allgather_u64(const uint64_t* d_send, uint64_t* d_recv, cudaStream_t st) = 0;
  // every rank's d_buf[0, bytes) = root's
  virtual void broadcast(void* d_buf, size_t bytes, int root, cudaStream_t st) = 0;
  virtual void group_start() {}
  virtual void group_end() {}
  // this rank failed: release the peers waiting in a collective (local groups)
  virtual void abort() {}
  virtual const char* kind() const = 0;
};
struct LocalGroup;

// One sampler launch over sample ids [first, first+count): its membership
// table and per-sample scratch.  Two of them let the IMM driver sample the
// next round speculatively while the greedy of the current round runs.
// Round output flags: source elimination (R22) drops each sample's root from
// its set; with RF_DROP_EMPTY the sets left empty are discarded and only
// the first `use` non-empty sets (in sample-id order) are kept.
enum : uint32_t { RF_DROP_ROOT = 1u, RF_DROP_EMPTY = 2u };

struct SampleResult {
  uint64_t edges = 0;     // (unused: examined edges accumulate on the device, edges_read)
  uint64_t spilled = 0;   // samples finished in the shared frontier queue
  uint32_t launches = 0;
  double kernel_ms = 0;
  uint64_t kept = 0;      // sets appended to the arena
  uint64_t consumed = 0;  // sample ids used (> kept when empty sets are dropped)
};

struct Round {
  DevBuf table, sizes, edges, fill, excl, ctl;  // ctl: SampleCtl + cancel/pause flags
  DevBuf roots, kidx, ksizes;                    // source elimination: roots, kept-set index, kept sizes
  DevBuf dbg;                                    // EIM_DEBUG_TIMELINE per-sample records
  DevBuf queue;                                  // IC task pool (u32 seeds) + descriptors (all-zero between rounds)
  DevBuf list;                                   // IC: s_local of the ids whose root has in-edges (pre-pass)
  uint64_t first = 0, count = 0, set_base = 0, seed = 0, pcap = 0, tcap = 0;
  bool qdirty = true;                            // descriptors need a memset before use
  uint32_t bits = 0;
  eim_model model = EIM_IC;
  cudaStream_t stream = nullptr;  // stream the sampler kernels were launched on
  static constexpr int MAX_LAUNCH = 8;
  cudaEvent_t ev[2 * MAX_LAUNCH] = {};  // start/stop of every sampler launch of the round
  int nlaunch = 0;
  bool launched = false;
  bool waited = false;  // the launch has finished (round_finalize with keep appends the rest later)
  bool hist = true;
  uint32_t rflags = 0;
  SampleResult pend;          // launch statistics not yet reported by round_finalize
  bool elim_ready = false;    // RF_DROP_EMPTY: roots dropped from the sizes, kidx scanned (round_elim_kept)
  uint64_t kept_total = 0;    // RF_DROP_EMPTY: non-empty sets of the launch
};

// Buffers and stream of one greedy NodeSelection (select.cu).  Two slots let
// the IMM driver run the selections of two rounds concurrently.
struct GreedySlot {
  DevBuf C_work, inv_off, inv_fill, inv, best, seeds, gains, cand, cidx, arena_c, selected, covered, scratch, dirty;
  cudaStream_t stream = nullptr;  // slot 0: the context's stream; slot 1: its own
  bool own_stream = false;
  cudaEvent_t ev[2] = {};          // around the pick kernel
  void release();
};

}  // namespace eim

struct eim_graph {
  uint32_t magic;
  eim_ctx* ctx;
  eim::GraphView view;
  void* d_off = nullptr;
  void* d_nbr = nullptr;
  void* d_thr = nullptr;
  bool packed = false;           // log-encoded store (EIM_G_LOG_ENCODE): pview, d_offw, d_nbrw
  eim::PackedGraphView pview{};
  void* d_offw = nullptr;
  void* d_nbrw = nullptr;
  bool weighted = false;         // general edge probabilities (eim_load_graph_csr_weighted): wview, d_x, d_cum
  eim::WeightedGraphView wview{};
  void* d_x = nullptr;
  void* d_cum = nullptr;
  eim::PackedWeightedGraphView pwview{};  // packed && weighted
  void* d_aug = nullptr;         // LT walk store of the plain graph, built on the first LT run (uint4 per in-edge)
  uint64_t aug_bytes = 0;
  bool aug_failed = false;       // the walk store did not fit: LT runs on the plain store
  bool lt_ok = true;             // weighted: every row's weights sum to <= 2^32 (LT usable)
  uint64_t bytes = 0;            // device bytes of the store
  int proper_edge = -1;  // has an edge u -> v, u != v (1/0; -1 = not yet computed)
};

struct eim_ctx {
  uint32_t magic;
  int device, rank, world;
  cudaStream_t stream;
  bool own_stream;
  eim::Comm* comm;
  std::string last_error;
  int sm_count;
  uint64_t kernel_launches;

  // arena (persistent, grows)
  eim::DevBuf arena, set_start, set_len;
  eim::DevBuf ctl;            // SampleCtl
  eim::Round rounds[2];                         // current + speculative sampler rounds
  cudaStream_t rstream[2] = {};                 // sampler streams of rounds[0], rounds[1]
  cudaStream_t aux_stream = nullptr;            // cancel-flag writes
  double est_mean_size = 0;                     // mean set size of earlier rounds (table sizing)
  uint64_t arena_used = 0;                      // arena elements in use (host is the authority)
  uint32_t arena_b = 32;                        // bits per arena element: 32 plain, else log-encoded (R24)
  // per-graph vectors
  eim::DevBuf C_total, C_snap, C_snap2;         // coverage counts of R; snapshots for concurrent selections
  eim::DevBuf edges_acc;                        // examined edges / walk steps of the current call (u64)
  eim::GreedySlot gs[3];                        // greedy NodeSelection slots
  eim::DevBuf scratch;        // CUB temp storage
  eim::DevBuf stage_a, stage_b, stage_c;  // export / exchange staging
  void* h_pinned = nullptr;   // small pinned host scratch
  cudaEvent_t ev0, ev1;
  eim_stats last_stats;       // statistics of the most recent hot-path call
  uint32_t cov_n = 0;         // n of the coverage counts C_total of the last imm_run / select_seeds (0: none)
};

namespace eim {

// Calls f with the device view of g's store (every kernel that walks the
// reverse CSR is a template over the view).
template <class F>
auto with_graph_view(const eim_graph* g, F&& f) {
  if (g->packed && g->weighted) return f(g->pwview);
  if (g->packed) return f(g->pview);
  if (g->weighted) return f(g->wview);
  return f(g->view);
}

constexpr uint32_t CTX_MAGIC = 0xE1A0C7A7u;
constexpr uint32_t GRAPH_MAGIC = 0xE1A06A7Fu;
constexpr uint32_t SENTINEL = 0xFFFFFFFFu;

// ---- graph.cu
void graph_validate_and_thresholds(eim_ctx* ctx, eim_graph* g);
// Replace the plain store by its log encoding (frees off/nbr/thr).
void graph_log_encode(eim_ctx* ctx, eim_graph* g);
// Attach per-edge probabilities x (host, m entries) to a validated plain store.
void graph_attach_weights(eim_ctx* ctx, eim_graph* g, const uint32_t* h_x);
bool graph_has_proper_edge(eim_ctx* ctx, const eim_graph* g);

// ---- sample.cu
// Sample ids per launch that keep the round's membership table within its
// memory budget (from the mean set size of earlier launches).
uint64_t max_launch_ids(const eim_ctx* ctx);
// Examined in-edges (IC) / walk steps (LT) of the appended sets accumulate
// in a device counter (no host round trip per launch): reset, read (syncs).
void edges_reset(eim_ctx* ctx);
uint64_t edges_read(eim_ctx* ctx);
// Samples ids [first, first+count) into ctx->arena; set index = id - set_base
// (in launches of at most max_launch_ids ids).
// Histogram into C when hist is true.  (= round_launch + round_finalize)
SampleResult sample_range(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed,
                          uint64_t first, uint64_t count, uint64_t set_base, bool hist, uint32_t rflags = 0);
// Launch the sampler for ids [first, first+count) into rd on stream st (no
// host synchronisation).  spare_sm_slot: leave one block slot per SM free
// (for a concurrent greedy kernel).
void round_launch(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed, uint64_t first,
                  uint64_t count, uint64_t set_base, bool hist, Round& rd, cudaStream_t st, bool spare_sm_slot,
                  uint32_t rflags = 0);
// Wait for rd, redo what overflowed, and append its first `use` sets to the
// arena (sample-id order) with their histogram.  With RF_DROP_EMPTY, `use`
// is the number of non-empty sets wanted (res.kept <= use, res.consumed ids).
// from/keep: append only s_local in [from, use) and keep the round for a
// later append of the rest (plain rounds; the IMM driver's lookahead).
// consume_all (RF_DROP_EMPTY, use = every non-empty set of the launch): all
// ids of the launch count as consumed (a multi-rank round whose cut lies on
// a later rank).
// cuts (plain rounds, one GPU): the append also leaves, for each cut j,
// snap[j] = C over the sets up to s_local cut[j] (C from before the append
// plus those sets' members) and total[j] = the arena elements up to that
// set -- the inputs of the run-ahead selections of the rounds the append
// covers, in one scan, one host read-back and one scatter instead of one per
// round.
struct AppendCuts {
  uint32_t n = 0;        // <= 2
  uint64_t cut[2] = {};  // s_local, from < cut < use
  uint32_t* snap[2] = {};
  uint64_t total[2] = {};  // out
};
SampleResult round_finalize(eim_ctx* ctx, const eim_graph* g, Round& rd, uint64_t use, uint64_t from = 0,
                            bool keep = false, bool consume_all = false, AppendCuts* cuts = nullptr);
// RF_DROP_EMPTY rounds: wait, drop the roots and count the non-empty sets
// of the whole launch (idempotent; round_finalize then keeps the first `use`).
uint64_t round_elim_kept(eim_ctx* ctx, const eim_graph* g, Round& rd);
// Stop a launched speculative round and wait for it.
void round_cancel(eim_ctx* ctx, Round& rd);
// Let a launched round take no new sample ids (its running samples finish);
// round_resume relaunches it on st, continuing with the remaining ids.
void round_pause(eim_ctx* ctx, Round& rd);
void round_resume(eim_ctx* ctx, const eim_graph* g, Round& rd, cudaStream_t st);
void round_release(Round& rd);
// Empty the arena; b = bits per element (32: plain u32; < 32: log-encoded,
// P:99-101, layout R24, written with atomicOr so concurrent writers of one
// container are safe -- the "thread-safe log encoding" of P:99).
void arena_reset(eim_ctx* ctx, uint32_t b = 32);
// Capacity for `elems` elements (contents kept; new containers zeroed when encoded).
void arena_ensure(eim_ctx* ctx, uint64_t elems);
inline uint64_t arena_words(uint64_t elems, uint32_t b) { return (elems * b + 31) / 32 + 2; }
uint32_t bit_width(uint64_t x);
void ensure_sets(eim_ctx* ctx, uint64_t num_sets);
uint64_t arena_cursor(eim_ctx* ctx);

// ---- arena.cu
// canonical export: offsets (count+1, device u64) + members (device u32), sets ascending
// (members are sorted only when the total fits members_cap: otherwise the
// caller reports EIM_E_CAPACITY and copies none)
uint64_t export_sets(eim_ctx* ctx, uint64_t count, uint64_t** d_offsets, uint32_t** d_members,
                     uint64_t members_cap = UINT64_MAX);
// histogram of sets [lo, hi) into C_total (sign -1: out of it)
void hist_sets(eim_ctx* ctx, uint64_t lo, uint64_t hi, int sign = 1);
// Remove the last sets [keep, R) of a plain (32-bit) arena: out of C_total
// and the arena; *edges = their examined edges (IC) / walk steps (LT).
void drop_sets(eim_ctx* ctx, const eim_graph* g, bool ic, uint64_t keep, uint64_t R, uint64_t* edges);
// append externally supplied canonical sets (device pointers) as set ids [base, base+count)
void append_sets(eim_ctx* ctx, uint64_t base, uint64_t count, const uint64_t* d_offsets,
                 const uint32_t* d_members, uint64_t total);

// ---- select.cu
// Greedy NodeSelection over sets [0, num_sets) (arena elements [0, total))
// with coverage counts C[0..n).  Writes seeds/gains (host), returns cov.
uint64_t greedy(eim_ctx* ctx, uint32_t n, uint64_t num_sets, uint32_t k, uint32_t* seeds_out,
                uint64_t* gains_out, double* kernel_ms = nullptr);
// The same, split: enqueue on slot `slot` (its stream waits for the context's
// stream first), then wait and read the result.  C and the arena prefix must
// stay unchanged until greedy_collect.
void greedy_launch(eim_ctx* ctx, int slot, uint32_t n, uint64_t num_sets, uint64_t total, const uint32_t* C,
                   uint32_t k);
// greedy_launch in two halves, so two slots' setups can overlap before the
// host reads their candidate counts
void greedy_setup(eim_ctx* ctx, int slot, uint32_t n, uint64_t num_sets, uint64_t total, const uint32_t* C);
// blocks_share: the blocks of this selection when several run at the same
// time (greedy_shares), 0 = one per SM
void greedy_picks(eim_ctx* ctx, int slot, uint32_t n, uint64_t num_sets, uint32_t k, uint32_t blocks_share);
void greedy_shares(eim_ctx* ctx, uint32_t nsel, const uint64_t* num_sets, uint32_t* blocks);
uint64_t greedy_collect(eim_ctx* ctx, int slot, uint32_t k, uint32_t* seeds_out, uint64_t* gains_out,
                        double* kernel_ms = nullptr);

// development (EIM_TRACE=1): host timestamps of the IMM phases on stderr,
// in ms since the last trace_reset (marks after a host synchronisation
// approximate the device's completion time)
void trace_reset();
void trace_mark(const char* what, uint64_t a = 0, uint64_t b = 0);

// ---- imm.cpp
void imm_params(uint32_t n, uint32_t k, double eps, double ell, eim_imm_params_t* out);
void imm_run(eim_ctx* ctx, const eim_graph* g, uint32_t k, double eps, double ell, eim_model model,
             uint64_t seed, uint32_t flags, uint32_t* seeds_out, uint64_t* theta_out, double* spread_out,
             eim_stats* st);

// ---- comm.cpp
Comm* comm_create(int rank, int world, const void* id);  // NCCL
LocalGroup* local_group_new(int world);
void delete_local_group(LocalGroup* grp);                // only if no comm holds it
Comm* comm_create_local(LocalGroup* grp, int rank);      // takes a reference on grp
void comm_destroy(Comm* c);
void comm_get_id(void* out);

inline uint32_t grid_for(eim_ctx* ctx, uint64_t work, uint32_t per_block, uint32_t blocks_per_sm = 8) {
  uint64_t b = (work + per_block - 1) / per_block;
  uint64_t cap = (uint64_t)ctx->sm_count * blocks_per_sm;
  if (b > cap) b = cap;
  if (b == 0) b = 1;
  return (uint32_t)b;
}

}  // namespace eim
