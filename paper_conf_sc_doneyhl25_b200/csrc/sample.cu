// sample.cu -- RRR-set samplers (Alg. 2, P:107 for IC; P:134-140 for LT).
//
// One sampler launch handles a contiguous range of sample ids [first,
// first+count) (a "round").  Membership of every set of the round is kept in
// ONE global open-addressing table keyed by (sample, vertex) (64-bit keys,
// ~32 MB at C2, L2-resident), so no set ever outgrows its storage: the
// per-sample state on chip is only the FRONTIER (discovered, not yet
// expanded vertices).  After the launch the per-sample sizes are scanned into
// arena offsets (sample-id order) and a scatter pass over the table writes
// every member into the arena and bumps the coverage histogram C (Alg. 2 l.25)
// -- placement is deterministic, no reservation atomics, no arena overflow.
//
// IC (ic_kernel<G>): persistent groups of G threads.  A group takes a sample
//   id and runs it in shared memory (local_sample): a batch of up to G
//   frontier vertices has its in-rows merged into one space of Philox quads
//   (4 consecutive edge ids share one Philox4x32-10 call, reading R1) that
//   the G threads sweep, so small rows do not idle threads and hub rows split
//   evenly.  An edge into u is live iff its draw <= T_u (R2); in_nbr[e] is
//   read only for live edges.  Under WC a few samples per round are huge
//   (~10^5 members, ~10^6 quads): on one group they would bound the round.
//   So after every spill_quads swept quads a traversal cuts its backlog into
//   pieces of about task_quads quads each, keeps one and pushes the others as
//   TASKS (a sample id and its seed vertices) that any group runs the same
//   way, before it takes a new id.  Membership stays in the round table (first insert wins
//   and expands the vertex), so nothing is redone and the union of the
//   traversals is the unique reachable set.
// LT (lt_kernel): one thread per reverse walk (sequential by nature),
//   visited set = the same global table; no capacity limit.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdio>
#include <type_traits>
#include <vector>
#include <cstdlib>
#include <string>

#include "arena_view.cuh"
#include "philox.cuh"

namespace eim {

namespace {

constexpr unsigned FULL = 0xFFFFFFFFu;
constexpr uint32_t MAX_PROBE = 256;

#ifndef EIM_IC_G
#define EIM_IC_G 256
#endif
#ifndef EIM_IC_NSG
#define EIM_IC_NSG 1
#endif
constexpr int IC_G = EIM_IC_G;      // threads per sub-group (one traversal at a time)
constexpr int IC_NSG = EIM_IC_NSG;  // sub-groups per block (one block per SM)

// ---------------------------------------------------------------- table
// key = (s_local + 1) << 32 | v ;  0 = empty slot.  The same 64-bit word is
// the item format of the shared frontier queue.
__device__ __forceinline__ unsigned long long table_key(uint32_t s_local, uint32_t v) {
  return ((unsigned long long)(s_local + 1u) << 32) | (unsigned long long)v;
}

__device__ __forceinline__ uint32_t table_hash(unsigned long long key, uint32_t bits) {
  unsigned long long h = key * 0x9E3779B97F4A7C15ull;
  h ^= h >> 29;
  h *= 0xBF58476D1CE4E5B9ull;
  return (uint32_t)(h >> (64 - bits));
}

// 1 = inserted (new member), 0 = already present, -1 = table too full
__device__ __forceinline__ int table_insert(unsigned long long* keys, uint32_t bits, unsigned long long key) {
  const uint32_t mask = (uint32_t)((1ull << bits) - 1ull);
  uint32_t i = table_hash(key, bits);
  for (uint32_t p = 0; p < MAX_PROBE; ++p) {
    const unsigned long long cur = atomicCAS(&keys[i], 0ull, key);
    if (cur == 0ull) return 1;
    if (cur == key) return 0;
    i = (i + 1u) & mask;
  }
  return -1;
}

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ unsigned long long vload(const unsigned long long* p) {
  return *(const volatile unsigned long long*)p;
}

// ---------------------------------------------------------------- groups
// A block is NSG sub-groups of G threads.  A sub-group runs one traversal at
// a time and synchronises on its own named barrier; the sub-groups of a
// block share nothing but the sweep jobs below (shared memory).
template <int G>
__device__ __forceinline__ void gsync(int gi) {
  asm volatile("bar.sync %0, %1;" ::"r"(gi + 1), "r"(G) : "memory");
}

// Sweep job of a sub-group's current batch.  Warps claim chunks of ch quads
// through `claim` = epoch << 48 | nchunks << 24 | next chunk (an old epoch or
// next >= nchunks claims nothing), so the warps of the other sub-groups of
// the block can join a heavy batch (open = 1) between their own batches or
// when they are idle.  done counts finished chunks of the epoch.
struct Job {
  unsigned long long claim;
  uint32_t done, open;
  uint32_t total, nrows, s_local, head, ch, hoist;
};

struct GroupCtl {
  uint32_t tail, flag, s_local, nlive;
  uint32_t pushed, action, nb, epoch;  // pushed: this traversal split off a task
  uint32_t hiq, pad_[3];               // hiq: a staged row reached Philox quads >= 2^32 (no hoisting)
  unsigned long long h, base;
  Job job;
  uint32_t wsum[32];  // one per warp (G <= 1024)
};

template <int G>
struct GroupRows {
  unsigned long long q0[G];  // first Philox quad of the row
  uint32_t qend[G];          // inclusive scan of quad counts
  uint32_t nq[G];            // quads of the row
  uint32_t T[G];             // IC threshold of the row's vertex
  uint8_t wlo[G], whi[G];    // first valid word of the first quad, last valid word of the last quad
};

template <int G>
__device__ __forceinline__ uint32_t group_incl_scan(uint32_t x, int gtid, int gi, GroupCtl& gc, uint32_t& total) {
  const int lane = gtid & 31, w = gtid >> 5;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += t;
  }
  if (lane == 31) gc.wsum[w] = x;
  gsync<G>(gi);
  uint32_t pre = 0, tot = 0;
#pragma unroll
  for (int i = 0; i < G / 32; ++i) {
    const uint32_t t = gc.wsum[i];
    pre += (i < w) ? t : 0u;
    tot += t;
  }
  total = tot;
  return x + pre;
}

enum : uint32_t { FLAG_TABLE = 2u, FLAG_CANCEL = 4u };
enum : uint32_t { ACT_EXIT = 0u, ACT_LOCAL = 1u, ACT_TASK = 2u, ACT_IDLE = 3u };

struct RoundView {
  unsigned long long* keys;
  uint32_t bits;
  uint32_t* sizes;               // [count] members per sample (s_local)
  unsigned long long* edges;     // [count] walk steps per sample (LT)
  const unsigned int* cancel;    // [0] cancel (round not needed), [1] pause (take no new work)
  uint64_t base;                 // sample id of s_local = 0
  uint32_t* pool;                // task seed vertices
  unsigned long long* tasks;     // task descriptors: [2i] pool offset, [2i+1] (s_local+1) << 32 | nv (0 = unwritten)
  uint64_t pcap, tcap;           // pool / descriptor capacity
  unsigned long long* dbg;       // [count][8] per root traversal (EIM_DEBUG_TIMELINE), nullable
  PhiloxKey K;                   // round keys of the seed (kernel parameter: read as constant operands)
  uint32_t nohoist;              // 1: never use the hoisted edge draws (tests exercise the general path)
  unsigned long long* qc;        // task queue q: head at qc[16 q], tail at qc[16 q + 1] (one 128-B line each)
  uint32_t prefetch;             // L2-prefetch in_nbr of parked live edges (EIM_NO_PREFETCH=1 turns it off)
  const uint32_t* list;          // IC: ticket t -> s_local (the ids whose root has in-edges; root pre-pass)
  uint32_t lt_evict;             // LT walk-store loads marked evict-first in L2 (EIM_LT_NO_EVICT=1: default policy)
};

// Split-off tasks go to TQ queues (descriptor segments of tcap / TQ each):
// a producer pushes to the queue of its block, a consumer claims from its
// own queue first and then from the others.  With one queue every claim of
// the round went through one CAS on one counter, about one claim per L2
// round trip for the whole GPU, which bounded the heavy configs.
constexpr uint32_t TQ = 16;
__device__ __forceinline__ uint32_t home_queue() { return blockIdx.x % TQ; }

constexpr uint32_t LIVE_CAP = 512;  // live in-edges parked per batch (more are visited inline)

// Row descriptors of queued frontier vertices, loaded when the vertex is
// discovered: the next batch stages its rows from shared memory.
struct RingRows {
  unsigned long long* e0;  // [W] first in-edge
  uint32_t* d;             // [W] in-degree
  uint32_t* T;             // [W] IC threshold
};

// One sub-group's shared-memory region.
template <int G>
struct SG {
  GroupCtl* gc;
  GroupRows<G>* rw;
  RingRows rr;
  uint32_t* ring;
  unsigned long long* live_e;  // parked live edges of the current batch
};

template <int G>
__host__ __device__ constexpr size_t sg_bytes(uint32_t W) {
  return (sizeof(GroupCtl) + sizeof(GroupRows<G>) + 20ull * W + 8ull * LIVE_CAP + 15) & ~(size_t)15;
}

template <int G>
__device__ __forceinline__ SG<G> sg_at(unsigned char* smem, int gi, uint32_t W) {
  unsigned char* p = smem + (size_t)gi * sg_bytes<G>(W);
  SG<G> r;
  r.gc = reinterpret_cast<GroupCtl*>(p);
  p += sizeof(GroupCtl);
  r.rw = reinterpret_cast<GroupRows<G>*>(p);
  p += sizeof(GroupRows<G>);
  r.rr.e0 = reinterpret_cast<unsigned long long*>(p);
  p += 8ull * W;
  r.ring = reinterpret_cast<uint32_t*>(p);
  p += 4ull * W;
  r.rr.d = reinterpret_cast<uint32_t*>(p);
  p += 4ull * W;
  r.rr.T = reinterpret_cast<uint32_t*>(p);
  p += 4ull * W;
  r.live_e = reinterpret_cast<unsigned long long*>(p);
  return r;
}

__device__ __forceinline__ void mark_fail(SampleCtl* ctl) {
  atomicOr(reinterpret_cast<unsigned int*>(&ctl->arena_fail), 1u);
}

// Publish task i: descriptor word 0 (pool offset) is made visible before
// word 1, which a consumer spins on.
__device__ __forceinline__ void task_write(const RoundView& R, unsigned long long i, unsigned long long poff,
                                           uint32_t s_local, uint32_t nv) {
  R.tasks[2 * i] = poff;
  __threadfence();
  *(volatile unsigned long long*)&R.tasks[2 * i + 1] = ((unsigned long long)(s_local + 1u) << 32) | nv;
}

// Push one vertex as a task of its own (ring overflow; rare).  outstanding is
// raised before the task becomes visible.
__device__ __forceinline__ void task_push1(const RoundView& R, SampleCtl* ctl, uint32_t s_local, uint32_t v) {
  atomicAdd(&ctl->outstanding, 1ull);
  const unsigned long long po = atomicAdd(&ctl->ptail, 1ull);
  const uint32_t q = home_queue();
  const unsigned long long tq = R.tcap / TQ;
  const unsigned long long qi = atomicAdd(&R.qc[16 * q + 1], 1ull);
  atomicAdd(&ctl->ttail, 1ull);  // hint: tasks pushed (all queues)
  const unsigned long long ti = q * tq + qi;
  if (qi >= tq) {  // descriptor segment full: host redoes the round larger
    mark_fail(ctl);
    atomicAdd(&ctl->outstanding, ~0ull);
    return;
  }
  if (po >= R.pcap) {  // pool full: an empty task keeps the claimed slot consumable
    mark_fail(ctl);
    task_write(R, ti, 0, s_local, 0);
    return;
  }
  R.pool[po] = v;
  __threadfence();
  task_write(R, ti, po, s_local, 1);
}

// visit v for the traversal of sub-group o (sample s_local, ring head `head`):
// table insert; a new member is appended to o's ring with its row (loaded
// alongside the insert), or becomes a one-vertex task when the ring is full.
template <int G, class GV>
__device__ __forceinline__ void visit_for(const GV& g, const RoundView& R, SampleCtl* ctl, const SG<G>& o,
                                          uint32_t s_local, uint32_t head, uint32_t W, uint32_t v) {
  const unsigned long long e0 = g_off(g, v), e1 = g_off(g, v + 1);
  const uint32_t T = g_thr(g, v, e1 - e0);
  const int ins = table_insert(R.keys, R.bits, table_key(s_local, v));
  if (ins > 0) {
    const uint32_t pos = atomicAdd(&o.gc->tail, 1u);
    if (pos - head < W) {
      const uint32_t sl = pos & (W - 1);
      o.ring[sl] = v;
      o.rr.e0[sl] = e0;
      o.rr.d[sl] = (uint32_t)(e1 - e0);
      o.rr.T[sl] = T;
    } else {
      task_push1(R, ctl, s_local, v);
      o.gc->pushed = 1u;
    }
  } else if (ins < 0) {
    atomicOr(&o.gc->flag, FLAG_TABLE);
  }
}

// Row cursor over the merged quad space of o's staged batch: merged index j
// lies in row r (qend[r] - nq[r] <= j < qend[r]); the row's Philox quad is
// (qhi, qlo) and its IC threshold T.
struct Cur {
  uint32_t j, qe, qlo, qhi, T;
  int r;
};

template <int G>
__device__ __forceinline__ void cur_row(const GroupRows<G>& rw, int r, uint32_t j, Cur& c) {
  c.r = r;
  c.j = j;
  c.qe = rw.qend[r];
  const unsigned long long q = rw.q0[r] + (j - (c.qe - rw.nq[r]));
  c.qlo = (uint32_t)q;
  c.qhi = (uint32_t)(q >> 32);
  c.T = rw.T[r];
}

// first row with qend > j (rows with no quads have qend equal to their predecessor's)
template <int G>
__device__ __forceinline__ void cur_seek(const GroupRows<G>& rw, uint32_t nrows, uint32_t j, Cur& c) {
  int lo = 0, hi = (int)nrows - 1;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (rw.qend[mid] > j) hi = mid;
    else lo = mid + 1;
  }
  cur_row<G>(rw, lo, j, c);
}

template <int G>
__device__ __forceinline__ void cur_step(const GroupRows<G>& rw, Cur& c) {
  ++c.j;
  if (++c.qlo == 0u) ++c.qhi;
  if (c.j == c.qe) {  // past the row: the next row with quads (only called while j < total)
    int r = c.r + 1;
    while (rw.qend[r] <= c.j) ++r;
    cur_row<G>(rw, r, c.j, c);
  }
}

template <bool HOIST>
__device__ __forceinline__ uint4 edge_draws(const Cur& c, const EdgeConsts& E, uint32_t c2, uint32_t c3,
                                            const PhiloxKey& K) {
  return HOIST ? philox_edge(c.qlo, E, K) : philox(c.qlo, c.qhi, c2, c3, K);
}

__device__ __forceinline__ uint32_t min4(const uint4& w) { return min(min(w.x, w.y), min(w.z, w.w)); }

// Rare branch: some word of the quad at c is <= T.  Word i is edge
// e = 4q + i; it belongs to c's row unless the quad is the row's first
// (i < wlo) or last (i > whi) and straddles a neighbour row.  A live edge is
// parked in o's live list (visited directly when the list is full).
template <int G, class GV>
__device__ __forceinline__ void park_live(const GV& g, const RoundView& R, SampleCtl* ctl, const SG<G>& o,
                                       const Cur& c, uint4 w, uint32_t s_local, uint32_t head, uint32_t W) {
  const GroupRows<G>& rw = *o.rw;
  const unsigned long long q = ((unsigned long long)c.qhi << 32) | c.qlo;
  uint32_t live = quad_live_mask(g, q, c.T, w);
  if (c.j == c.qe - rw.nq[c.r]) live &= 0xFu << rw.wlo[c.r];
  if (c.j == c.qe - 1u) live &= 0xFu >> (3u - rw.whi[c.r]);
  while (live) {
    const int i = __ffs(live) - 1;
    live &= live - 1;
    const unsigned long long e = (q << 2) + i;
    const uint32_t p = atomicAdd(&o.gc->nlive, 1u);
    if (p < LIVE_CAP) {
      o.live_e[p] = e;
      if (R.prefetch) g_prefetch_nbr(g, e);  // the visit phase reads nbr[e]: start it on its way to L2 now
    }
    else visit_for<G>(g, R, ctl, o, s_local, head, W, g_nbr(g, e));
  }
}

// NT threads (thread t) sweep quads [lo, hi) of o's staged batch (nrows
// rows; sample counter words c2, c3): thread t takes one contiguous run and
// walks it as U interleaved sub-runs (U independent Philox chains in flight).
// An edge into the row's vertex is live iff its draw <= T (R2); the common
// case is one 4-way min and one compare per quad.  HOIST: every quad of the
// batch has qhi = 0, so the sample-constant Philox work is hoisted
// (philox_edge: 18 instead of 20 wide multiplies per quad).
#ifndef EIM_SWEEP_U
#define EIM_SWEEP_U 2
#endif
template <int G, int NT, bool HOIST, int U, class GV>
__device__ __forceinline__ void sweep_runs(const GV& g, const RoundView& R, SampleCtl* ctl, const SG<G>& o,
                                           uint32_t nrows, uint32_t lo, uint32_t hi, int t, uint32_t c2, uint32_t c3,
                                           const EdgeConsts& E, uint32_t s_local, uint32_t head, uint32_t W) {
  const GroupRows<G>& rw = *o.rw;
  const uint32_t per = (hi - lo + NT - 1) / NT;
  const uint32_t a0 = lo + (uint32_t)t * per;
  if (per == 0 || a0 >= hi) return;
  const uint32_t a1 = min(a0 + per, hi);
  const uint32_t sub = (a1 - a0 + U - 1) / U;
  Cur c[U];
  uint32_t n[U];
#pragma unroll
  for (int k = 0; k < U; ++k) {
    const uint32_t st = a0 + (uint32_t)k * sub;
    n[k] = st < a1 ? min(sub, a1 - st) : 0u;
    if (k == 0 || n[k]) cur_seek<G>(rw, nrows, st, c[k]);
    else c[k] = c[0];
  }
  for (uint32_t i = 0;;) {
    uint4 w[U];
#pragma unroll
    for (int k = 0; k < U; ++k) w[k] = edge_draws<HOIST>(c[k], E, c2, c3, R.K);
#pragma unroll
    for (int k = 0; k < U; ++k)
      if ((k == 0 || i < n[k]) && quad_any_live(g, ((unsigned long long)c[k].qhi << 32) | c[k].qlo, c[k].T, w[k]))
        park_live<G>(g, R, ctl, o, c[k], w[k], s_local, head, W);
    if (++i >= sub) break;
#pragma unroll
    for (int k = 0; k < U; ++k)
      if (k == 0 || i < n[k]) cur_step<G>(rw, c[k]);
  }
}

template <int G, int NT, class GV>
__device__ __forceinline__ void sweep_any(const GV& g, const RoundView& R, SampleCtl* ctl, const SG<G>& o,
                                          uint32_t nrows, uint32_t lo, uint32_t hi, int t, uint64_t s,
                                          uint32_t s_local, uint32_t head, uint32_t W, bool hoist) {
  const uint32_t c2 = (uint32_t)s, c3 = ctr_hi(s, TAG_EDGE);
  const EdgeConsts E = edge_consts(0u, c2, c3, R.K);
  if (hoist) sweep_runs<G, NT, true, EIM_SWEEP_U>(g, R, ctl, o, nrows, lo, hi, t, c2, c3, E, s_local, head, W);
  else sweep_runs<G, NT, false, 1>(g, R, ctl, o, nrows, lo, hi, t, c2, c3, E, s_local, head, W);
}

// A warp claims and sweeps chunks of o's current job until none is left.
// Returns true if it swept anything.
template <int G, class GV>
__device__ __forceinline__ bool work_job(const GV& g, const RoundView& R, SampleCtl* ctl, const SG<G>& o,
                                         int lane, uint32_t W) {
  Job& j = o.gc->job;
  bool any = false;
  for (;;) {
    unsigned long long old = 0;
    if (lane == 0) {
      old = *(volatile unsigned long long*)&j.claim;
      if ((old & 0xFFFFFFull) < ((old >> 24) & 0xFFFFFFull)) old = atomicAdd(&j.claim, 1ull);
    }
    old = __shfl_sync(FULL, old, 0);
    const uint32_t c = (uint32_t)(old & 0xFFFFFFull), n = (uint32_t)((old >> 24) & 0xFFFFFFull);
    if (c >= n) return any;
    // the job's fields are stable until this chunk is counted done
    const uint32_t ch = *(volatile uint32_t*)&j.ch, total = *(volatile uint32_t*)&j.total;
    const uint32_t nrows = *(volatile uint32_t*)&j.nrows, s_local = *(volatile uint32_t*)&j.s_local;
    const uint32_t head = *(volatile uint32_t*)&j.head, hoist = *(volatile uint32_t*)&j.hoist;
    const uint64_t s = R.base + s_local;
    const uint32_t lo = c * ch, hi = min(lo + ch, total);
    sweep_any<G, 32>(g, R, ctl, o, nrows, lo, hi, lane, s, s_local, head, W, hoist != 0u);
    __syncwarp();
    __threadfence_block();  // parks and ring writes before the chunk counts as done
    if (lane == 0) atomicAdd(&j.done, 1u);
    any = true;
  }
}

// Warp-level: join the open jobs of the other sub-groups of the block.
template <int G, int NSG, class GV>
__device__ __forceinline__ bool help_others(const GV& g, const RoundView& R, SampleCtl* ctl,
                                            unsigned char* smem, int gi, int lane, uint32_t W) {
  bool any = false;
  if (NSG < 2) return false;
#pragma unroll 1
  for (int k = 1; k < NSG; ++k) {
    const int o = (gi + k) % NSG;
    const SG<G> so = sg_at<G>(smem, o, W);
    if (!*(volatile uint32_t*)&so.gc->job.open) continue;
    any |= work_job<G>(g, R, ctl, so, lane, W);
  }
  return any;
}

// Stage one row (in-edges [e0, e1), threshold T) into slot gtid of rw;
// returns its quad count.
template <int G>
__device__ __forceinline__ uint32_t stage_row(GroupRows<G>& rw, int gtid, unsigned long long e0,
                                              unsigned long long e1, uint32_t T) {
  uint32_t nq = 0;
  if (e1 > e0) {
    nq = (uint32_t)(((e1 - 1) >> 2) - (e0 >> 2) + 1);
    rw.q0[gtid] = e0 >> 2;
    rw.wlo[gtid] = (uint8_t)(e0 & 3);
    rw.whi[gtid] = (uint8_t)((e1 - 1) & 3);
    rw.T[gtid] = T;
  }
  rw.nq[gtid] = nq;
  return nq;
}

// One traversal of sample s_local (Alg. 2 l.5-20) by sub-group gi in shared
// memory: from the root, or from the nseed vertices of a task at pool[poff..]
// (already members).  The ring is the frontier backlog of capacity W (a
// power of two) with prefetched rows.  A batch: (1) stage up to G queued
// rows and scan their Philox-quad counts; (2) sweep the quads as a job whose
// chunks the sub-group's warps -- and, for a heavy batch, the idle warps of
// the block's other sub-groups -- claim; (3) visit the parked live neighbours
// in parallel (one table insert each; a new member joins the ring with its
// row).  Between batches the sub-group helps the open jobs of its block.
// After every spill_quads swept quads the backlog is cut into pieces of
// about task_quads quads (heavy samples are chains of hub rows: few
// vertices, many quads); one piece stays, the others become tasks that any
// sub-group of the launch runs the same way.  Membership lives in the round
// table (first insert wins, the winner expands the vertex), so the union of
// the traversals is the unique reachable set of the sampled world, whatever
// the split.  Returns 0, FLAG_TABLE or FLAG_CANCEL; found = new members
// inserted by this traversal.
template <int G, int NSG, class GV>
__device__ __forceinline__ uint32_t traverse(const GV& g, const RoundView& R, SampleCtl* ctl,
                                             unsigned char* smem, int gi, uint32_t s_local, bool root,
                                             unsigned long long poff, uint32_t nseed, uint32_t W, int gtid,
                                             uint32_t& found, uint32_t spill_quads, uint32_t task_quads,
                                             uint32_t help_min, uint32_t probe_quads, bool& split_any) {
  const SG<G> me = sg_at<G>(smem, gi, W);
  GroupCtl& gc = *me.gc;
  GroupRows<G>& rw = *me.rw;
  const int lane = gtid & 31;
  const uint64_t s = R.base + s_local;
  uint32_t head = 0, extra = 0;  // extra: members found here that left the ring (split off / overflow)
  uint32_t swept = 0;
  unsigned long long nbatch = 0, nquads = 0, t0 = (R.dbg && root && gtid == 0) ? gtimer() : 0ull;
  unsigned long long ph[3] = {0, 0, 0}, tp = 0, nlive_tot = 0;  // ns in stage+scan, sweep, visit
  auto dbg_end = [&]() {
    if (R.dbg && root && gtid == 0) {
      unsigned long long* d = R.dbg + 8ull * s_local;
      d[0] = nbatch;
      d[1] = nquads;
      d[2] = t0;
      d[3] = gtimer();
      d[4] = ph[0];
      d[5] = ph[1];
      d[6] = ph[2];
      d[7] = nlive_tot;
    }
  };
  auto mark = [&](int i) {
    if (R.dbg && gtid == 0) {
      const unsigned long long t = gtimer();
      if (i >= 0) ph[i] += t - tp;
      tp = t;
    }
  };
  if (gtid == 0) {
    gc.flag = 0;
    gc.hiq = R.nohoist;
    gc.nlive = 0;
    gc.pushed = 0;
    gc.tail = nseed;
  }
  if (root) {
    gsync<G>(gi);
    if (gtid == 0) visit_for<G>(g, R, ctl, me, s_local, 0, W, draw_root(s, g.n, R.K));
  } else {
    // pool lines may be cached from a neighbouring task: read through L2
    for (uint32_t t = gtid; t < nseed; t += G) {
      const uint32_t v = __ldcg(R.pool + poff + t);
      const unsigned long long e0 = g_off(g, v), e1 = g_off(g, v + 1);
      me.ring[t] = v;
      me.rr.e0[t] = e0;
      me.rr.d[t] = (uint32_t)(e1 - e0);
      me.rr.T[t] = g_thr(g, v, e1 - e0);
    }
  }
  gsync<G>(gi);
  for (;;) {
    uint32_t tail = *(volatile uint32_t*)&gc.tail;
    const uint32_t flag = *(volatile uint32_t*)&gc.flag;
    if (flag) {
      found = tail + extra - nseed;
      split_any = gc.pushed || extra;
      return flag;
    }
    if (tail - head > W) {  // positions past head + W went out as one-vertex tasks
      extra += tail - head - W;
      tail = head + W;
    }
    uint32_t npieces = 1;
    // probe-first rounds: a root traversal that has swept probe_quads quads
    // is suspended -- its whole backlog leaves as tasks, run after every id
    // of the round has been probed -- so the heavy samples of a round all
    // continue from the start of the round's tail phase instead of starting
    // whenever their id comes up (longest-processing-time order without
    // knowing the sizes in advance)
    const bool suspend = root && probe_quads && swept >= probe_quads && tail > head;
    if (suspend || (spill_quads && swept >= spill_quads && tail - head >= 2)) {
      // quads of the backlog (rows are in rr) -> number of pieces
      const uint32_t B = tail - head;
      uint32_t q = 0;
      for (uint32_t i = gtid; i < B; i += G) q += (me.rr.d[(head + i) & (W - 1)] + 3u) >> 2;
      for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(FULL, q, o);
      gsync<G>(gi);  // every thread has read gc.tail; wsum is free
      if (lane == 0) gc.wsum[gtid >> 5] = q;
      gsync<G>(gi);
      uint32_t qb = 0;
#pragma unroll
      for (int i = 0; i < G / 32; ++i) qb += gc.wsum[i];
      npieces = min(B, qb / max(task_quads, 1u));
      if (suspend) npieces = max(npieces, 1u);
      else if (npieces < 2) swept = spill_quads / 2;  // look again after a few batches
    }
    if (suspend || npieces >= 2) {
      // ---- split: keep the first piece of tv vertices (none when suspended),
      // push the rest as tasks of <= tv
      const uint32_t B = tail - head;
      const uint32_t tv = (B + npieces - 1) / npieces;
      const uint32_t keep = suspend ? 0u : tv;
      const uint32_t npush = B - keep;
      const uint32_t ntasks = (npush + tv - 1) / tv;
      gsync<G>(gi);  // every thread has read wsum
      if (gtid == 0) {
        atomicAdd(&ctl->outstanding, (unsigned long long)ntasks);
        gc.base = atomicAdd(&ctl->ptail, (unsigned long long)npush);
        gc.h = atomicAdd(&R.qc[16 * home_queue() + 1], (unsigned long long)ntasks);  // index in the block's queue
        atomicAdd(&ctl->ttail, (unsigned long long)ntasks);
        atomicAdd(&ctl->tasks_pushed, (unsigned long long)ntasks);
      }
      gsync<G>(gi);
      const unsigned long long po = gc.base, qi = gc.h, tq = R.tcap / TQ, ti = home_queue() * tq + qi;
      const bool ok = po + npush <= R.pcap;
      if (ok)
        for (uint32_t i = gtid; i < npush; i += G) R.pool[po + i] = me.ring[(head + keep + i) & (W - 1)];
      __threadfence();
      gsync<G>(gi);
      for (uint32_t t = gtid; t < ntasks; t += G) {
        if (qi + t >= tq) continue;
        const uint32_t nv = min(tv, npush - t * tv);
        task_write(R, ti + t, po + (unsigned long long)t * tv, s_local, ok ? nv : 0u);
      }
      if (gtid == 0) {
        if (!ok || qi + ntasks > tq) {
          mark_fail(ctl);
          const unsigned long long lost = qi + ntasks > tq ? qi + ntasks - max(qi, tq) : 0;
          if (lost) atomicAdd(&ctl->outstanding, 0ull - lost);
        }
        gc.tail = head + keep;
      }
      extra += npush;
      tail = head + keep;
      swept = 0;
      gsync<G>(gi);
    } else if (tail != *(volatile uint32_t*)&gc.tail) {
      gsync<G>(gi);
      if (gtid == 0) gc.tail = tail;
      gsync<G>(gi);
    }
    if (head >= tail) {
      found = tail + extra - nseed;
      split_any = extra != 0;
      dbg_end();
      return 0;
    }
    if (*(volatile const unsigned int*)R.cancel) {
      gsync<G>(gi);  // every thread has read the control words above
      found = 0;
      return FLAG_CANCEL;
    }
    // ---- help the heavy batches of the other sub-groups, then stage
    if (NSG > 1) {
      help_others<G, NSG>(g, R, ctl, smem, gi, lane, W);
      gsync<G>(gi);
    }
    mark(-1);
    const uint32_t nb = min((uint32_t)G, tail - head);
    uint32_t nq = 0;
    if (gtid < nb) {
      const uint32_t sl = (head + gtid) & (W - 1);
      const unsigned long long e0 = me.rr.e0[sl];
      nq = stage_row<G>(rw, gtid, e0, e0 + me.rr.d[sl], me.rr.T[sl]);
      if (nq && ((e0 + me.rr.d[sl] - 1) >> 34)) gc.hiq = 1u;  // sticky for the traversal
    }
    if (gtid == 0) gc.nlive = 0;
    uint32_t total;
    const uint32_t incl = group_incl_scan<G>(nq, gtid, gi, gc, total);
    if (gtid < nb) rw.qend[gtid] = incl;
    const bool hoist = *(volatile uint32_t*)&gc.hiq == 0u;  // written before the scan's barrier
    head += nb;  // ring slots [old head, head) are free again: their rows are staged
    // ---- heavy batch: post it as a job the block's warps claim in chunks
    const bool heavy = NSG > 1 && total >= help_min;
    const uint32_t ch = 256u;
    const uint32_t nchunks = heavy ? (total + ch - 1) / ch : 0u;
    if (heavy && gtid == 0) {
      Job& j = gc.job;
      j.total = total;
      j.nrows = nb;
      j.s_local = s_local;
      j.head = head;
      j.ch = ch;
      j.hoist = hoist ? 1u : 0u;
      j.done = 0;
      gc.epoch = (gc.epoch + 1) & 0xFFFFu;
      __threadfence_block();
      atomicExch(&j.claim, ((unsigned long long)gc.epoch << 48) | ((unsigned long long)nchunks << 24));
      __threadfence_block();
      j.open = 1u;
    }
    gsync<G>(gi);
    mark(0);
    // ---- sweep
    if (heavy) {
      work_job<G>(g, R, ctl, me, lane, W);
      if (gtid == 0) {
        gc.job.open = 0;
        while (*(volatile uint32_t*)&gc.job.done < nchunks) __nanosleep(20);
        __threadfence_block();
      }
    } else {
      sweep_any<G, G>(g, R, ctl, me, nb, 0, total, gtid, s, s_local, head, W, hoist);
    }
    gsync<G>(gi);
    mark(1);
    // ---- visit the parked live neighbours, one per thread
    const uint32_t nl = min(*(volatile uint32_t*)&gc.nlive, LIVE_CAP);
    for (uint32_t t = gtid; t < nl; t += G) visit_for<G>(g, R, ctl, me, s_local, head, W, g_nbr(g, me.live_e[t]));
    swept += total;
    nbatch++;
    nquads += total;
    nlive_tot += nl;
    gsync<G>(gi);
    mark(2);
  }
}

// Thread 0 of a sub-group: what to do next.  Tasks first (they belong to
// the heavy samples that bound the round), then a new sample id; idle while
// work is outstanding elsewhere (a running traversal may still split); exit
// when every id is taken and nothing is outstanding.
__device__ __forceinline__ bool take_id(const RoundView& R, SampleCtl* ctl, uint64_t count, uint32_t& s_local) {
  if (vload(&ctl->ticket) < count) {
    atomicAdd(&ctl->outstanding, 1ull);  // before the ticket: an observer never sees "all taken, none outstanding" early
    const unsigned long long t = atomicAdd(&ctl->ticket, 1ull);
    if (t == 0) ctl->t_first = gtimer();
    if (t == count - 1) ctl->t_last_id = gtimer();
    if (t < count) {
      s_local = R.list[t];
      return true;
    }
    atomicAdd(&ctl->outstanding, ~0ull);
  }
  return false;
}

__device__ __forceinline__ bool take_id(const RoundView& R, SampleCtl* ctl, uint64_t count, GroupCtl& gc) {
  uint32_t s_local;
  if (!take_id(R, ctl, count, s_local)) return false;
  gc.s_local = s_local;
  gc.nb = 0;
  return true;
}

// probe_first: new ids before tasks (the tasks are the suspended heavy
// samples, which then all continue together once every id is taken)
__device__ __forceinline__ uint32_t decide(const RoundView& R, SampleCtl* ctl, uint64_t count, GroupCtl& gc,
                                           bool probe_first) {
  const volatile unsigned int* cp = R.cancel;
  if (cp[0] || cp[1]) return ACT_EXIT;  // cancelled or paused
  if (probe_first && take_id(R, ctl, count, gc)) return ACT_LOCAL;
  const unsigned long long tq = R.tcap / TQ;
  const uint32_t home = home_queue();
  // hint (pushed vs claimed, all queues): scan the queues only when some
  // task may be waiting; a task missed here is seen by the next call (a
  // group exits only when nothing is outstanding)
  const bool any_task = vload(&ctl->ttail) > vload(&ctl->thead);
  for (uint32_t k = 0; any_task && k < TQ; ++k) {
    const uint32_t q = (home + k) % TQ;
    unsigned long long* head = &R.qc[16 * q];
    unsigned long long h = vload(head);
    for (;;) {
      const unsigned long long t = min(vload(head + 1), tq);
      if (h >= t) break;
      const unsigned long long old = atomicCAS(head, h, h + 1);
      if (old != h) {
        h = old;
        continue;
      }
      atomicAdd(&ctl->thead, 1ull);
      unsigned long long* d = R.tasks + 2 * (q * tq + h);
      unsigned long long w1;
      while ((w1 = vload(d + 1)) == 0ull) __nanosleep(32);  // claimed before it was written
      __threadfence();
      gc.base = vload(d);
      d[0] = 0ull;
      d[1] = 0ull;  // consumed: the descriptors are all-zero again when the round ends
      gc.s_local = (uint32_t)(w1 >> 32) - 1u;
      gc.nb = (uint32_t)w1;
      return ACT_TASK;
    }
  }
  if (!probe_first && take_id(R, ctl, count, gc)) return ACT_LOCAL;
  if (vload(&ctl->arena_fail)) return ACT_EXIT;  // the host redoes the round
  if (vload(&ctl->outstanding) == 0ull) {
    atomicMax(&ctl->t_end, gtimer());
    return ACT_EXIT;
  }
  return ACT_IDLE;
}

// The IC sampler of one round: persistent blocks of NSG sub-groups over
// sample ids [0, count) and the tasks split off heavy samples.
#ifndef EIM_IDLE_MAX_NS
#define EIM_IDLE_MAX_NS 2048  // longest back-off of an idle group between polls of the round's control words
#endif
#ifndef EIM_IC_THREADS_SM
#define EIM_IC_THREADS_SM 1280  // resident sampler threads per SM the register budget is cut for
#endif
template <int G, int NSG>
constexpr int ic_min_blocks() {
  return EIM_IC_THREADS_SM / (G * NSG) > 0 ? EIM_IC_THREADS_SM / (G * NSG) : 1;
}

template <int G, int NSG, class GV>
__global__ void __launch_bounds__(G* NSG, ic_min_blocks<G, NSG>()) ic_kernel(GV g, RoundView R, uint64_t count, uint32_t W,
                                                      SampleCtl* ctl, uint32_t spill_quads, uint32_t task_quads,
                                                      uint32_t help_min, uint32_t probe_quads) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int gi = threadIdx.x / G, gtid = threadIdx.x % G, lane = threadIdx.x & 31;
  const SG<G> me = sg_at<G>(smem_raw, gi, W);
  GroupCtl& gc = *me.gc;
  count = vload(&ctl->ntickets);  // the ids the root pre-pass left for a traversal
  if (gtid == 0) {
    gc.job.claim = 0;
    gc.job.open = 0;
    gc.job.done = 0;
    gc.epoch = 0;
  }
  __syncthreads();  // every sub-group's job is initialised before anyone helps
  uint32_t backoff = 256;
  for (;;) {
    if (gtid == 0) gc.action = decide(R, ctl, count, gc, probe_quads != 0u);
    gsync<G>(gi);
    const uint32_t act = gc.action;
    if (act == ACT_EXIT) break;
    if (act == ACT_IDLE && NSG == 1) {
      if (gtid == 0) __nanosleep(backoff);
      backoff = min(backoff * 2u, (uint32_t)EIM_IDLE_MAX_NS);
    } else if (act == ACT_IDLE) {
      // poll the block's jobs (shared memory) for ~backoff ns before the
      // next global poll
      bool helped = false;
      const unsigned long long t_end = __shfl_sync(FULL, gtimer(), 0) + backoff;
      do {
        helped |= help_others<G, NSG>(g, R, ctl, smem_raw, gi, lane, W);
        __nanosleep(64);
      } while (__shfl_sync(FULL, gtimer(), 0) < t_end);  // warp-uniform exit
      backoff = helped ? 256u : min(backoff * 2u, 4096u);
    } else {
      backoff = 256;
      const uint32_t s_local = gc.s_local, nseed = gc.nb;
      const unsigned long long poff = gc.base;
      uint32_t found = 0;
      bool split_any = false;
      const uint32_t flag = traverse<G, NSG>(g, R, ctl, smem_raw, gi, s_local, act == ACT_LOCAL, poff, nseed, W,
                                                   gtid, found, spill_quads, task_quads, help_min, probe_quads,
                                                   split_any);
      if (gtid == 0) {
        if (found) atomicAdd(&R.sizes[s_local], found);
        if (split_any && act == ACT_LOCAL) atomicAdd(&ctl->spilled, 1ull);
        if (flag & FLAG_TABLE) mark_fail(ctl);
        __threadfence();  // tasks pushed above are counted before this unit leaves `outstanding`
        atomicAdd(&ctl->outstanding, ~0ull);  // -1
      }
    }
    gsync<G>(gi);
  }
}

template <int G, int NSG>
size_t ic_smem(uint32_t W) {
  return NSG * sg_bytes<G>(W);
}

// Root pre-pass of an IC launch (Alg. 2 l.6): a thread per sample id draws
// the root; a root without in-edges is the whole set (Alg. 2 l.10-20 examine
// nothing), so its membership is recorded here, and every other id is
// listed for ic_kernel's tickets.  On R-MAT most roots have no in-edges
// (C2: 55 %): their samples no longer cost a group's decide/traverse round
// trips and barriers.
template <class GV>
__global__ void ic_prepass_kernel(GV g, RoundView R, uint64_t count, SampleCtl* ctl, uint32_t* list, bool all) {
  const int lane = threadIdx.x & 31;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i0 = (uint64_t)blockIdx.x * blockDim.x; i0 < count; i0 += stride) {
    const uint64_t i = i0 + threadIdx.x;
    bool trav = false;
    if (i < count) {
      const uint32_t root = all ? 0u : draw_root(R.base + i, g.n, R.K);
      if (!all && g_off(g, (uint64_t)root + 1) == g_off(g, root)) {
        if (table_insert(R.keys, R.bits, table_key((uint32_t)i, root)) < 0) mark_fail(ctl);
        R.sizes[i] = 1;
      } else {
        trav = true;
      }
    }
    // warp-aggregated append to the ticket list
    const unsigned m = __ballot_sync(FULL, trav);
    unsigned long long base = 0;
    if (lane == 0 && m) base = atomicAdd(&ctl->ntickets, (unsigned long long)__popc(m));
    base = __shfl_sync(FULL, base, 0);
    if (trav) list[base + __popc(m & ((1u << lane) - 1u))] = (uint32_t)i;
  }
}

// ---------------------------------------------------------------- LT
// Reverse LT walk (R3-R5): at u with d^-(u) > 0, tau_u is the
// LT-tagged draw of u and the chosen in-neighbour is position
// floor(tau * d / 2^32) of u's row (the prefix-scan choice under WC
// weights); the walk stops when d^-(u) = 0 or the chosen vertex is already in
// the set.  One thread per walk; visited set = the round table.
template <class GV>
__global__ void __launch_bounds__(256) lt_kernel(GV g, RoundView R, uint64_t count, SampleCtl* ctl) {
  const PhiloxKey& K = R.K;
  unsigned long long edges_acc = 0;
  for (;;) {
    const volatile unsigned int* cp = R.cancel;
    if (cp[0] || cp[1]) break;  // cancelled or paused
    const unsigned long long t = atomicAdd(&ctl->ticket, 1ull);
    if (t >= count) break;
    const uint32_t s_local = (uint32_t)t;
    const uint64_t s = R.base + s_local;
    uint32_t u = draw_root(s, g.n, K);
    // A step's critical path is off[u] -> nbr[e0 + j] -> the membership
    // insert of v.  The insert only decides whether the walk stops, so v's
    // row and threshold are loaded and drawn before its result is awaited:
    // two dependent memory round trips per step instead of three.
    unsigned long long e0 = g_off(g, u), e1 = g_off(g, u + 1);
    uint32_t tau = word_of(philox_at((uint64_t)(u >> 2), s, TAG_LT, K), u & 3u);
    bool ok = table_insert(R.keys, R.bits, table_key(s_local, u)) >= 0;
    uint32_t L = 1;
    unsigned long long steps = 0;
    while (ok) {
      if (e1 == e0) break;
      ++steps;
      const unsigned long long j = lt_choose(g, e0, e1, tau);
      if (j == ~0ull) break;  // general weights: no in-neighbour activated (R25)
      const uint32_t v = g_nbr(g, e0 + j);
      const unsigned long long f0 = g_off(g, v), f1 = g_off(g, v + 1);
      const uint32_t tv = word_of(philox_at((uint64_t)(v >> 2), s, TAG_LT, K), v & 3u);
      const int ins = table_insert(R.keys, R.bits, table_key(s_local, v));
      if (ins == 0) break;
      if (ins < 0) ok = false;
      ++L;
      u = v;
      e0 = f0;
      e1 = f1;
      tau = tv;
    }
    if (ok) {
      R.sizes[s_local] = L;
      R.edges[s_local] = steps;
      edges_acc += steps;
    } else {
      atomicOr(reinterpret_cast<unsigned int*>(&ctl->arena_fail), 1u);
    }
  }
  if (edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

// LT walk store of the plain graph: aug[e] = (v, d^-(v), lo32 off[v],
// hi32 off[v]) for v = in_nbr[e].  One 16-byte load per walk step then gives
// the chosen in-neighbour AND its row, so a step is one dependent memory
// round trip (the row-offset load of v disappears from the critical path).
// 16 B per in-edge (C3: 1.9 GB), built once per graph on the first LT run.
__global__ void lt_aug_build_kernel(GraphView g, uint4* __restrict__ aug) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < g.m; e += stride) {
    const uint32_t v = __ldg(g.nbr + e);
    const uint64_t o0 = __ldg(g.off + v), o1 = __ldg(g.off + v + 1);
    aug[e] = make_uint4(v, (uint32_t)(o1 - o0), (uint32_t)o0, (uint32_t)(o0 >> 32));
  }
}

// A key of no sample (its sample field decodes to 0xFFFFFFFE, above every
// round's count, so the scatter skips it): written over a speculative insert
// that the walk turned out not to reach.
constexpr unsigned long long TABLE_TOMB = 0xFFFFFFFF00000000ull;

// Second half of table_insert, for a first CAS issued earlier at slot i
// whose result is cur: 1 = inserted (*slot = its slot), 0 = present, -1 =
// table too full (same probe budget as table_insert).
__device__ __forceinline__ int table_resolve(unsigned long long* keys, uint32_t bits, unsigned long long key,
                                             uint32_t i, unsigned long long cur, uint32_t* slot) {
  const uint32_t mask = (uint32_t)((1ull << bits) - 1ull);
  for (uint32_t p = 1;; ++p) {
    if (cur == 0ull) {
      *slot = i;
      return 1;
    }
    if (cur == key) return 0;
    if (p == MAX_PROBE) return -1;
    i = (i + 1u) & mask;
    cur = atomicCAS(&keys[i], 0ull, key);
  }
}

// lt_kernel on the walk store (same walk, same draws, same outputs).  The
// walk runs one step ahead of its stop test: the membership insert of the
// next vertex and the load of the entry after it are issued before the
// insert of the current vertex is resolved, so a step costs one memory round
// trip.  When the current vertex turns out to be a revisit (the walk stops,
// P:136), the speculative insert is overwritten with TABLE_TOMB.
__device__ __forceinline__ uint4 aug_load(const uint4* p, unsigned long long pol) {
  if (pol == 0ull) return __ldg(p);
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p), "l"(pol));
  return r;
}

__global__ void __launch_bounds__(256) lt_aug_kernel(GraphView g, const uint4* __restrict__ aug, RoundView R,
                                                     uint64_t count, SampleCtl* ctl) {
  const PhiloxKey& K = R.K;
  unsigned long long pol = 0ull;  // L2 policy of the walk-store loads (0: default)
  if (R.lt_evict) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  unsigned long long edges_acc = 0;
  for (;;) {
    const volatile unsigned int* cp = R.cancel;
    if (cp[0] || cp[1]) break;  // cancelled or paused
    const unsigned long long t = atomicAdd(&ctl->ticket, 1ull);
    if (t >= count) break;
    const uint32_t s_local = (uint32_t)t;
    const uint64_t s = R.base + s_local;
    const uint32_t u = draw_root(s, g.n, K);
    const uint64_t e0 = __ldg(g.off + u);
    const uint32_t d = (uint32_t)(__ldg(g.off + u + 1) - e0);
    const uint32_t tau = word_of(philox_at((uint64_t)(u >> 2), s, TAG_LT, K), u & 3u);
    bool ok = table_insert(R.keys, R.bits, table_key(s_local, u)) >= 0;
    uint32_t L = 1;
    unsigned long long steps = 0;
    if (ok && d) {
      // the step from the root: entry a -> vertex v (insert pending), nx = the entry chosen from v
      const uint4 a = aug_load(aug + e0 + __umul64hi((unsigned long long)tau << 32, d), pol);
      steps = 1;
      uint32_t v = a.x;
      unsigned long long key = table_key(s_local, v);
      uint32_t slot = table_hash(key, R.bits);
      unsigned long long cur = atomicCAS(&R.keys[slot], 0ull, key);
      bool nxt = a.y != 0u;
      uint4 nx = a;
      if (nxt) {
        const uint32_t tv = word_of(philox_at((uint64_t)(v >> 2), s, TAG_LT, K), v & 3u);
        nx = aug_load(aug + ((uint64_t)a.z | ((uint64_t)a.w << 32)) + __umul64hi((unsigned long long)tv << 32, a.y), pol);
      }
      for (;;) {
        // speculate the step from v: v2 = nx.x, its insert and the entry chosen from v2
        uint32_t v2 = 0, slot2 = 0;
        unsigned long long key2 = 0, cur2 = 0;
        bool nxt2 = false;
        uint4 nx2 = nx;
        if (nxt) {
          v2 = nx.x;
          key2 = table_key(s_local, v2);
          slot2 = table_hash(key2, R.bits);
          cur2 = atomicCAS(&R.keys[slot2], 0ull, key2);
          nxt2 = nx.y != 0u;
          if (nxt2) {
            const uint32_t tv2 = word_of(philox_at((uint64_t)(v2 >> 2), s, TAG_LT, K), v2 & 3u);
            nx2 = aug_load(aug + ((uint64_t)nx.z | ((uint64_t)nx.w << 32)) + __umul64hi((unsigned long long)tv2 << 32, nx.y),
                           pol);
          }
        }
        // resolve v's insert
        uint32_t got = 0;
        const int ins = table_resolve(R.keys, R.bits, key, slot, cur, &got);
        if (ins <= 0) {
          if (ins < 0) ok = false;
          // v was a revisit (or the table is full): undo v2's insert if it landed
          if (nxt) {
            uint32_t got2 = 0;
            if (table_resolve(R.keys, R.bits, key2, slot2, cur2, &got2) > 0) R.keys[got2] = TABLE_TOMB;
          }
          break;
        }
        ++L;
        if (!nxt) break;  // d^-(v) = 0
        ++steps;          // the step from v is real
        v = v2;
        key = key2;
        slot = slot2;
        cur = cur2;
        nxt = nxt2;
        nx = nx2;
      }
    }
    if (ok) {
      R.sizes[s_local] = L;
      R.edges[s_local] = steps;
      edges_acc += steps;
    } else {
      atomicOr(reinterpret_cast<unsigned int*>(&ctl->arena_fail), 1u);
    }
  }
  if (edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

// The walk store is a cache next to the graph store (not counted in
// eim_graph_bytes); if it does not fit in device memory the walks run on the
// plain store (lt_kernel), with the same results.
static const uint4* lt_aug(eim_ctx* ctx, const eim_graph* gc, cudaStream_t st) {
  if (std::getenv("EIM_NO_LT_AUG") || gc->packed || gc->weighted || gc->aug_failed) return nullptr;
  eim_graph* g = const_cast<eim_graph*>(gc);  // lazily built cache of the (immutable) store
  if (!g->d_aug) {
    const uint64_t bytes = std::max<uint64_t>(g->view.m, 1) * sizeof(uint4);
    if (cudaMallocAsync(&g->d_aug, bytes, st) != cudaSuccess) {
      cudaGetLastError();
      g->d_aug = nullptr;
      g->aug_failed = true;
      return nullptr;
    }
    lt_aug_build_kernel<<<grid_for(ctx, g->view.m, 256), 256, 0, st>>>(g->view, static_cast<uint4*>(g->d_aug));
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
    g->aug_bytes = bytes;
  }
  return static_cast<const uint4*>(g->d_aug);
}

// ---------------------------------------------------------------- output
__global__ void add_u64_kernel(unsigned long long* acc, const unsigned long long* x) { *acc += *x; }

__global__ void sizes_to_offsets_kernel(const uint32_t* __restrict__ sizes, uint64_t count,
                                        uint64_t* __restrict__ out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= count; i += stride)
    out[i] = i < count ? (uint64_t)sizes[i] : 0ull;
}

__global__ void place_sets_kernel(const uint64_t* __restrict__ excl, const uint32_t* __restrict__ sizes,
                                  uint64_t count, uint64_t arena_base, uint64_t set_index0,
                                  uint64_t* __restrict__ set_start, uint32_t* __restrict__ set_len) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
    set_start[set_index0 + i] = arena_base + excl[i];
    set_len[set_index0 + i] = sizes[i];
  }
}

// Source-vertex elimination (R22).  roots[i] = root of sample
// first+i (Alg. 2 l.6, the same draw the traversal started from).
__global__ void roots_kernel(uint64_t first, uint64_t count, uint32_t n, PhiloxKey K, uint32_t* __restrict__ roots) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride)
    roots[i] = draw_root(first + i, n, K);
}

// sizes[i] -= 1 (the root leaves the set); keep[i] = set non-empty.
__global__ void drop_root_sizes_kernel(uint32_t* __restrict__ sizes, uint64_t count, uint32_t* __restrict__ keep) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= count; i += stride) {
    if (i == count) {
      if (keep) keep[i] = 0;
      continue;
    }
    const uint32_t z = sizes[i] - 1u;
    sizes[i] = z;
    if (keep) keep[i] = z != 0u;
  }
}

// kidx = exclusive scan of keep.  The need-th kept sample (kidx[i] ==
// need-1, kept) ends the ids taken: *consumed = i + 1.
__global__ void find_consumed_kernel(const uint32_t* __restrict__ kidx, uint64_t count, uint32_t need,
                                     unsigned long long* __restrict__ consumed) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride)
    if (kidx[i] == need - 1u && kidx[i + 1] == need) *consumed = i + 1;
}

// Kept sets, compacted: ksizes[kidx[i]] = sizes[i] for the kept i < consumed.
__global__ void compact_sizes_kernel(const uint32_t* __restrict__ sizes, const uint32_t* __restrict__ kidx,
                                     uint64_t consumed, uint32_t* __restrict__ ksizes) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < consumed; i += stride)
    if (kidx[i + 1] != kidx[i]) ksizes[kidx[i]] = sizes[i];
}

// Every live table entry is a member: arena[start(s) + fill[s]++] = v.
// IC (off != nullptr): the in-edges examined by a set are exactly the
// in-edges of its members (each member is expanded once), summed into *esum.
// With roots (source elimination) the root entry of a sample is not stored
// (its edges still count: the traversal examined them) and, with kidx, the
// set index of sample s is set_index0 + kidx[s] (empty sets dropped).
template <class GV>
__global__ void scatter_kernel(const unsigned long long* __restrict__ keys, uint64_t nslots,
                               const uint64_t* __restrict__ set_start, uint64_t set_index0, uint32_t from,
                               uint32_t use,
                               uint32_t* __restrict__ fill, uint32_t* __restrict__ arena, uint32_t ab,
                               uint32_t* __restrict__ C, GV g, bool ic, unsigned long long* __restrict__ esum,
                               const uint32_t* __restrict__ roots, const uint32_t* __restrict__ kidx,
                               uint32_t* __restrict__ snap0, uint32_t cut0, uint32_t* __restrict__ snap1,
                               uint32_t cut1) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  unsigned long long e = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nslots; i += stride) {
    const unsigned long long k = keys[i];
    if (k == 0ull) continue;
    const uint32_t s_local = (uint32_t)(k >> 32) - 1u;
    if (s_local >= use || s_local < from) continue;  // samples outside the appended range
    const uint32_t v = (uint32_t)k;
    if (ic) e += g_off(g, v + 1) - g_off(g, v);
    if (roots && v == roots[s_local]) continue;
    const uint64_t si = set_index0 + (kidx ? kidx[s_local] : s_local);
    const uint32_t p = atomicAdd(&fill[s_local], 1u);
    arena_put(arena, set_start[si] + p, ab, v);
    if (C) atomicAdd(&C[v], 1u);
    if (snap0 && s_local < cut0) atomicAdd(&snap0[v], 1u);  // round snapshots (AppendCuts)
    if (snap1 && s_local < cut1) atomicAdd(&snap1[v], 1u);
  }
  if (ic) {
    for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(FULL, e, o);
    if ((threadIdx.x & 31) == 0 && e) atomicAdd(esum, e);
  }
}


#ifdef EIM_SWEEP_BENCH
// Development probe (built only with -DEIM_SWEEP_BENCH): one group sweeps a
// staged batch of nrows rows of d in-edges each, `reps` times with different
// sample ids; parks live edges (no visit).  Measures the sweep alone.
template <int G>
__global__ void __launch_bounds__(G, EIM_IC_THREADS_SM / G) sweep_bench_kernel(GraphView g, RoundView R, SampleCtl* ctl, uint32_t nrows,
                                                           uint32_t d, uint32_t reps, unsigned long long* out) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const SG<G> me = sg_at<G>(smem_raw, 0, 32);
  const int gtid = threadIdx.x;
  uint32_t nq = 0;
  if (gtid < (int)nrows) {
    const unsigned long long e0 = (unsigned long long)gtid * d * 3 + 1;  // spaced rows, ragged quads
    nq = stage_row<G>(*me.rw, gtid, e0, e0 + d, 0xFFFFFFFFu / d);
  }
  if (gtid == 0) me.gc->hiq = 0;
  uint32_t total;
  const uint32_t incl = group_incl_scan<G>(nq, gtid, 0, *me.gc, total);
  if (gtid < (int)nrows) me.rw->qend[gtid] = incl;
  unsigned long long t0 = 0, nl = 0;
  for (uint32_t r = 0; r < reps; ++r) {
    if (gtid == 0) me.gc->nlive = 0;
    gsync<G>(0);
    if (r == 1 && gtid == 0) t0 = gtimer();
    sweep_any<G, G>(g, R, ctl, me, nrows, 0, total, gtid, 1000 + r + blockIdx.x * reps, 0, 0, 32, true);
    gsync<G>(0);
    nl += min(me.gc->nlive, LIVE_CAP);
  }
  if (gtid == 0) {
    out[3 * blockIdx.x] = gtimer() - t0;
    out[3 * blockIdx.x + 1] = (unsigned long long)total * (reps - 1);
    out[3 * blockIdx.x + 2] = nl;
  }
}
#endif

constexpr uint32_t IC_W = 1024;  // shared-memory frontier ring per group

}  // namespace

// ------------------------------------------------------------------ host
void arena_reset(eim_ctx* ctx, uint32_t b) {
  ctx->arena_b = b;
  ctx->arena.reserve(sizeof(uint32_t) * (1u << 22), false, ctx->stream);
  if (b < 32) EIM_CUDA(cudaMemsetAsync(ctx->arena.p, 0, ctx->arena.bytes, ctx->stream));
  ctx->ctl.reserve(sizeof(SampleCtl) + 2 * sizeof(unsigned long long), false, ctx->stream);
  EIM_CUDA(cudaMemsetAsync(ctx->ctl.p, 0, sizeof(SampleCtl) + 2 * sizeof(unsigned long long), ctx->stream));
  ctx->est_mean_size = 0;
  ctx->arena_used = 0;
}

uint64_t arena_cursor(eim_ctx* ctx) { return ctx->arena_used; }

void arena_ensure(eim_ctx* ctx, uint64_t elems) {
  const uint32_t b = ctx->arena_b;
  const size_t before = ctx->arena.bytes;
  ctx->arena.reserve(std::max<uint64_t>(arena_words(elems, b), 1) * sizeof(uint32_t), true, ctx->stream);
  // encoded: containers past the last used bit stay zero (writers OR into them)
  if (b < 32 && ctx->arena.bytes > before) {
    const uint64_t used = (ctx->arena_used * b + 31) / 32;
    EIM_CUDA(cudaMemsetAsync(ctx->arena.as<uint32_t>() + used, 0, ctx->arena.bytes - used * sizeof(uint32_t),
                             ctx->stream));
  }
}

void ensure_sets(eim_ctx* ctx, uint64_t num_sets) {
  ctx->set_start.reserve(num_sets * sizeof(uint64_t), true, ctx->stream);
  ctx->set_len.reserve(num_sets * sizeof(uint32_t), true, ctx->stream);
}

void round_release(Round& rd) {
  DevBuf* b[] = {&rd.table, &rd.sizes, &rd.edges, &rd.fill, &rd.excl, &rd.ctl, &rd.queue, &rd.dbg, &rd.list,
                 &rd.roots, &rd.kidx, &rd.ksizes};
  for (DevBuf* x : b) x->release();
  for (cudaEvent_t& e : rd.ev) {
    if (e) cudaEventDestroy(e);
    e = nullptr;
  }
  rd.launched = false;
  rd.qdirty = true;
}

static uint32_t env_u32(const char* name, uint32_t dflt) {
  const char* e = std::getenv(name);
  return (e && *e) ? (uint32_t)std::strtoul(e, nullptr, 10) : dflt;
}

// Spill threshold (quads swept by one group before a sample moves to the
// shared queue) and ring size; EIM_SPILL_QUADS / EIM_RING_W override them
// (tests force the spill paths with tiny values; 0 = spill only on overflow).
static uint32_t spill_quads() { return env_u32("EIM_SPILL_QUADS", 8192); }
static uint32_t task_quads() { return env_u32("EIM_TASK_QUADS", 8192); }
static uint32_t ring_w() {
  uint32_t w = env_u32("EIM_RING_W", IC_W);
  if (w < 32 || (w & (w - 1)) || w > IC_W) fail(EIM_E_INVAL, "EIM_RING_W must be a power of two in [32, 1024]");
  return w;
}

static uint32_t help_min() { return env_u32("EIM_HELP_QUADS", 1024); }
// probe-first rounds (EIM_PROBE_QUADS=0: off): root traversals are suspended
// after this many swept quads.  C2 (tools/ab_env.py, 2 x 5 IMMs): sampler
// kernels 9.23 ms off, 9.02 at 256, 8.92 at 1024, 8.93 at 4096 per IMM.
static uint32_t probe_quads() { return env_u32("EIM_PROBE_QUADS", 1024); }

template <int G, int NSG, class K, class GV>
static void launch_ic_on(eim_ctx* ctx, K kern, const GV& gv, const RoundView& R, uint64_t count, SampleCtl* ctl,
                         cudaStream_t st, bool spare_sm_slot, uint32_t W, size_t smem) {
  EIM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 0;
  EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, G * NSG, smem));
  if (per_sm < 1) fail(EIM_E_CUDA, "sampler does not fit on an SM");
  if (spare_sm_slot && per_sm > 1) per_sm -= 1;
  per_sm = std::min<int>(per_sm, (int)env_u32("EIM_IC_BLOCKS_SM", 64));  // development: resident groups per SM
  const uint64_t blocks = std::max<uint64_t>(1, (uint64_t)per_sm * ctx->sm_count);
  kern<<<(uint32_t)blocks, G * NSG, smem, st>>>(gv, R, count, W, ctl, spill_quads(), task_quads(), help_min(),
                                                probe_quads());
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches++;
}

template <int G, int NSG>
static void launch_ic(eim_ctx* ctx, const eim_graph* g, const RoundView& R, uint64_t count, SampleCtl* ctl,
                      cudaStream_t st, bool spare_sm_slot) {
  const uint32_t W = ring_w();
  const size_t smem = ic_smem<G, NSG>(W);
  with_graph_view(g, [&](const auto& gv) {
    using GV = std::decay_t<decltype(gv)>;
    launch_ic_on<G, NSG>(ctx, ic_kernel<G, NSG, GV>, gv, R, count, ctl, st, spare_sm_slot, W, smem);
  });
}


// the TQ task-queue counters follow the SampleCtl and the cancel/pause flags
constexpr size_t QC_OFFSET = (sizeof(SampleCtl) + 16 + 127) / 128 * 128;
constexpr size_t CTL_BYTES = QC_OFFSET + TQ * 128;
static unsigned long long* round_queues(Round& rd) {
  return reinterpret_cast<unsigned long long*>(static_cast<char*>(rd.ctl.p) + QC_OFFSET);
}

static RoundView round_view(Round& rd) {
  return RoundView{rd.table.as<unsigned long long>(),
                   rd.bits,
                   rd.sizes.as<uint32_t>(),
                   rd.edges.as<unsigned long long>(),
                   reinterpret_cast<const unsigned int*>(rd.ctl.as<SampleCtl>() + 1),
                   rd.first,
                   rd.queue.as<uint32_t>(),
                   reinterpret_cast<unsigned long long*>(static_cast<char*>(rd.queue.p) + 4ull * rd.pcap),
                   rd.pcap,
                   rd.tcap,
                   rd.dbg.as<unsigned long long>(),
                   philox_key(rd.seed),
                   std::getenv("EIM_NO_HOIST") ? 1u : 0u,
                   round_queues(rd),
                   std::getenv("EIM_NO_PREFETCH") ? 0u : 1u,
                   rd.list.as<uint32_t>(),
                   std::getenv("EIM_LT_NO_EVICT") ? 0u : 1u};
}

// one sampler launch over rd's remaining work, bracketed by events
static void round_kernel(eim_ctx* ctx, const eim_graph* g, Round& rd, cudaStream_t st, bool spare_sm_slot) {
  if (rd.nlaunch >= Round::MAX_LAUNCH) fail(EIM_E_STATE, "too many sampler launches in one round");
  SampleCtl* ctl = rd.ctl.as<SampleCtl>();
  const RoundView R = round_view(rd);
  const uint4* aug = rd.model == EIM_IC ? nullptr : lt_aug(ctx, g, st);  // built outside the launch's events
  EIM_CUDA(cudaEventRecord(rd.ev[2 * rd.nlaunch], st));
  if (rd.model == EIM_IC) {
    launch_ic<IC_G, IC_NSG>(ctx, g, R, rd.count, ctl, st, spare_sm_slot);
  } else {
    int per_sm = 0;
    EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lt_kernel<GraphView>, 256, 0));
    if (spare_sm_slot && per_sm > 1) per_sm -= 1;
    uint64_t blocks = std::min<uint64_t>((uint64_t)std::max(1, per_sm) * ctx->sm_count, (rd.count + 255) / 256);
    const uint32_t grid = (uint32_t)std::max<uint64_t>(blocks, 1);
    if (aug) lt_aug_kernel<<<grid, 256, 0, st>>>(g->view, aug, R, rd.count, ctl);
    else with_graph_view(g, [&](const auto& gv) { lt_kernel<<<grid, 256, 0, st>>>(gv, R, rd.count, ctl); });
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
  }
  EIM_CUDA(cudaEventRecord(rd.ev[2 * rd.nlaunch + 1], st));
  rd.nlaunch++;
  rd.stream = st;
  rd.launched = true;
}

// table + queue sizing, memsets and the first launch of rd's range on st
static void round_start(eim_ctx* ctx, const eim_graph* g, Round& rd, cudaStream_t st, bool spare_sm_slot) {
  const uint64_t count = rd.count;
  if (st != ctx->stream) {
    // the round's buffers may still be read by the previous round's
    // finalize (scatter) on the context's stream: start after it
    EIM_CUDA(cudaEventRecord(ctx->ev0, ctx->stream));
    EIM_CUDA(cudaStreamWaitEvent(st, ctx->ev0, 0));
  }
  rd.table.reserve(8ull << rd.bits, false, st);
  EIM_CUDA(cudaMemsetAsync(rd.table.p, 0, 8ull << rd.bits, st));
  if (rd.model == EIM_IC) {
    // task pool: half the table's slots (a task seed is a distinct member,
    // and the table is sized for >= 4x the expected members), descriptors
    // for half of that.  Consumers zero the descriptors they take, so
    // only fresh or abandoned memory needs a memset (the pool is written
    // before its descriptor is published).
    const uint64_t old_pcap = rd.pcap;
    rd.pcap = 1ull << (rd.bits - 1);
    rd.tcap = rd.pcap / 2;  // TQ segments of tcap / TQ descriptors
    void* before = rd.queue.p;
    rd.queue.reserve(4ull * rd.pcap + 16ull * rd.tcap, false, st);
    // the descriptors start at 4 * pcap: with another pool size they lie where
    // an earlier round's pool (non-zero seed ids) may have been
    if (rd.queue.p != before || rd.pcap != old_pcap) rd.qdirty = true;
    if (rd.qdirty) {
      EIM_CUDA(cudaMemsetAsync(static_cast<char*>(rd.queue.p) + 4ull * rd.pcap, 0, 16ull * rd.tcap, st));
      rd.qdirty = false;
    }
  } else {
    rd.pcap = rd.tcap = 0;
  }
  EIM_CUDA(cudaMemsetAsync(rd.sizes.p, 0, count * sizeof(uint32_t), st));
  EIM_CUDA(cudaMemsetAsync(rd.edges.p, 0, count * sizeof(unsigned long long), st));
  EIM_CUDA(cudaMemsetAsync(rd.ctl.p, 0, CTL_BYTES, st));
  if (std::getenv("EIM_DEBUG_TIMELINE")) {
    rd.dbg.reserve(64 * count, false, st);
    EIM_CUDA(cudaMemsetAsync(rd.dbg.p, 0, 64 * count, st));
  }
  rd.nlaunch = 0;
  rd.waited = false;
  rd.elim_ready = false;
  if (rd.model == EIM_IC) {
    rd.list.reserve(count * sizeof(uint32_t), false, st);
    const RoundView R = round_view(rd);
    with_graph_view(g, [&](const auto& gv) {
      // EIM_NO_PREPASS=1: every id gets a traversal (the singleton path is off)
      ic_prepass_kernel<<<grid_for(ctx, count, 256), 256, 0, st>>>(gv, R, count, rd.ctl.as<SampleCtl>(),
                                                                    rd.list.as<uint32_t>(),
                                                                    std::getenv("EIM_NO_PREPASS") != nullptr);
    });
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
  }
  round_kernel(ctx, g, rd, st, spare_sm_slot);
}

static unsigned int* round_flags(Round& rd) { return reinterpret_cast<unsigned int*>(rd.ctl.as<SampleCtl>() + 1); }

void round_pause(eim_ctx* ctx, Round& rd) {
  if (!rd.launched) return;
  EIM_CUDA(cudaMemsetAsync(round_flags(rd) + 1, 0xFF, sizeof(unsigned int), ctx->aux_stream));
}

void round_resume(eim_ctx* ctx, const eim_graph* g, Round& rd, cudaStream_t st) {
  if (!rd.launched) return;
  EIM_CUDA(cudaStreamSynchronize(ctx->aux_stream));  // an earlier pause write lands before the clear below
  EIM_CUDA(cudaStreamWaitEvent(st, rd.ev[2 * rd.nlaunch - 1], 0));
  EIM_CUDA(cudaMemsetAsync(round_flags(rd) + 1, 0, sizeof(unsigned int), st));
  round_kernel(ctx, g, rd, st, false);
}

void round_launch(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed, uint64_t first,
                  uint64_t count, uint64_t set_base, bool hist, Round& rd, cudaStream_t st, bool spare_sm_slot,
                  uint32_t rflags) {
  if (count == 0) return;
  rd.rflags = rflags;
  if (count >= 0x3FFFFFF0ull) fail(EIM_E_INVAL, "at most 2^30 sets per sampler launch");
  if (!rd.ev[0])
    for (cudaEvent_t& e : rd.ev) EIM_CUDA(cudaEventCreate(&e));
  rd.first = first;
  rd.count = count;
  rd.set_base = set_base;
  rd.pend = SampleResult{};
  rd.seed = seed;
  rd.model = model;
  rd.hist = hist;
  rd.sizes.reserve(count * sizeof(uint32_t), false, st);
  rd.edges.reserve(count * sizeof(unsigned long long), false, st);
  rd.fill.reserve(count * sizeof(uint32_t), false, st);
  rd.excl.reserve((count + 1) * sizeof(uint64_t), false, st);
  rd.ctl.reserve(CTL_BYTES, false, st);
  // table capacity: >= 4x the expected members (mean set size of earlier
  // rounds, else 64), at least 2^20 slots
  const double mean = ctx->est_mean_size > 0 ? ctx->est_mean_size : 64.0;
  // EIM_TABLE_BITS: smallest table (tests force overflow and the redo path)
  uint32_t bits = std::min<uint32_t>(std::max<uint32_t>(env_u32("EIM_TABLE_BITS", 20), 4), 31);
  const char* tf = std::getenv("EIM_TABLE_FACTOR");  // development: slots per expected member (default 4)
  const double factor = tf ? std::max(1.1, std::strtod(tf, nullptr)) : 4.0;
  while (bits < 31 && (double)(1ull << bits) < factor * mean * (double)count) bits++;
  // LT: twice as many slots while the table stays within the 2^30-slot
  // launch budget (fewer probe collisions on the walk's critical path: C3
  // walk kernel 0.963 -> 0.869 ms; 4x more cost the scatter more than it saves)
  if (model == EIM_LT && !tf && bits < 30) bits++;
  rd.bits = bits;
  round_start(ctx, g, rd, st, spare_sm_slot);
}

void round_cancel(eim_ctx* ctx, Round& rd) {
  if (!rd.launched) return;
  EIM_CUDA(cudaMemsetAsync(round_flags(rd), 0xFF, sizeof(unsigned int), ctx->aux_stream));
  EIM_CUDA(cudaStreamSynchronize(ctx->aux_stream));
  EIM_CUDA(cudaStreamSynchronize(rd.stream));
  rd.launched = false;
  rd.qdirty = true;  // items may be left in the queue
}

// Wait for rd's launches (resuming a paused round), redo an overflowed round
// with a larger table; accumulates the launch statistics in rd.pend.
static void round_wait(eim_ctx* ctx, const eim_graph* g, Round& rd) {
  cudaStream_t st = ctx->stream;
  SampleCtl* ctl = rd.ctl.as<SampleCtl>();
  SampleCtl* h = static_cast<SampleCtl*>(ctx->h_pinned);
  auto elapsed = [&](int from) {
    float total = 0, ms = 0;
    for (int i = from; i < rd.nlaunch; ++i) {
      EIM_CUDA(cudaEventElapsedTime(&ms, rd.ev[2 * i], rd.ev[2 * i + 1]));
      total += ms;
    }
    return (double)total;
  };
  for (int attempt = 0; !rd.waited; ++attempt) {
    int counted = 0;
    for (;;) {  // until every id is taken and no task is outstanding (a paused round is resumed here)
      EIM_CUDA(cudaStreamWaitEvent(st, rd.ev[2 * rd.nlaunch - 1], 0));
      EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl), cudaMemcpyDeviceToHost, st));
      EIM_CUDA(cudaStreamSynchronize(st));
      const uint64_t ntk = rd.model == EIM_IC ? h->ntickets : rd.count;
      trace_mark("sampler done", rd.first, rd.count);
      if ((h->ticket >= ntk && h->outstanding == 0) || h->arena_fail) break;
      round_resume(ctx, g, rd, st);
    }
    rd.pend.kernel_ms += elapsed(counted);
    rd.pend.launches += rd.nlaunch - counted;
    rd.pend.spilled += h->spilled;
    if (std::getenv("EIM_DEBUG_TIMELINE") && rd.model == EIM_IC) {
      std::fprintf(stderr, "timeline count=%llu ids_taken_us=%.1f tail_us=%.1f tasks=%llu spilled=%llu kernel_ms=%.3f\n",
                   (unsigned long long)rd.count, (h->t_last_id - h->t_first) * 1e-3, (h->t_end - h->t_last_id) * 1e-3,
                   h->tasks_pushed, h->spilled, elapsed(counted));
      std::vector<unsigned long long> d(8 * rd.count);
      EIM_CUDA(cudaMemcpy(d.data(), rd.dbg.p, d.size() * 8, cudaMemcpyDeviceToHost));
      std::vector<uint64_t> idx(rd.count);
      for (uint64_t i = 0; i < rd.count; ++i) idx[i] = i;
      std::sort(idx.begin(), idx.end(), [&](uint64_t a, uint64_t b) { return d[8 * a + 3] - d[8 * a + 2] > d[8 * b + 3] - d[8 * b + 2]; });
      for (int j = 0; j < 5 && j < (int)rd.count; ++j) {
        const unsigned long long* x = &d[8 * idx[j]];
        const double us = (x[3] - x[2]) * 1e-3, nb = std::max(1.0, (double)x[0]);
        std::fprintf(stderr, "  s=%llu batches=%llu quads=%llu live=%llu start_us=%.1f dur_us=%.1f us/batch=%.2f "
                     "stage=%.2f sweep=%.2f visit=%.2f\n",
                     (unsigned long long)idx[j], x[0], x[1], x[7], (x[2] - h->t_first) * 1e-3, us, us / nb,
                     x[4] * 1e-3 / nb, x[5] * 1e-3 / nb, x[6] * 1e-3 / nb);
      }
    }
    counted = rd.nlaunch;
    if (h->arena_fail) {  // rare: redo the whole range with a 4x larger table (and task pool)
      if (attempt >= 4 || rd.bits >= 31) fail(EIM_E_NOMEM, "membership table overflow");
      rd.bits = std::min<uint32_t>(rd.bits + 2, 31);
      rd.qdirty = true;
      round_start(ctx, g, rd, st, false);
      continue;
    }
    rd.waited = true;
  }
}

// Source elimination with empty sets dropped (R22): after the launch, the
// roots leave the sets (sizes - 1) and kidx = exclusive scan of the
// non-empty flags over the whole launch.  Returns the number of non-empty
// sets of the launch (once per launch; round_finalize reuses it).
uint64_t round_elim_kept(eim_ctx* ctx, const eim_graph* g, Round& rd) {
  if (!rd.launched || rd.count == 0) return 0;
  if ((rd.rflags & (RF_DROP_ROOT | RF_DROP_EMPTY)) != (RF_DROP_ROOT | RF_DROP_EMPTY))
    fail(EIM_E_STATE, "round_elim_kept on a round that keeps empty sets");
  round_wait(ctx, g, rd);
  if (rd.elim_ready) return rd.kept_total;
  cudaStream_t st = ctx->stream;
  SampleCtl* h = static_cast<SampleCtl*>(ctx->h_pinned);
  const uint64_t span = rd.count;
  rd.roots.reserve(span * sizeof(uint32_t), false, st);
  rd.kidx.reserve((span + 1) * sizeof(uint32_t), false, st);
  rd.ksizes.reserve(span * sizeof(uint32_t), false, st);
  uint32_t* roots = rd.roots.as<uint32_t>();
  uint32_t* kidx = rd.kidx.as<uint32_t>();
  roots_kernel<<<grid_for(ctx, span, 256), 256, 0, st>>>(rd.first, span, g->view.n, philox_key(rd.seed), roots);
  EIM_CUDA(cudaGetLastError());
  drop_root_sizes_kernel<<<grid_for(ctx, span + 1, 256), 256, 0, st>>>(rd.sizes.as<uint32_t>(), span, kidx);
  EIM_CUDA(cudaGetLastError());
  size_t tmp = 0;
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, kidx, kidx, span + 1, st));
  ctx->scratch.reserve(std::max<size_t>(tmp, 1 << 20), false, st);
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(ctx->scratch.p, tmp, kidx, kidx, span + 1, st));
  ctx->kernel_launches += 3;
  uint32_t* h32 = reinterpret_cast<uint32_t*>(&h->consumed);
  EIM_CUDA(cudaMemcpyAsync(h32, kidx + span, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  rd.kept_total = *h32;
  rd.elim_ready = true;
  return rd.kept_total;
}

SampleResult round_finalize(eim_ctx* ctx, const eim_graph* g, Round& rd, uint64_t use, uint64_t from, bool keep,
                            bool consume_all, AppendCuts* cuts) {
  SampleResult res;
  if (!rd.launched || rd.count == 0) return res;
  if (use > rd.count || from > use) fail(EIM_E_STATE, "round_finalize beyond the launched range");
  if (from > 0 && (rd.rflags & RF_DROP_ROOT)) fail(EIM_E_STATE, "partial appends of an eliminating round");
  cudaStream_t st = ctx->stream;
  SampleCtl* ctl = rd.ctl.as<SampleCtl>();
  SampleCtl* h = static_cast<SampleCtl*>(ctx->h_pinned);
  const bool drop_root = (rd.rflags & RF_DROP_ROOT) != 0;
  const bool drop_empty = drop_root && (rd.rflags & RF_DROP_EMPTY) != 0;
  if (drop_empty) round_elim_kept(ctx, g, rd);
  else round_wait(ctx, g, rd);
  res.kernel_ms = rd.pend.kernel_ms;
  res.launches = rd.pend.launches;
  res.spilled = rd.pend.spilled;
  rd.pend = SampleResult{};
  // ---- append the sets of s_local in [from, use); with keep the round's
  // table stays for a later append of the rest
  if (!keep) {
    rd.launched = false;
    rd.waited = false;
    rd.elim_ready = false;
  }
  res.kept = res.consumed = use - from;
  if (drop_empty) {
    // nothing kept and nothing consumed (a rank past the cut of a multi-rank round)
    if (use == 0 && !consume_all) {
      res.consumed = 0;
      return res;
    }
    if (consume_all && use != rd.kept_total) fail(EIM_E_STATE, "consume_all needs every non-empty set kept");
  } else if (use == from) {
    return res;
  }
  uint32_t* sizes = rd.sizes.as<uint32_t>() + from;
  uint32_t* roots = nullptr;
  uint32_t* kidx = nullptr;
  uint64_t consumed = use, nsets = use - from;
  size_t tmp = 0, tmp2 = 0;
  if (drop_empty) {
    // ---- source elimination (R22): only the first `use` non-empty sets are
    // kept and the ids up to the last kept one are consumed (round_elim_kept
    // has dropped the roots from the sizes and scanned the non-empty flags).
    roots = rd.roots.as<uint32_t>();
    kidx = rd.kidx.as<uint32_t>();
    const uint64_t span = rd.count;
    const uint64_t kept_total = rd.kept_total;
    consumed = span;
    nsets = kept_total;
    if (kept_total >= use && !consume_all) {
      nsets = use;
      find_consumed_kernel<<<grid_for(ctx, span, 256), 256, 0, st>>>(kidx, span, (uint32_t)use, &ctl->consumed);
      EIM_CUDA(cudaGetLastError());
      EIM_CUDA(cudaMemcpyAsync(&h->consumed, &ctl->consumed, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
      EIM_CUDA(cudaStreamSynchronize(st));
      consumed = h->consumed;
      ctx->kernel_launches += 1;
    }
    if (nsets)
      compact_sizes_kernel<<<grid_for(ctx, consumed, 256), 256, 0, st>>>(sizes, kidx, consumed,
                                                                        rd.ksizes.as<uint32_t>());
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches += 1;
    sizes = rd.ksizes.as<uint32_t>();
  } else if (drop_root) {
    // ---- source elimination without dropping sets (eim_sample_rrr_ex)
    rd.roots.reserve(use * sizeof(uint32_t), false, st);
    roots = rd.roots.as<uint32_t>();
    roots_kernel<<<grid_for(ctx, use, 256), 256, 0, st>>>(rd.first, use, g->view.n, philox_key(rd.seed), roots);
    EIM_CUDA(cudaGetLastError());
    drop_root_sizes_kernel<<<grid_for(ctx, use + 1, 256), 256, 0, st>>>(sizes, use, nullptr);
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches += 2;
  }
  res.kept = nsets;
  res.consumed = consumed - from;
  // ---- sizes -> offsets (sample-id order) -> arena placement -> scatter + histogram
  uint64_t* excl = rd.excl.as<uint64_t>();
  const uint64_t set_index0 = rd.first - rd.set_base;
  ensure_sets(ctx, set_index0 + from + std::max<uint64_t>(nsets, 1));
  sizes_to_offsets_kernel<<<grid_for(ctx, nsets + 1, 256), 256, 0, st>>>(sizes, nsets, excl);
  EIM_CUDA(cudaGetLastError());
  const bool ic = rd.model == EIM_IC;
  // examined edges go to the context's device accumulator (edges_read):
  // IC summed by the scatter, LT reduced from the per-walk steps and added
  unsigned long long* d_edges_acc = ctx->edges_acc.as<unsigned long long>();
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, excl, excl, nsets + 1, st));
  if (!ic) EIM_CUDA(cub::DeviceReduce::Sum(nullptr, tmp2, rd.edges.as<unsigned long long>() + from, &ctl->edges,
                                           consumed - from, st));
  ctx->scratch.reserve(std::max<size_t>(std::max(tmp, tmp2), 1 << 20), false, st);
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(ctx->scratch.p, tmp, excl, excl, nsets + 1, st));
  if (!ic) {
    EIM_CUDA(cub::DeviceReduce::Sum(ctx->scratch.p, tmp2, rd.edges.as<unsigned long long>() + from, &ctl->edges,
                                    consumed - from, st));
    add_u64_kernel<<<1, 1, 0, st>>>(d_edges_acc, &ctl->edges);
    EIM_CUDA(cudaGetLastError());
  }
  EIM_CUDA(cudaMemcpyAsync(&h->ticket, excl + nsets, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  const uint32_t ncut = cuts ? cuts->n : 0u;
  uint64_t* hcut = reinterpret_cast<uint64_t*>(static_cast<char*>(ctx->h_pinned) + 3600);
  if (ncut) {
    if (ncut > 2 || drop_root || !rd.hist) fail(EIM_E_STATE, "append cuts need a plain round with its histogram");
    for (uint32_t j = 0; j < ncut; ++j) {
      if (cuts->cut[j] <= from || cuts->cut[j] >= use) fail(EIM_E_STATE, "append cut outside the appended range");
      EIM_CUDA(cudaMemcpyAsync(hcut + j, excl + (cuts->cut[j] - from), sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    }
  }
  EIM_CUDA(cudaStreamSynchronize(st));
  const uint64_t total = h->ticket, cursor = ctx->arena_used;
  for (uint32_t j = 0; j < ncut; ++j) {
    cuts->total[j] = cursor + hcut[j];
    // the snapshot starts as C before this append; the scatter adds the sets below the cut
    EIM_CUDA(cudaMemcpyAsync(cuts->snap[j], ctx->C_total.p, (uint64_t)g->view.n * sizeof(uint32_t),
                             cudaMemcpyDeviceToDevice, st));
  }
  trace_mark("append sizes", from, use);
  arena_ensure(ctx, cursor + total);
  if (nsets) {
    place_sets_kernel<<<grid_for(ctx, nsets, 256), 256, 0, st>>>(excl, sizes, nsets, cursor, set_index0 + from,
                                                                  ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>());
    EIM_CUDA(cudaGetLastError());
  }
  EIM_CUDA(cudaMemsetAsync(rd.fill.as<uint32_t>() + from, 0, (consumed - from) * sizeof(uint32_t), st));
  const uint64_t nslots = 1ull << rd.bits;
  auto scatter = [&](auto gv) {
    scatter_kernel<<<grid_for(ctx, nslots, 256), 256, 0, st>>>(
        rd.table.as<unsigned long long>(), nslots, ctx->set_start.as<uint64_t>(), set_index0,
        (uint32_t)from, (uint32_t)consumed, rd.fill.as<uint32_t>(), ctx->arena.as<uint32_t>(), ctx->arena_b,
        rd.hist ? ctx->C_total.as<uint32_t>() : nullptr, gv, ic, d_edges_acc, roots, kidx,
        ncut > 0 ? cuts->snap[0] : nullptr, ncut > 0 ? (uint32_t)cuts->cut[0] : 0u,
        ncut > 1 ? cuts->snap[1] : nullptr, ncut > 1 ? (uint32_t)cuts->cut[1] : 0u);
  };
  with_graph_view(g, scatter);
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches += 6;
  ctx->arena_used = cursor + total;
  ctx->est_mean_size = std::max(1.0, (double)(total + (drop_root ? consumed : 0)) / (double)(consumed - from));
  return res;
}

void edges_reset(eim_ctx* ctx) {
  ctx->edges_acc.reserve(64, false, ctx->stream);
  EIM_CUDA(cudaMemsetAsync(ctx->edges_acc.p, 0, sizeof(unsigned long long), ctx->stream));
}

uint64_t edges_read(eim_ctx* ctx) {
  uint64_t* h = reinterpret_cast<uint64_t*>(static_cast<char*>(ctx->h_pinned) + 3584);
  EIM_CUDA(cudaMemcpyAsync(h, ctx->edges_acc.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  EIM_CUDA(cudaStreamSynchronize(ctx->stream));
  return *h;
}

uint64_t max_launch_ids(const eim_ctx* ctx) {
  const uint32_t forced = env_u32("EIM_MAX_LAUNCH_IDS", 0);  // tests: force several launches per range
  if (forced) return forced;
  // the membership table of a launch holds >= 4 slots per expected member;
  // keep it within 2^30 slots (8 GiB; the task pool adds 2 GiB)
  const double mean = ctx->est_mean_size > 0 ? ctx->est_mean_size : 64.0;
  const double cap = std::floor((double)(1ull << 30) / (4.0 * mean));
  return (uint64_t)std::max(65536.0, std::min(cap, (double)(1ull << 29)));
}

SampleResult sample_range(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed,
                          uint64_t first, uint64_t count, uint64_t set_base, bool hist, uint32_t rflags) {
  SampleResult tot;
  Round& rd = ctx->rounds[0];
  for (uint64_t done = 0; done < count;) {  // launches sized for the table budget
    const uint64_t c = std::min(count - done, max_launch_ids(ctx));
    round_launch(ctx, g, model, seed, first + done, c, set_base, hist, rd, ctx->stream, false, rflags);
    const SampleResult r = round_finalize(ctx, g, rd, c);
    tot.edges += r.edges;
    tot.spilled += r.spilled;
    tot.launches += r.launches;
    tot.kernel_ms += r.kernel_ms;
    tot.kept += r.kept;
    tot.consumed += r.consumed;
    done += c;
  }
  return tot;
}

}  // namespace eim

#ifdef EIM_SWEEP_BENCH
extern "C" int eim_dev_sweep_bench(int blocks, uint32_t nrows, uint32_t d, uint32_t reps, double* ns_per_batch,
                                   double* quads_per_ns) {
  using namespace eim;
  RoundView R{};
  R.K = philox_key(1);
  GraphView g{};
  unsigned long long* out = nullptr;
  SampleCtl* ctl = nullptr;
  cudaMalloc(&out, 3 * 8 * blocks);
  cudaMalloc(&ctl, sizeof(SampleCtl));
  const size_t smem = sg_bytes<IC_G>(32);
  cudaFuncSetAttribute(sweep_bench_kernel<IC_G>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  for (int it = 0; it < 2; ++it) sweep_bench_kernel<IC_G><<<blocks, IC_G, smem>>>(g, R, ctl, nrows, d, reps, out);
  std::vector<unsigned long long> h(3 * blocks);
  cudaMemcpy(h.data(), out, h.size() * 8, cudaMemcpyDeviceToHost);
  double ns = 0, q = 0;
  for (int b = 0; b < blocks; ++b) {
    ns = std::max(ns, (double)h[3 * b]);
    q += (double)h[3 * b + 1];
  }
  *ns_per_batch = ns / (reps - 1);
  *quads_per_ns = q / ns;
  cudaFree(out);
  cudaFree(ctl);
  return (int)cudaGetLastError();
}
#endif
