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
// IC (ic_group_kernel<G, GLOBAL_RING>): G threads cooperate on one sample.  A
//   batch of up to G frontier vertices has its in-rows merged into one space
//   of Philox quads (4 consecutive edge ids share one Philox4x32-10 call,
//   reading R1) that the G threads sweep, so small rows do not idle threads
//   and hub rows split evenly.  An edge into u is live iff its draw <= T_u
//   (R2); in_nbr[e] is read only for live edges.  Heavy samples under WC are
//   chains of ~100 hub expansions, so G threads per sample (not a warp) keep
//   the per-level latency low, and they start as soon as their id is drawn.
//   The frontier lives in a shared-memory ring (tier 1); a sample whose
//   backlog outgrows the ring is redone by a 512-thread group with the ring
//   in global memory (tier 2, capacity n) under a distinct key tag.
// LT (lt_kernel): one thread per reverse walk (sequential by nature),
//   visited set = the same global table; no capacity limit.
#include <cub/cub.cuh>

#include <cstdio>
#include <cstdlib>
#include <string>

#include "eim_internal.h"
#include "philox.cuh"

namespace eim {

namespace {

constexpr unsigned FULL = 0xFFFFFFFFu;
constexpr uint32_t MAX_PROBE = 256;
__device__ unsigned long long* g_dbg_group = nullptr;  // EIM_DEBUG_TIMES (development)

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
constexpr int IC_G = 256;          // threads per sample (one block), tier 1
constexpr int IC_NG = 1;           // groups per block
constexpr int IC_U = 2;            // consecutive quads per thread per sweep iteration

// ---------------------------------------------------------------- table
// key = ((s_local + 1) | tier << 31) << 32 | v ;  0 = empty slot.
__device__ __forceinline__ unsigned long long table_key(uint32_t s_local, uint32_t tier, uint32_t v) {
  return ((unsigned long long)((s_local + 1u) | (tier << 31)) << 32) | (unsigned long long)v;
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

// ---------------------------------------------------------------- groups
// One group = one block (G = blockDim.x), so a group barrier is __syncthreads.
template <int G>
__device__ __forceinline__ void gsync(int) {
  __syncthreads();
}

struct GroupCtl {
  uint32_t tail, flag, s_local, pad;
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
  if constexpr (G == 32) {
    total = __shfl_sync(FULL, x, 31);
    return x;
  } else {
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
}

enum : uint32_t { FLAG_RING = 1u, FLAG_TABLE = 2u };

struct RoundView {
  unsigned long long* keys;
  uint32_t bits;
  uint32_t* sizes;     // [count] members per sample (s_local)
  uint8_t* failed;     // [count] 1 = tier-1 attempt abandoned (its tier-0 keys are ignored)
  uint64_t base;       // sample id of s_local = 0
};

// One IC RRR set (Alg. 2 l.5-20) by a group of G threads.  ring = frontier
// backlog of capacity W (W a power of two).  Returns the flag (0 = success);
// size = number of members.
template <int G, int U>
__device__ __forceinline__ uint32_t ic_group_sample(const GraphView& g, const PhiloxKey& K, const RoundView& R,
                                                    uint32_t s_local, uint32_t tier, uint32_t* ring, uint32_t W,
                                                    GroupRows<G>& rw, GroupCtl& gc, int gtid, int gi,
                                                    unsigned long long& se, uint32_t& size) {
  const uint64_t s = R.base + s_local;
  if (gtid == 0) {
    const uint32_t root = draw_root(s, g.n, K);
    const int r = table_insert(R.keys, R.bits, table_key(s_local, tier, root));
    ring[0] = root;
    gc.tail = 1;
    gc.flag = (r < 0) ? FLAG_TABLE : 0u;
  }
  gsync<G>(gi);
  uint32_t head = 0;
  se = 0;
#ifdef EIM_DEV_TIMING
  unsigned long long* dbg = g_dbg_group;
#else
  constexpr unsigned long long* dbg = nullptr;  // per-phase timing only in development builds
#endif
  unsigned long long t_begin = 0, t_stage = 0, t_sweep = 0, nbatch = 0, nquads = 0, ta = 0;
  if (dbg && gtid == 0) t_begin = gtimer();
  for (;;) {
    const uint32_t tail = *(volatile uint32_t*)&gc.tail;
    const uint32_t flag = *(volatile uint32_t*)&gc.flag;
    if (flag || head >= tail) {
      size = tail;
      if (dbg && gtid == 0 && tier == 0) {
        unsigned long long* d = dbg + 6ull * s_local;
        d[0] = t_begin; d[1] = gtimer(); d[2] = nbatch; d[3] = t_stage; d[4] = t_sweep; d[5] = nquads;
      }
      return flag;
    }
    if (dbg && gtid == 0) ta = gtimer();
    const uint32_t nb = min((uint32_t)G, tail - head);
    uint32_t nq = 0;
    if (gtid < nb) {
      const uint32_t u = ring[(head + gtid) & (W - 1)];
      const unsigned long long e0 = g.off[u], e1 = g.off[u + 1];
      if (e1 > e0) {
        nq = (uint32_t)(((e1 - 1) >> 2) - (e0 >> 2) + 1);
        rw.q0[gtid] = e0 >> 2;
        rw.wlo[gtid] = (uint8_t)(e0 & 3);
        rw.whi[gtid] = (uint8_t)((e1 - 1) & 3);
        rw.T[gtid] = g.thr[u];
      }
      rw.nq[gtid] = nq;
      se += e1 - e0;
    }
    uint32_t total;
    const uint32_t incl = group_incl_scan<G>(nq, gtid, gi, gc, total);
    if (gtid < nb) rw.qend[gtid] = incl;
    head += nb;  // ring slots [old head, head) are free again: their rows are staged
    gsync<G>(gi);
    unsigned long long tb = 0;
    if (dbg && gtid == 0) { tb = gtimer(); t_stage += tb - ta; nbatch++; nquads += total; }
    // Sweep the batch's quad space; each thread takes U quads per iteration
    // (j, j+G, .., j+(U-1)G) whose Philox chains are independent (ILP).
    int r = -1;
    uint32_t qe = 0, qb = 0, nq_r = 0, T_r = 0, wlo_r = 0, whi_r = 0;
    unsigned long long q0_r = 0;
    for (uint32_t base = 0; base < total; base += U * G) {
      unsigned long long qk[U];
      uint32_t Tk[U], mk[U];
#pragma unroll
      for (int k = 0; k < U; ++k) {
        const uint32_t j = base + k * G + gtid;
        mk[k] = 0u;
        qk[k] = 0ull;
        Tk[k] = 0u;
        if (j < total) {
          if (j >= qe) {
            do {
              ++r;
              qe = rw.qend[r];
            } while (j >= qe);
            nq_r = rw.nq[r];
            qb = qe - nq_r;
            q0_r = rw.q0[r];
            T_r = rw.T[r];
            wlo_r = rw.wlo[r];
            whi_r = rw.whi[r];
          }
          const uint32_t li = j - qb;
          uint32_t m = 0xFu;
          if (li == 0) m &= 0xFu << wlo_r;
          if (li == nq_r - 1) m &= 0xFu >> (3u - whi_r);
          mk[k] = m;
          qk[k] = q0_r + li;
          Tk[k] = T_r;
        }
      }
      uint4 wk[U];
#pragma unroll
      for (int k = 0; k < U; ++k) wk[k] = philox_at(qk[k], s, TAG_EDGE, K);
#pragma unroll
      for (int k = 0; k < U; ++k) {
        const uint32_t T = Tk[k];
        uint32_t live = (wk[k].x <= T ? 1u : 0u) | (wk[k].y <= T ? 2u : 0u) | (wk[k].z <= T ? 4u : 0u) |
                        (wk[k].w <= T ? 8u : 0u);
        live &= mk[k];
        while (live) {
          const int i = __ffs(live) - 1;
          live &= live - 1;
          const uint32_t v = g.nbr[(qk[k] << 2) + i];
          const int ins = table_insert(R.keys, R.bits, table_key(s_local, tier, v));
          if (ins > 0) {
            const uint32_t pos = atomicAdd(&gc.tail, 1u);
            if (pos - head < W) ring[pos & (W - 1)] = v;
            else atomicOr(&gc.flag, FLAG_RING);
          } else if (ins < 0) {
            atomicOr(&gc.flag, FLAG_TABLE);
          }
        }
      }
    }
    gsync<G>(gi);
    if (dbg && gtid == 0) t_sweep += gtimer() - tb;
  }
}

// tier 1 (GLOBAL_RING = false): shared-memory ring of W entries per group,
// over the contiguous ids [0, count).  tier 2 (GLOBAL_RING = true): ring of W
// entries per group slot in global memory, over a list of failed ids.
template <int G, bool GLOBAL_RING>
__global__ void __launch_bounds__(G) ic_group_kernel(GraphView g, uint64_t seed, RoundView R,
                                                                        uint64_t count,
                                                                        const uint32_t* __restrict__ ids,
                                                                        uint32_t W, SampleCtl* ctl,
                                                                        uint32_t* retry_out, uint32_t* gring) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int gi = threadIdx.x / G, gtid = threadIdx.x % G;
  const size_t per_group = sizeof(GroupCtl) + sizeof(GroupRows<G>) + (GLOBAL_RING ? 0 : (size_t)4 * W);
  unsigned char* base = smem_raw + (size_t)gi * per_group;
  GroupCtl& gc = *reinterpret_cast<GroupCtl*>(base);
  GroupRows<G>& rw = *reinterpret_cast<GroupRows<G>*>(base + sizeof(GroupCtl));
  const uint64_t slot = (uint64_t)blockIdx.x * (blockDim.x / G) + gi;
  uint32_t* ring = GLOBAL_RING ? gring + slot * (uint64_t)W
                               : reinterpret_cast<uint32_t*>(base + sizeof(GroupCtl) + sizeof(GroupRows<G>));
  const uint32_t tier = GLOBAL_RING ? 1u : 0u;
  const PhiloxKey K = philox_key(seed);
  unsigned long long edges_acc = 0;
  for (;;) {
    if (gtid == 0) {
      const unsigned long long t = atomicAdd(&ctl->ticket, 1ull);
      gc.s_local = t < count ? (ids ? ids[t] : (uint32_t)t) : 0xFFFFFFFFu;
    }
    gsync<G>(gi);
    const uint32_t s_local = gc.s_local;
    if (s_local == 0xFFFFFFFFu) break;
    unsigned long long se = 0;
    uint32_t size = 0;
    const uint32_t flag = ic_group_sample<G, IC_U>(g, K, R, s_local, tier, ring, W, rw, gc, gtid, gi, se, size);
    if (gtid == 0) {
      if (flag == 0) {
        R.sizes[s_local] = size;
      } else if (flag & FLAG_TABLE) {
        atomicOr(reinterpret_cast<unsigned int*>(&ctl->arena_fail), 1u);  // table too full: host redoes the round
      } else {
        R.failed[s_local] = 1;
        retry_out[atomicAdd(&ctl->retry_count, 1ull)] = s_local;
      }
    }
    if (flag == 0) edges_acc += se;
    gsync<G>(gi);
  }
  for (int o = 16; o > 0; o >>= 1) edges_acc += __shfl_xor_sync(FULL, edges_acc, o);
  if ((threadIdx.x & 31) == 0 && edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

// ---------------------------------------------------------------- fused IC
// Tier 1: one block traverses MANY samples at once (fused traversals).  The
// block keeps up to FS active samples in shared-memory slots; its frontier
// ring holds (slot, vertex) entries of all of them.  Each batch takes up to
// FG entries from the ring -- whatever samples they belong to -- merges their
// in-rows into one Philox-quad space and sweeps it with all FG threads, so
// the batch stays full while light samples come and go, and a heavy sample
// (a long chain of hub expansions) advances one frontier batch per iteration
// without holding back the rest.  Before each batch, free slots are refilled
// with new sample ids from the launch ticket (up to one per thread).
constexpr int FG = 512;                 // threads per block
constexpr int FS = 512;                 // sample slots per block
constexpr uint32_t FW = 4096;           // frontier ring entries per block
constexpr int FU = 4;                   // consecutive quads per thread per sweep iteration

struct FusedSlot {
  uint32_t s_local, members, pending, flag;
  unsigned long long edges;
  unsigned long long t_start;  // debug timing (EIM_DEBUG_TIMES)
  uint32_t levels, last_batch;
};

struct FusedShared {
  FusedSlot slot[FS];
  uint32_t ring_v[FW];
  uint16_t ring_s[FW];
  unsigned long long q0[FG];
  uint32_t qend[FG], nq[FG], T[FG];
  uint16_t rslot[FG];
  uint8_t wlo[FG], whi[FG];
  uint16_t free_stack[FS];
  uint32_t free_count, tail, exhausted, wsum[FG / 32];
  unsigned long long t0;
};

// A live in-edge reached v for the sample in slot sl: insert (sample, v) into
// the round table; a new member joins the block's frontier ring.
__device__ __forceinline__ void fused_visit(const GraphView& g, const RoundView& R, FusedShared& S, uint32_t v,
                                            uint32_t sl, uint32_t sloc, uint32_t head) {
  FusedSlot& q = S.slot[sl];
  const int ins = table_insert(R.keys, R.bits, table_key(sloc, 0, v));
  if (ins > 0) {
    atomicAdd(&q.members, 1u);
    const uint32_t pos = atomicAdd(&S.tail, 1u);
    if (pos - head < FW) {
      atomicAdd(&q.pending, 1u);
      S.ring_v[pos & (FW - 1)] = v;
      S.ring_s[pos & (FW - 1)] = (uint16_t)sl;
    } else {
      atomicOr(&q.flag, FLAG_RING);  // entry lost: the sample is redone by tier 2
    }
  } else if (ins < 0) {
    atomicOr(&q.flag, FLAG_TABLE);
  }
}

__global__ void __launch_bounds__(FG, 2) ic_fused_kernel(GraphView g, uint64_t seed, RoundView R, uint64_t count,
                                                      SampleCtl* ctl, uint32_t* retry_out, uint32_t chunk,
                                                      unsigned long long* dbg) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  FusedShared& S = *reinterpret_cast<FusedShared*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const PhiloxKey K = philox_key(seed);
  for (int i = tid; i < FS; i += FG) S.free_stack[i] = (uint16_t)(FS - 1 - i);
  if (tid == 0) {
    S.free_count = FS;
    S.tail = 0;
    S.exhausted = 0;
  }
  __syncthreads();
  uint32_t head = 0, batch_no = 0;
  unsigned long long edges_acc = 0;
  for (;;) {
    ++batch_no;
    // ---- (1) refill free slots with new samples while the backlog is short
    uint32_t tail = S.tail;
    const uint32_t backlog = tail - head;
    uint32_t want = 0;
    if (!S.exhausted && backlog < (uint32_t)FG) want = min(min(S.free_count, (uint32_t)FG - backlog), chunk);
    __syncthreads();  // everyone has read free_count / tail / exhausted
    if (want > 0) {
      if (tid == 0) {
        const unsigned long long t0 = atomicAdd(&ctl->ticket, (unsigned long long)want);
        S.t0 = t0;
        if (t0 + want >= count) S.exhausted = 1;
      }
      __syncthreads();
      const unsigned long long t0 = S.t0;
      const uint32_t got = t0 >= count ? 0u : (uint32_t)min((unsigned long long)want, count - t0);
      if ((uint32_t)tid < got) {
        const uint16_t sl = S.free_stack[S.free_count - 1 - tid];
        const uint32_t s_local = (uint32_t)(t0 + tid);
        const uint32_t root = draw_root(R.base + s_local, g.n, K);
        const int r = table_insert(R.keys, R.bits, table_key(s_local, 0, root));
        FusedSlot& q = S.slot[sl];
        q.s_local = s_local;
        q.members = 1;
        q.pending = 1;
        q.flag = r < 0 ? FLAG_TABLE : 0u;
        q.edges = 0;
        if (dbg) {
          unsigned long long tnow;
          asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tnow));
          q.t_start = tnow;
          q.levels = 0;
          q.last_batch = 0xFFFFFFFFu;
        }
        S.ring_v[(tail + tid) & (FW - 1)] = root;
        S.ring_s[(tail + tid) & (FW - 1)] = sl;
      }
      __syncthreads();
      if (tid == 0) {
        S.free_count -= got;
        S.tail = tail + got;
      }
      __syncthreads();
      tail = S.tail;
    }
    if (head == tail) {
      if (S.exhausted) break;  // uniform: all threads read the same shared words after a barrier
      continue;
    }
    // ---- (2) stage the rows of up to FG frontier entries
    const uint32_t nb = min((uint32_t)FG, tail - head);
    uint32_t nq = 0;
    if ((uint32_t)tid < nb) {
      const uint32_t e = (head + tid) & (FW - 1);
      const uint32_t u = S.ring_v[e];
      const uint16_t sl = S.ring_s[e];
      S.rslot[tid] = sl;
      if (dbg && atomicExch(&S.slot[sl].last_batch, batch_no) != batch_no) atomicAdd(&S.slot[sl].levels, 1u);
      if (S.slot[sl].flag == 0) {  // rows of failed samples are skipped
        const unsigned long long e0 = g.off[u], e1 = g.off[u + 1];
        if (e1 > e0) {
          nq = (uint32_t)(((e1 - 1) >> 2) - (e0 >> 2) + 1);
          S.q0[tid] = e0 >> 2;
          S.wlo[tid] = (uint8_t)(e0 & 3);
          S.whi[tid] = (uint8_t)((e1 - 1) & 3);
          S.T[tid] = g.thr[u];
        }
        atomicAdd(&S.slot[sl].edges, e1 - e0);
      }
      S.nq[tid] = nq;
    }
    // block inclusive scan of nq
    uint32_t x = nq;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += t;
    }
    if (lane == 31) S.wsum[wid] = x;
    __syncthreads();
    uint32_t pre = 0, total = 0;
#pragma unroll
    for (int i = 0; i < FG / 32; ++i) {
      const uint32_t t = S.wsum[i];
      pre += (i < wid) ? t : 0u;
      total += t;
    }
    if ((uint32_t)tid < nb) S.qend[tid] = x + pre;
    head += nb;
    __syncthreads();
    // ---- (3) sweep the merged quad space.  Thread t takes FU = 4 CONSECUTIVE
    // quads per iteration.  Their row is found by a binary search over the
    // staged quad ends (no linear walk over small rows).  When the run lies
    // inside one row (the common case for hub rows) the four Philox calls
    // share the sample counter and are issued back to back; each quad is
    // first tested with one 4-way min against T (live edges are rare: ~1 per
    // expanded row under WC) before the exact per-word test.
    for (uint32_t base = (uint32_t)tid * FU; base < total; base += FU * FG) {
      // row r: first row with qend[r] > base
      uint32_t lo = 0, hi = nb - 1;
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (S.qend[mid] > base) hi = mid;
        else lo = mid + 1;
      }
      uint32_t r = lo;
      uint32_t qe = S.qend[r], nq_r = S.nq[r];
      uint32_t qb = qe - nq_r;
      if (base + FU <= qe) {
        // fast path: the whole run is inside row r
        const uint32_t li = base - qb;
        const unsigned long long q = S.q0[r] + li;
        const uint32_t T = S.T[r];
        const uint32_t sl = S.rslot[r];
        const uint32_t sloc = S.slot[sl].s_local;
        const uint64_t sid = R.base + sloc;
        uint4 wk[FU];
#pragma unroll
        for (int k = 0; k < FU; ++k) wk[k] = philox_at(q + k, sid, TAG_EDGE, K);
        uint32_t mk[FU];
#pragma unroll
        for (int k = 0; k < FU; ++k) mk[k] = 0xFu;
        if (li == 0) mk[0] &= 0xFu << S.wlo[r];
        if (li + FU == nq_r) mk[FU - 1] &= 0xFu >> (3u - S.whi[r]);
        bool any = false;
#pragma unroll
        for (int k = 0; k < FU; ++k) any |= min(min(wk[k].x, wk[k].y), min(wk[k].z, wk[k].w)) <= T;
        if (!any) continue;
#pragma unroll
        for (int k = 0; k < FU; ++k) {
          uint32_t live = (wk[k].x <= T ? 1u : 0u) | (wk[k].y <= T ? 2u : 0u) | (wk[k].z <= T ? 4u : 0u) |
                          (wk[k].w <= T ? 8u : 0u);
          live &= mk[k];
          while (live) {
            const int i = __ffs(live) - 1;
            live &= live - 1;
            fused_visit(g, R, S, g.nbr[((q + k) << 2) + i], sl, sloc, head);
          }
        }
        continue;
      }
      // general path: the run crosses row ends
#pragma unroll 1
      for (int k = 0; k < FU; ++k) {
        const uint32_t j = base + k;
        if (j >= total) break;
        while (j >= qe) {
          ++r;
          qe = S.qend[r];
          nq_r = S.nq[r];
        }
        qb = qe - nq_r;
        const uint32_t li = j - qb;
        uint32_t m = 0xFu;
        if (li == 0) m &= 0xFu << S.wlo[r];
        if (li == nq_r - 1) m &= 0xFu >> (3u - S.whi[r]);
        const unsigned long long q = S.q0[r] + li;
        const uint32_t T = S.T[r];
        const uint32_t sl = S.rslot[r];
        const uint32_t sloc = S.slot[sl].s_local;
        const uint4 w = philox_at(q, R.base + sloc, TAG_EDGE, K);
        uint32_t live = (w.x <= T ? 1u : 0u) | (w.y <= T ? 2u : 0u) | (w.z <= T ? 4u : 0u) | (w.w <= T ? 8u : 0u);
        live &= m;
        while (live) {
          const int i = __ffs(live) - 1;
          live &= live - 1;
          fused_visit(g, R, S, g.nbr[(q << 2) + i], sl, sloc, head);
        }
      }
    }
    __syncthreads();
    // ---- (4) retire the batch's entries; a sample with nothing pending is done
    if ((uint32_t)tid < nb) {
      const uint16_t sl = S.rslot[tid];
      FusedSlot& q = S.slot[sl];
      if (atomicSub(&q.pending, 1u) == 1u) {
        const uint32_t f = q.flag;
        if (dbg) {
          unsigned long long tnow;
          asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tnow));
          dbg[4ull * q.s_local + 0] = q.t_start;
          dbg[4ull * q.s_local + 1] = tnow;
          dbg[4ull * q.s_local + 2] = q.levels;
          dbg[4ull * q.s_local + 3] = blockIdx.x | ((unsigned long long)q.edges << 20);
        }
        if (f == 0u) {
          R.sizes[q.s_local] = q.members;
          edges_acc += q.edges;
        } else if (f & FLAG_TABLE) {
          atomicOr(reinterpret_cast<unsigned int*>(&ctl->arena_fail), 1u);
        } else {
          R.failed[q.s_local] = 1;
          retry_out[atomicAdd(&ctl->retry_count, 1ull)] = q.s_local;
        }
        S.free_stack[atomicAdd(&S.free_count, 1u)] = sl;
      }
    }
    __syncthreads();
  }
  for (int o = 16; o > 0; o >>= 1) edges_acc += __shfl_xor_sync(FULL, edges_acc, o);
  if (lane == 0 && edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

// ---------------------------------------------------------------- pool IC
// Tier 1 default: ONE global task pool per round, no per-sample on-chip
// state.  A task is a chunk of at most PQ Philox quads of one in-row of one
// sample: (s_local, first quad, quad count, edge-word masks, T).  Whoever
// discovers a new member v of sample s (table insert succeeded) loads v's row
// bounds and publishes ceil(quads / PQ) chunk tasks; any warp claims tasks,
// merges the quads of its claimed tasks into one space swept by its 32 lanes,
// and publishes the tasks of the members it discovers.  BFS order is
// irrelevant to the result (the set is the reverse reachability of the root
// in the live-edge world), so there are no levels and no barriers: a hub row
// found in a deep chain is split across the whole GPU the moment it is found,
// and the round ends when the count of unfinished tasks reaches zero.
constexpr uint32_t PQ = 64;  // quads per chunk task

struct PoolView {
  ulonglong2* q;                 // task slots (zeroed; y != 0 marks a published task)
  unsigned long long cap;
  unsigned long long* head;      // claim counter
  unsigned long long* tail;      // reservation counter
  unsigned long long* pending;   // seeds not yet processed + tasks published and not yet finished
  unsigned int* flags;           // bit 0: queue full, bit 1: table full, bit 2: watchdog
};

__device__ __forceinline__ void pool_push_row(const GraphView& g, const PoolView& P, uint32_t s_local, uint32_t v) {
  const unsigned long long e0 = g.off[v], e1 = g.off[v + 1];
  if (e1 == e0) return;
  const unsigned long long q0 = e0 >> 2;
  const unsigned long long nq = ((e1 - 1) >> 2) - q0 + 1;
  const uint32_t T = g.thr[v];
  const unsigned long long nch = (nq + PQ - 1) / PQ;
  atomicAdd(P.pending, nch);
  const unsigned long long base = atomicAdd(P.tail, nch);
  unsigned long long ok = nch;
  if (base + nch > P.cap) {
    ok = base >= P.cap ? 0ull : P.cap - base;
    atomicAdd(P.pending, 0ull - (nch - ok));
    atomicOr(P.flags, 1u);
  }
  for (unsigned long long c = 0; c < ok; ++c) {
    const unsigned long long cq0 = q0 + c * PQ;
    P.q[base + c].x = (cq0 & 0xFFFFFFFFull) | ((unsigned long long)T << 32);
  }
  __threadfence();
  for (unsigned long long c = 0; c < ok; ++c) {
    const unsigned long long cq0 = q0 + c * PQ;
    const uint32_t cn = (uint32_t)min((unsigned long long)PQ, nq - c * PQ);
    const uint32_t wlo = c == 0 ? (uint32_t)(e0 & 3) : 0u;
    const uint32_t whi = c == nch - 1 ? (uint32_t)((e1 - 1) & 3) : 3u;
    const uint32_t meta = cn | (wlo << 16) | (whi << 18) | ((uint32_t)(cq0 >> 32) << 20);
    *(volatile unsigned long long*)&P.q[base + c].y = (unsigned long long)meta | ((unsigned long long)(s_local + 1) << 32);
  }
}

__global__ void __launch_bounds__(256) ic_pool_kernel(GraphView g, uint64_t seed, RoundView R, uint64_t count,
                                                      PoolView P, SampleCtl* ctl, uint32_t total_warps) {
  const int lane = threadIdx.x & 31;
  const PhiloxKey K = philox_key(seed);
  unsigned long long edges_acc = 0;
  // ---- seeds: roots of the round's samples (Alg. 2 l.6-9)
  for (;;) {
    unsigned long long t0 = 0;
    if (lane == 0) t0 = atomicAdd(&ctl->ticket, 32ull);
    t0 = __shfl_sync(FULL, t0, 0);
    if (t0 >= count) break;
    const unsigned long long t = t0 + lane;
    if (t < count) {
      const uint32_t s_local = (uint32_t)t;
      const uint32_t root = draw_root(R.base + s_local, g.n, K);
      const int r = table_insert(R.keys, R.bits, table_key(s_local, 0, root));
      if (r < 0) atomicOr(P.flags, 2u);
      atomicAdd(&R.sizes[s_local], 1u);
      pool_push_row(g, P, s_local, root);
    }
    const uint32_t nseed = (uint32_t)min(32ull, count - t0);
    __threadfence();
    __syncwarp();
    if (lane == 0) atomicAdd(P.pending, 0ull - (unsigned long long)nseed);
  }
  // ---- tasks
  unsigned long long spins = 0;
  for (;;) {
    // claim n consecutive slots; n adapts to the backlog so that in a thin
    // tail consecutive tasks (the chunks of one hub row) go to different warps
    unsigned long long h = 0, n = 0;
    if (lane == 0) {
      const unsigned long long hv = *(volatile unsigned long long*)P.head;
      const unsigned long long tv = *(volatile unsigned long long*)P.tail;
      const unsigned long long avail = tv > hv ? tv - hv : 0ull;
      n = min(32ull, max(1ull, avail / total_warps));
      h = atomicAdd(P.head, n);
    }
    h = __shfl_sync(FULL, h, 0);
    n = __shfl_sync(FULL, n, 0);
    bool mine = (unsigned long long)lane < n && h + lane < P.cap;
    bool done = !mine;
    for (;;) {
      // wait until some claimed slot is published, or the round is over
      unsigned long long y = 0;
      if (!done) y = *(volatile unsigned long long*)&P.q[h + lane].y;
      const bool ready = !done && y != 0ull;
      const unsigned rmask = __ballot_sync(FULL, ready);
      if (rmask == 0u) {
        if (__ballot_sync(FULL, !done) == 0u) break;  // all claimed slots handled
        unsigned long long pend = 0;
        if (lane == 0) pend = *(volatile unsigned long long*)P.pending;
        pend = __shfl_sync(FULL, pend, 0);
        if (pend == 0ull) break;  // nothing will be published any more
        if (++spins > (1ull << 26)) {
          if (lane == 0) atomicOr(P.flags, 4u);
          break;
        }
        __nanosleep(200);
        continue;
      }
      __threadfence();
      // decode this lane's task
      uint32_t cn = 0, T = 0, wlo = 0, whi = 3, s_local = 0;
      unsigned long long cq0 = 0;
      if (ready) {
        const unsigned long long x = __ldcg(&P.q[h + lane].x);
        const uint32_t meta = (uint32_t)y;
        s_local = (uint32_t)(y >> 32) - 1u;
        cn = meta & 0xFFFFu;
        wlo = (meta >> 16) & 3u;
        whi = (meta >> 18) & 3u;
        cq0 = (x & 0xFFFFFFFFull) | ((unsigned long long)(meta >> 20) << 32);
        T = (uint32_t)(x >> 32);
        edges_acc += 4ull * cn - wlo - (3u - whi);
        done = true;
      }
      // merge the ready tasks' quads into one space swept by the warp
      uint32_t incl = cn;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t v = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += v;
      }
      const uint32_t total = __shfl_sync(FULL, incl, 31);
      for (uint32_t base = 0; base < total; base += 32u) {
        const uint32_t j = base + lane;
        // owner lane of quad j: the first lane whose inclusive quad sum exceeds j
        int src = 0;
#pragma unroll
        for (int b = 16; b > 0; b >>= 1) {
          const uint32_t ib = __shfl_sync(FULL, incl, src + b - 1);
          if (ib <= j) src += b;
        }
        const uint32_t r_incl = __shfl_sync(FULL, incl, src);
        const uint32_t r_cn = __shfl_sync(FULL, cn, src);
        const uint32_t r_T = __shfl_sync(FULL, T, src);
        const uint32_t r_wlo = __shfl_sync(FULL, wlo, src);
        const uint32_t r_whi = __shfl_sync(FULL, whi, src);
        const uint32_t r_s = __shfl_sync(FULL, s_local, src);
        const unsigned long long r_q0 = __shfl_sync(FULL, cq0, src);
        if (j < total) {
          const uint32_t li = j - (r_incl - r_cn);
          const unsigned long long q = r_q0 + li;
          const uint4 w = philox_at(q, R.base + r_s, TAG_EDGE, K);
          uint32_t m = 0xFu;
          if (li == 0) m &= 0xFu << r_wlo;
          if (li == r_cn - 1) m &= 0xFu >> (3u - r_whi);
          uint32_t live = (w.x <= r_T ? 1u : 0u) | (w.y <= r_T ? 2u : 0u) | (w.z <= r_T ? 4u : 0u) |
                          (w.w <= r_T ? 8u : 0u);
          live &= m;
          while (live) {
            const int i = __ffs(live) - 1;
            live &= live - 1;
            const uint32_t v = g.nbr[(q << 2) + i];
            const int ins = table_insert(R.keys, R.bits, table_key(r_s, 0, v));
            if (ins > 0) {
              atomicAdd(&R.sizes[r_s], 1u);
              pool_push_row(g, P, r_s, v);
            } else if (ins < 0) {
              atomicOr(P.flags, 2u);
            }
          }
        }
      }
      // finished tasks leave the pending count only after their children
      // were counted in (fence + warp barrier order the lanes' increments first)
      __threadfence();
      __syncwarp();
      if (lane == 0) atomicAdd(P.pending, 0ull - (unsigned long long)__popc(rmask));
    }
    if (*(volatile unsigned int*)P.flags & 4u) break;
    unsigned long long pend = 0;
    if (lane == 0) pend = *(volatile unsigned long long*)P.pending;
    pend = __shfl_sync(FULL, pend, 0);
    if (pend == 0ull) break;
  }
  for (int o = 16; o > 0; o >>= 1) edges_acc += __shfl_xor_sync(FULL, edges_acc, o);
  if (lane == 0 && edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

// ---------------------------------------------------------------- LT
// Reverse LT walk (R3-R5): at u with d^-(u) > 0, tau_u is the
// LT-tagged draw of u and the chosen in-neighbour is position
// floor(tau * d / 2^32) of u's row (the prefix-scan choice under WC
// weights); the walk stops when d^-(u) = 0 or the chosen vertex is already in
// the set.  One thread per walk; visited set = the round table.
__global__ void __launch_bounds__(256) lt_kernel(GraphView g, uint64_t seed, RoundView R, uint64_t count,
                                                 SampleCtl* ctl) {
  const PhiloxKey K = philox_key(seed);
  unsigned long long edges_acc = 0;
  for (;;) {
    const unsigned long long t = atomicAdd(&ctl->ticket, 1ull);
    if (t >= count) break;
    const uint32_t s_local = (uint32_t)t;
    const uint64_t s = R.base + s_local;
    uint32_t u = draw_root(s, g.n, K);
    bool ok = table_insert(R.keys, R.bits, table_key(s_local, 0, u)) >= 0;
    uint32_t L = 1;
    unsigned long long steps = 0;
    while (ok) {
      const unsigned long long e0 = g.off[u], e1 = g.off[u + 1];
      if (e1 == e0) break;
      ++steps;
      const uint4 w = philox_at((uint64_t)(u >> 2), s, TAG_LT, K);
      const uint32_t tau = word_of(w, u & 3u);
      const unsigned long long j = __umul64hi((unsigned long long)tau << 32, e1 - e0);
      const uint32_t v = g.nbr[e0 + j];
      const int ins = table_insert(R.keys, R.bits, table_key(s_local, 0, v));
      if (ins == 0) break;
      if (ins < 0) ok = false;
      ++L;
      u = v;
    }
    if (ok) {
      R.sizes[s_local] = L;
      edges_acc += steps;
    } else {
      atomicOr(reinterpret_cast<unsigned int*>(&ctl->arena_fail), 1u);
    }
  }
  if (edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

// ---------------------------------------------------------------- output
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

// Every live table entry is a member: arena[start(s) + fill[s]++] = v.
__global__ void scatter_kernel(const unsigned long long* __restrict__ keys, uint64_t nslots,
                               const uint8_t* __restrict__ failed, const uint64_t* __restrict__ set_start,
                               uint64_t set_index0, uint32_t* __restrict__ fill, uint32_t* __restrict__ arena,
                               uint32_t* __restrict__ C) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nslots; i += stride) {
    const unsigned long long k = keys[i];
    if (k == 0ull) continue;
    const uint32_t hi = (uint32_t)(k >> 32);
    const uint32_t tier = hi >> 31;
    const uint32_t s_local = (hi & 0x7FFFFFFFu) - 1u;
    if (tier == 0 && failed[s_local]) continue;  // abandoned tier-1 attempt; redone under tier-2 keys
    const uint32_t v = (uint32_t)k;
    const uint32_t p = atomicAdd(&fill[s_local], 1u);
    arena[set_start[set_index0 + s_local] + p] = v;
    if (C) atomicAdd(&C[v], 1u);
  }
}

constexpr uint32_t IC_W = 1024;    // shared-memory frontier ring per group
constexpr int IC_G2 = 512;         // tier 2 (global ring of capacity >= n)

template <int G, bool GR>
size_t ic_smem_per_group(uint32_t W) {
  return sizeof(GroupCtl) + sizeof(GroupRows<G>) + (GR ? 0 : (size_t)4 * W);
}

}  // namespace

// ------------------------------------------------------------------ host
void arena_reset(eim_ctx* ctx) {
  ctx->arena.reserve(sizeof(uint32_t) * (1u << 22), false, ctx->stream);
  ctx->ctl.reserve(sizeof(SampleCtl) + 2 * sizeof(unsigned long long), false, ctx->stream);
  // ctl layout: [SampleCtl][cursor][valid_end]
  EIM_CUDA(cudaMemsetAsync(ctx->ctl.p, 0, sizeof(SampleCtl) + 2 * sizeof(unsigned long long), ctx->stream));
  ctx->est_mean_size = 0;
}

uint64_t arena_cursor(eim_ctx* ctx) {
  unsigned long long* cur = reinterpret_cast<unsigned long long*>(ctx->ctl.as<SampleCtl>() + 1);
  unsigned long long v = 0;
  EIM_CUDA(cudaMemcpyAsync(&v, cur, sizeof(v), cudaMemcpyDeviceToHost, ctx->stream));
  EIM_CUDA(cudaStreamSynchronize(ctx->stream));
  return v;
}

void ensure_sets(eim_ctx* ctx, uint64_t num_sets) {
  ctx->set_start.reserve(num_sets * sizeof(uint64_t), true, ctx->stream);
  ctx->set_len.reserve(num_sets * sizeof(uint32_t), true, ctx->stream);
}

template <int G, bool GR>
static void launch_ic(eim_ctx* ctx, const eim_graph* g, uint64_t seed, const RoundView& R, uint64_t count,
                      const uint32_t* ids, uint32_t W, SampleCtl* ctl, uint32_t* retry_out, uint32_t* gring,
                      int NG, uint64_t max_groups) {
  const size_t smem = ic_smem_per_group<G, GR>(W) * NG;
  auto kern = ic_group_kernel<G, GR>;
  EIM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 0;
  EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, G * NG, smem));
  if (per_sm < 1) fail(EIM_E_CUDA, "sampler tier does not fit on an SM");
  uint64_t blocks = (uint64_t)per_sm * ctx->sm_count;
  blocks = std::min<uint64_t>(blocks, (count + NG - 1) / NG);
  blocks = std::min<uint64_t>(blocks, std::max<uint64_t>(1, max_groups / NG));
  blocks = std::max<uint64_t>(blocks, 1);
  kern<<<(uint32_t)blocks, G * NG, smem, ctx->stream>>>(g->view, seed, R, count, ids, W, ctl, retry_out, gring);
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches++;
}

SampleResult sample_range(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed,
                          uint64_t first, uint64_t count, uint64_t set_base, bool hist) {
  SampleResult res;
  if (count == 0) return res;
  if (count >= 0x7FFFFFF0ull) fail(EIM_E_INVAL, "at most 2^31 sets per sampler launch");
  cudaStream_t st = ctx->stream;
  ensure_sets(ctx, first + count - set_base);
  SampleCtl* ctl = ctx->ctl.as<SampleCtl>();
  unsigned long long* d_cursor = reinterpret_cast<unsigned long long*>(ctl + 1);
  SampleCtl* h = static_cast<SampleCtl*>(ctx->h_pinned);
  unsigned long long* h_cursor = reinterpret_cast<unsigned long long*>(h + 1);
  ctx->rsizes.reserve(count * sizeof(uint32_t), false, st);
  ctx->rfailed.reserve(count, false, st);
  ctx->rfill.reserve(count * sizeof(uint32_t), false, st);
  ctx->retry_a.reserve(count * sizeof(uint32_t), false, st);
  ctx->stage_a.reserve((count + 1) * sizeof(uint64_t), false, st);

  // table capacity: >= 4x the expected members of the round (mean set size
  // of earlier rounds, else 64), at least 2^20 slots
  const double mean = ctx->est_mean_size > 0 ? ctx->est_mean_size : 64.0;
  uint32_t bits = 20;
  while (bits < 32 && (double)(1ull << bits) < 4.0 * mean * (double)count) bits++;

  for (int attempt = 0;; ++attempt) {
    ctx->table.reserve((8ull << bits), false, st);
    RoundView R{ctx->table.as<unsigned long long>(), bits, ctx->rsizes.as<uint32_t>(), ctx->rfailed.as<uint8_t>(),
                first};
    EIM_CUDA(cudaMemsetAsync(R.keys, 0, 8ull << bits, st));
    EIM_CUDA(cudaMemsetAsync(R.failed, 0, count, st));
    EIM_CUDA(cudaMemsetAsync(R.sizes, 0, count * sizeof(uint32_t), st));
    EIM_CUDA(cudaMemsetAsync(ctl, 0, sizeof(SampleCtl), st));
    EIM_CUDA(cudaEventRecord(ctx->ev0, st));
    const char* var = getenv("EIM_IC_KERNEL");  // development switch: default "group" / "fused" / "pool"
    const std::string variant = var ? std::string(var) : std::string("group");
    if (model == EIM_IC && variant == "pool") {
      // task pool capacity from the chunks per sample of earlier rounds
      const double cps = ctx->est_chunks_per_sample > 0 ? ctx->est_chunks_per_sample : 256.0;
      uint64_t cap = std::max<uint64_t>(1ull << 20, (uint64_t)(2.0 * cps * (double)count) + 4096);
      if (attempt > 0) cap = std::max<uint64_t>(cap, ctx->pool_cap_hint);
      const size_t old_bytes = ctx->pool.bytes;
      ctx->pool.reserve(cap * 16, false, st);
      cap = ctx->pool.bytes / 16;
      if (ctx->pool.bytes != old_bytes) ctx->pool_dirty = cap;  // fresh allocation: zero all of it
      const uint64_t dirty = std::min<uint64_t>(ctx->pool_dirty, cap);
      if (dirty) EIM_CUDA(cudaMemsetAsync(ctx->pool.p, 0, dirty * 16, st));
      ctx->pool_ctl.reserve(64, false, st);
      unsigned long long* pc = ctx->pool_ctl.as<unsigned long long>();
      unsigned long long* hpc = reinterpret_cast<unsigned long long*>(static_cast<char*>(ctx->h_pinned) + 2048);
      hpc[0] = 0; hpc[1] = 0; hpc[2] = count; hpc[3] = 0;
      EIM_CUDA(cudaMemcpyAsync(pc, hpc, 32, cudaMemcpyHostToDevice, st));
      PoolView P{ctx->pool.as<ulonglong2>(), cap, pc, pc + 1, pc + 2, reinterpret_cast<unsigned int*>(pc + 3)};
      int per_sm = 0;
      EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, ic_pool_kernel, 256, 0));
      const uint32_t blocks = (uint32_t)std::max(1, per_sm) * ctx->sm_count;
      ic_pool_kernel<<<blocks, 256, 0, st>>>(g->view, seed, R, count, P, ctl, blocks * 8);
      EIM_CUDA(cudaGetLastError());
      ctx->kernel_launches++;
      EIM_CUDA(cudaMemcpyAsync(hpc, pc, 32, cudaMemcpyDeviceToHost, st));
      EIM_CUDA(cudaStreamSynchronize(st));
      const uint64_t used = hpc[1];
      const unsigned int pflags = (unsigned int)hpc[3];
      ctx->pool_dirty = std::max<uint64_t>(ctx->pool_dirty, std::min<uint64_t>(used, cap));
      if (pflags & 4u) fail(EIM_E_CUDA, "sampler watchdog fired (task pool stalled)");
      if (pflags & 1u) {  // task pool overflow: redo the round with a larger pool
        ctx->pool_cap_hint = std::max<uint64_t>(cap * 2, used + used / 4);
        if (attempt >= 6) fail(EIM_E_NOMEM, "task pool overflow");
        continue;
      }
      if (pflags & 2u) {
        if (attempt >= 4 || bits >= 31) fail(EIM_E_NOMEM, "membership table overflow");
        bits += 2;
        continue;
      }
      ctx->est_chunks_per_sample = std::max(1.0, (double)used / (double)count);
    } else if (model == EIM_IC && variant == "group") {
      const char* dbgpath = getenv("EIM_DEBUG_TIMES");
      unsigned long long* dbgp = nullptr;
      if (dbgpath) {
        ctx->stage_c.reserve(count * 48, false, st);
        dbgp = ctx->stage_c.as<unsigned long long>();
        EIM_CUDA(cudaMemsetAsync(dbgp, 0, count * 48, st));
      }
      EIM_CUDA(cudaMemcpyToSymbolAsync(g_dbg_group, &dbgp, sizeof(dbgp), 0, cudaMemcpyHostToDevice, st));
      const char* gs = getenv("EIM_IC_G");  // development: group size 256 / 512 / 1024
      const int gsel = gs ? atoi(gs) : IC_G;
      if (gsel == 256)
        launch_ic<256, false>(ctx, g, seed, R, count, nullptr, IC_W, ctl, ctx->retry_a.as<uint32_t>(), nullptr, 1, ~0ull);
      else if (gsel == 512)
        launch_ic<512, false>(ctx, g, seed, R, count, nullptr, IC_W, ctl, ctx->retry_a.as<uint32_t>(), nullptr, 1, ~0ull);
      else
        launch_ic<1024, false>(ctx, g, seed, R, count, nullptr, IC_W, ctl, ctx->retry_a.as<uint32_t>(), nullptr, 1, ~0ull);
      if (dbgpath) {
        std::vector<unsigned long long> hd(count * 6);
        EIM_CUDA(cudaMemcpyAsync(hd.data(), dbgp, count * 48, cudaMemcpyDeviceToHost, st));
        EIM_CUDA(cudaStreamSynchronize(st));
        FILE* f = fopen(dbgpath, "ab");
        if (f) {
          const unsigned long long hdr[2] = {first, count};
          fwrite(hdr, 8, 2, f);
          fwrite(hd.data(), 8, hd.size(), f);
          fclose(f);
        }
        unsigned long long* nul = nullptr;
        EIM_CUDA(cudaMemcpyToSymbolAsync(g_dbg_group, &nul, sizeof(nul), 0, cudaMemcpyHostToDevice, st));
      }
    } else if (model == EIM_IC) {
      const size_t smem = sizeof(FusedShared);
      EIM_CUDA(cudaFuncSetAttribute(ic_fused_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      int per_sm = 0;
      EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, ic_fused_kernel, FG, smem));
      uint64_t blocks = (uint64_t)std::max(1, per_sm) * ctx->sm_count;
      blocks = std::max<uint64_t>(1, std::min<uint64_t>(blocks, count));
      // new samples per block per batch: small enough that every block gets a share of the round
      const uint32_t chunk = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(64, count / (blocks * 8)));
      const char* dbgpath = getenv("EIM_DEBUG_TIMES");
      unsigned long long* dbg = nullptr;
      if (dbgpath) {
        ctx->stage_c.reserve(count * 32, false, st);
        dbg = ctx->stage_c.as<unsigned long long>();
        EIM_CUDA(cudaMemsetAsync(dbg, 0, count * 32, st));
      }
      ic_fused_kernel<<<(uint32_t)blocks, FG, smem, st>>>(g->view, seed, R, count, ctl, ctx->retry_a.as<uint32_t>(),
                                                          chunk, dbg);
      if (dbgpath) {
        std::vector<unsigned long long> hd(count * 4);
        EIM_CUDA(cudaMemcpyAsync(hd.data(), dbg, count * 32, cudaMemcpyDeviceToHost, st));
        EIM_CUDA(cudaStreamSynchronize(st));
        FILE* f = fopen(dbgpath, "ab");
        if (f) {
          const unsigned long long hdr[2] = {first, count};
          fwrite(hdr, 8, 2, f);
          fwrite(hd.data(), 8, hd.size(), f);
          fclose(f);
        }
      }
      EIM_CUDA(cudaGetLastError());
      ctx->kernel_launches++;
    } else {
      int per_sm = 0;
      EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lt_kernel, 256, 0));
      uint64_t blocks = std::min<uint64_t>((uint64_t)std::max(1, per_sm) * ctx->sm_count, (count + 255) / 256);
      lt_kernel<<<(uint32_t)blocks, 256, 0, st>>>(g->view, seed, R, count, ctl);
      EIM_CUDA(cudaGetLastError());
      ctx->kernel_launches++;
    }
    EIM_CUDA(cudaEventRecord(ctx->ev1, st));
    EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl) + 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    float ms = 0;
    EIM_CUDA(cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1));
    res.kernel_ms += ms;
    res.launches++;
    uint64_t edges = h->edges;
    bool table_full = h->arena_fail != 0;
    if (!table_full && h->retry_count > 0) {
      // tier 2: frontier backlog outgrew the shared ring; redo with a global ring of capacity >= n
      const uint64_t nretry = h->retry_count;
      res.tier2 += nretry;
      uint32_t W2 = 1;
      while (W2 < g->view.n) W2 <<= 1;
      uint64_t slots = std::min<uint64_t>(nretry, std::max<uint64_t>(1, (1ull << 30) / (4ull * W2)));
      slots = std::min<uint64_t>(slots, (uint64_t)ctx->sm_count);
      ctx->tier_queue.reserve(slots * (uint64_t)W2 * 4, false, st);
      EIM_CUDA(cudaMemsetAsync(ctl, 0, sizeof(SampleCtl), st));
      EIM_CUDA(cudaEventRecord(ctx->ev0, st));
      launch_ic<IC_G2, true>(ctx, g, seed, R, nretry, ctx->retry_a.as<uint32_t>(), W2, ctl, nullptr,
                             ctx->tier_queue.as<uint32_t>(), 1, slots);
      EIM_CUDA(cudaEventRecord(ctx->ev1, st));
      EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl), cudaMemcpyDeviceToHost, st));
      EIM_CUDA(cudaStreamSynchronize(st));
      float ms2 = 0;
      EIM_CUDA(cudaEventElapsedTime(&ms2, ctx->ev0, ctx->ev1));
      res.kernel_ms += ms2;
      res.launches++;
      edges += h->edges;
      table_full = h->arena_fail != 0;
      if (!table_full && h->retry_count) fail(EIM_E_CUDA, "tier-2 sampler failed with a ring of capacity n");
    }
    if (table_full) {
      if (attempt >= 4 || bits >= 31) fail(EIM_E_NOMEM, "membership table overflow");
      bits += 2;  // rare: redo the whole round with a 4x larger table
      continue;
    }
    res.edges += edges;
    // ---- sizes -> offsets (sample-id order) -> arena placement -> scatter + histogram
    uint64_t* excl = ctx->stage_a.as<uint64_t>();
    sizes_to_offsets_kernel<<<grid_for(ctx, count + 1, 256), 256, 0, st>>>(ctx->rsizes.as<uint32_t>(), count, excl);
    EIM_CUDA(cudaGetLastError());
    size_t tmp = 0;
    EIM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, excl, excl, count + 1, st));
    ctx->scratch.reserve(std::max<size_t>(tmp, 1 << 20), false, st);
    EIM_CUDA(cub::DeviceScan::ExclusiveSum(ctx->scratch.p, tmp, excl, excl, count + 1, st));
    EIM_CUDA(cudaMemcpyAsync(&h->ticket, excl + count, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    EIM_CUDA(cudaMemcpyAsync(h_cursor, d_cursor, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    const uint64_t total = h->ticket, cursor = h_cursor[0];
    ctx->arena.reserve((cursor + total) * sizeof(uint32_t), true, st);
    const uint64_t set_index0 = first - set_base;
    place_sets_kernel<<<grid_for(ctx, count, 256), 256, 0, st>>>(excl, ctx->rsizes.as<uint32_t>(), count, cursor,
                                                                  set_index0, ctx->set_start.as<uint64_t>(),
                                                                  ctx->set_len.as<uint32_t>());
    EIM_CUDA(cudaGetLastError());
    EIM_CUDA(cudaMemsetAsync(ctx->rfill.p, 0, count * sizeof(uint32_t), st));
    const uint64_t nslots = 1ull << bits;
    scatter_kernel<<<grid_for(ctx, nslots, 256), 256, 0, st>>>(
        R.keys, nslots, R.failed, ctx->set_start.as<uint64_t>(), set_index0, ctx->rfill.as<uint32_t>(),
        ctx->arena.as<uint32_t>(), hist ? ctx->C_total.as<uint32_t>() : nullptr);
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches += 5;
    h_cursor[0] = cursor + total;
    h_cursor[1] = cursor + total;
    EIM_CUDA(cudaMemcpyAsync(d_cursor, h_cursor, 2 * sizeof(uint64_t), cudaMemcpyHostToDevice, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    ctx->est_mean_size = std::max(1.0, (double)total / (double)count);
    return res;
  }
}

}  // namespace eim
