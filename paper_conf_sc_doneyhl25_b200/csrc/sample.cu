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

constexpr int IC_G = 256;          // threads per sample (one block), tier 1
constexpr int IC_NG = 1;           // groups per block
constexpr int IC_U = 2;            // consecutive quads per thread per sweep iteration

// ---------------------------------------------------------------- table
// key = ((s_local + 1) | tier << 30) << 32 | v ;  0 = empty slot.  tier =
// attempt number of the sample (0, 1, 2): the scatter keeps only the keys of
// the attempt that succeeded.
__device__ __forceinline__ unsigned long long table_key(uint32_t s_local, uint32_t tier, uint32_t v) {
  return ((unsigned long long)((s_local + 1u) | (tier << 30)) << 32) | (unsigned long long)v;
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
  uint32_t tail, flag, s_local, nlive;
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

enum : uint32_t { FLAG_RING = 1u, FLAG_TABLE = 2u, FLAG_CANCEL = 4u, FLAG_HANDOFF = 8u };

struct RoundView {
  unsigned long long* keys;
  uint32_t bits;
  uint32_t* sizes;               // [count] members per sample (s_local)
  uint8_t* failed;               // [count] attempt (tier) whose keys are the sample's members
  unsigned long long* edges;     // [count] examined in-edges (IC) / walk steps (LT) per sample
  const unsigned int* cancel;    // [0] cancel (round not needed), [1] pause (take no new ids)
  uint64_t base;                 // sample id of s_local = 0
  PhiloxKey K;                   // round keys of the seed (kernel parameter: read as constant operands)
};

// One IC RRR set (Alg. 2 l.5-20) by a group of G threads.  ring = frontier
// backlog of capacity W (W a power of two).  Returns the flag (0 = success);
// size = number of members.
// Row descriptors of queued frontier vertices, loaded when the vertex is
// discovered (tier 1): the next batch stages its rows from shared memory.
struct RingRows {
  unsigned long long* e0;  // [W] first in-edge
  uint32_t* d;             // [W] in-degree
  uint32_t* T;             // [W] IC threshold
};

constexpr uint32_t LIVE_CAP = 512;  // live in-edges buffered per batch (more are visited inline)

// One IC RRR set (Alg. 2 l.5-20) by a group of G threads.  ring = frontier
// backlog of capacity W (W a power of two); rr (nullable) = prefetched rows
// of the ring entries.  A batch is three phases separated by group
// barriers: stage up to G queued rows and scan their Philox-quad counts;
// sweep the quads (Philox + compare only; the in-neighbour of a live edge is
// loaded and parked in a shared list); visit the parked neighbours in
// parallel (one table insert each; a new member joins the ring with its row
// bounds).  Separating the visits keeps the long-latency loads and atomics of
// the rare live edges off the Philox sweep and runs them side by side, which
// bounds the per-level latency of long chains.  Returns the flag (0 = ok).
template <int G, int U>
__device__ __forceinline__ uint32_t ic_group_sample(const GraphView& g, const PhiloxKey& K, const RoundView& R,
                                                    uint32_t s_local, uint32_t tier, uint32_t* ring, uint32_t W,
                                                    const RingRows* rr, uint32_t* live_v, GroupRows<G>& rw,
                                                    GroupCtl& gc, int gtid, int gi, unsigned long long& se,
                                                    uint32_t& size, const SampleCtl* ctl, uint64_t count,
                                                    uint32_t handoff) {
  const uint64_t s = R.base + s_local;
  uint32_t head = 0;
  // visit v: table insert; a new member is appended to the ring (with its row)
  auto visit = [&](uint32_t v) {
    const int ins = table_insert(R.keys, R.bits, table_key(s_local, tier, v));
    if (ins > 0) {
      const uint32_t pos = atomicAdd(&gc.tail, 1u);
      if (pos - head < W) {
        const uint32_t sl = pos & (W - 1);
        ring[sl] = v;
        if (rr) {
          const unsigned long long e0 = g.off[v];
          rr->e0[sl] = e0;
          rr->d[sl] = (uint32_t)(g.off[v + 1] - e0);
          rr->T[sl] = g.thr[v];
        }
      } else {
        atomicOr(&gc.flag, FLAG_RING);
      }
    } else if (ins < 0) {
      atomicOr(&gc.flag, FLAG_TABLE);
    }
  };
  if (gtid == 0) {
    gc.tail = 0;
    gc.flag = 0;
    gc.nlive = 0;
    visit(draw_root(s, g.n, K));
  }
  gsync<G>(gi);
  se = 0;
  for (;;) {
    const uint32_t tail = *(volatile uint32_t*)&gc.tail;
    const uint32_t flag = *(volatile uint32_t*)&gc.flag;
    if (flag || head >= tail) {
      size = tail;
      return flag;
    }
    if (*(volatile const unsigned int*)R.cancel) {
      gsync<G>(gi);  // every thread has read the control words above
      return FLAG_CANCEL;
    }
    // ---- stage
    const uint32_t nb = min((uint32_t)G, tail - head);
    uint32_t nq = 0;
    if (gtid < nb) {
      const uint32_t sl = (head + gtid) & (W - 1);
      unsigned long long e0, e1;
      uint32_t T;
      if (rr) {
        e0 = rr->e0[sl];
        e1 = e0 + rr->d[sl];
        T = rr->T[sl];
      } else {
        const uint32_t u = ring[sl];
        e0 = g.off[u];
        e1 = g.off[u + 1];
        T = g.thr[u];
      }
      if (e1 > e0) {
        nq = (uint32_t)(((e1 - 1) >> 2) - (e0 >> 2) + 1);
        rw.q0[gtid] = e0 >> 2;
        rw.wlo[gtid] = (uint8_t)(e0 & 3);
        rw.whi[gtid] = (uint8_t)((e1 - 1) & 3);
        rw.T[gtid] = T;
      }
      rw.nq[gtid] = nq;
      se += e1 - e0;
    }
    if (gtid == 0) gc.nlive = 0;
    uint32_t total;
    const uint32_t incl = group_incl_scan<G>(nq, gtid, gi, gc, total);
    if (gtid < nb) rw.qend[gtid] = incl;
    head += nb;  // ring slots [old head, head) are free again: their rows are staged
    gsync<G>(gi);
    // ---- sweep: each thread takes U quads per iteration (j, j+G, ..) whose
    // Philox chains are independent (ILP)
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
      // all U Philox calls before any branch (independent chains interleave);
      // one 4-way min per quad against T decides whether the rare exact test runs
      uint4 wk[U];
#pragma unroll
      for (int k = 0; k < U; ++k) wk[k] = philox_at(qk[k], s, TAG_EDGE, K);
      bool any = false;
#pragma unroll
      for (int k = 0; k < U; ++k) any |= (min(min(wk[k].x, wk[k].y), min(wk[k].z, wk[k].w)) <= Tk[k]) & (mk[k] != 0u);
      if (!any) continue;
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
          const uint32_t p = atomicAdd(&gc.nlive, 1u);
          if (p < LIVE_CAP) live_v[p] = v;
          else visit(v);
        }
      }
    }
    gsync<G>(gi);
    // ---- visit the parked live neighbours, one per thread
    const uint32_t nl = min(*(volatile uint32_t*)&gc.nlive, LIVE_CAP);
    for (uint32_t t = gtid; t < nl; t += G) visit(live_v[t]);
    // tail hand-off: once the launch has no new ids left and only a few
    // samples are still running (the long chains), give this one up; the
    // host redoes it with a whole SM per sample (tier 2)
    if (handoff && gtid == 0 && *(volatile const unsigned long long*)&ctl->ticket >= count &&
        *(volatile const unsigned long long*)&ctl->active <= handoff)
      atomicOr(&gc.flag, FLAG_HANDOFF);
    gsync<G>(gi);
  }
}

// tier 1 (GLOBAL_RING = false): shared-memory ring of W entries per group,
// over the contiguous ids [0, count).  tier 2 (GLOBAL_RING = true): ring of W
// entries per group slot in global memory, over a list of failed ids.
template <int G, bool GLOBAL_RING>
__global__ void __launch_bounds__(G, (G >= 1024 ? 1 : (G >= 512 ? 2 : 6))) ic_group_kernel(GraphView g, uint64_t seed, RoundView R,
                                                                        uint64_t count,
                                                                        const uint32_t* __restrict__ ids,
                                                                        uint32_t W, SampleCtl* ctl,
                                                                        uint32_t* retry_out, uint32_t* gring,
                                                                        uint32_t tier, uint32_t handoff) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int gi = threadIdx.x / G, gtid = threadIdx.x % G;
  const size_t per_group = sizeof(GroupCtl) + sizeof(GroupRows<G>) + 4 * LIVE_CAP + (GLOBAL_RING ? 0 : (size_t)20 * W);
  unsigned char* base = smem_raw + (size_t)gi * per_group;
  GroupCtl& gc = *reinterpret_cast<GroupCtl*>(base);
  GroupRows<G>& rw = *reinterpret_cast<GroupRows<G>*>(base + sizeof(GroupCtl));
  const uint64_t slot = (uint64_t)blockIdx.x * (blockDim.x / G) + gi;
  unsigned char* dyn = base + sizeof(GroupCtl) + sizeof(GroupRows<G>);
  uint32_t* live_v = reinterpret_cast<uint32_t*>(dyn);
  dyn += 4 * LIVE_CAP;
  uint32_t* ring = GLOBAL_RING ? gring + slot * (uint64_t)W : reinterpret_cast<uint32_t*>(dyn);
  RingRows rows_smem;
  if (!GLOBAL_RING) {  // tier 1: ring + prefetched rows in shared memory
    rows_smem.e0 = reinterpret_cast<unsigned long long*>(dyn + 4ull * W);
    rows_smem.d = reinterpret_cast<uint32_t*>(dyn + 12ull * W);
    rows_smem.T = reinterpret_cast<uint32_t*>(dyn + 16ull * W);
  }
  const RingRows* rr = GLOBAL_RING ? nullptr : &rows_smem;
  const PhiloxKey& K = R.K;
  unsigned long long edges_acc = 0;
  for (;;) {
    if (gtid == 0) {
      // cancelled or paused: take no new id (a resumed launch continues the ticket)
      const volatile unsigned int* cp = R.cancel;
      bool stop = cp[0] || cp[1];
      unsigned long long t = 0;
      if (!stop) {
        t = atomicAdd(&ctl->ticket, 1ull);
        stop = t >= count;
      }
      gc.s_local = stop ? 0xFFFFFFFFu : (ids ? ids[t] : (uint32_t)t);
      if (!stop) atomicAdd(&ctl->active, 1ull);
    }
    gsync<G>(gi);
    const uint32_t s_local = gc.s_local;
    if (s_local == 0xFFFFFFFFu) break;
    unsigned long long se = 0;
    uint32_t size = 0;
    const uint32_t flag = ic_group_sample<G, IC_U>(g, K, R, s_local, tier, ring, W, rr, live_v, rw, gc, gtid, gi, se,
                                                       size, ctl, count, handoff);
    if (gtid == 0) {
      if (flag == 0) {
        R.sizes[s_local] = size;
      } else if (flag & FLAG_TABLE) {
        atomicOr(reinterpret_cast<unsigned int*>(&ctl->arena_fail), 1u);  // table too full: host redoes the round
      } else if (flag & (FLAG_RING | FLAG_HANDOFF)) {
        R.failed[s_local] = (uint8_t)(tier + 1);  // the next attempt's keys will be the members
        retry_out[atomicAdd(&ctl->retry_count, 1ull)] = s_local;
      }
      atomicAdd(&ctl->active, ~0ull);  // -1
    }
    if (flag == 0) {
      edges_acc += se;
      unsigned long long ws = se;
      for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(FULL, ws, o);
      if ((threadIdx.x & 31) == 0 && ws) atomicAdd(&R.edges[s_local], ws);
    }
    gsync<G>(gi);
  }
  for (int o = 16; o > 0; o >>= 1) edges_acc += __shfl_xor_sync(FULL, edges_acc, o);
  if ((threadIdx.x & 31) == 0 && edges_acc) atomicAdd(&ctl->edges, edges_acc);
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
    const volatile unsigned int* cp = R.cancel;
    if (cp[0] || cp[1]) break;  // cancelled or paused
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
      R.edges[s_local] = steps;
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
                               uint64_t set_index0, uint32_t use, uint32_t* __restrict__ fill,
                               uint32_t* __restrict__ arena, uint32_t* __restrict__ C) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nslots; i += stride) {
    const unsigned long long k = keys[i];
    if (k == 0ull) continue;
    const uint32_t hi = (uint32_t)(k >> 32);
    const uint32_t tier = hi >> 30;
    const uint32_t s_local = (hi & 0x3FFFFFFFu) - 1u;
    if (s_local >= use) continue;                // speculative samples beyond the ones kept
    if (tier != failed[s_local]) continue;       // an abandoned attempt of a sample that was redone
    const uint32_t v = (uint32_t)k;
    const uint32_t p = atomicAdd(&fill[s_local], 1u);
    arena[set_start[set_index0 + s_local] + p] = v;
    if (C) atomicAdd(&C[v], 1u);
  }
}

constexpr uint32_t IC_W = 1024;    // shared-memory frontier ring per group
constexpr int IC_G2 = 1024;        // tier 2: a whole SM per sample (tail hand-off and ring overflow)
constexpr uint32_t IC_W2 = 4096;   // tier-2 shared-memory ring
constexpr int IC_G3 = 512;         // tier 3: global ring of capacity >= n (never fails)

template <int G, bool GR>
size_t ic_smem_per_group(uint32_t W) {
  return sizeof(GroupCtl) + sizeof(GroupRows<G>) + 4 * LIVE_CAP + (GR ? 0 : (size_t)20 * W);
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

void round_release(Round& rd) {
  DevBuf* b[] = {&rd.table, &rd.sizes, &rd.failed, &rd.edges, &rd.fill, &rd.retry, &rd.excl, &rd.ctl};
  for (DevBuf* x : b) x->release();
  for (cudaEvent_t& e : rd.ev) {
    if (e) cudaEventDestroy(e);
    e = nullptr;
  }
  rd.launched = false;
}

template <int G, bool GR>
static void launch_ic(eim_ctx* ctx, const eim_graph* g, uint64_t seed, const RoundView& R, uint64_t count,
                      const uint32_t* ids, uint32_t W, SampleCtl* ctl, uint32_t* retry_out, uint32_t* gring,
                      uint64_t max_blocks, cudaStream_t st, bool spare_sm_slot, uint32_t tier, uint32_t handoff) {
  const size_t smem = ic_smem_per_group<G, GR>(W);
  auto kern = ic_group_kernel<G, GR>;
  EIM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 0;
  EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, G, smem));
  if (per_sm < 1) fail(EIM_E_CUDA, "sampler tier does not fit on an SM");
  if (spare_sm_slot && per_sm > 1) per_sm -= 1;
  uint64_t blocks = (uint64_t)per_sm * ctx->sm_count;
  blocks = std::max<uint64_t>(1, std::min<uint64_t>(std::min<uint64_t>(blocks, count), max_blocks));
  kern<<<(uint32_t)blocks, G, smem, st>>>(g->view, seed, R, count, ids, W, ctl, retry_out, gring, tier, handoff);
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches++;
}

// Tail hand-off threshold of tier 1 (samples still running when the launch
// has no ids left), off by default: measured on C2 it did not shorten the
// rounds (a restarted chain costs about what it had left).  EIM_HANDOFF=<n>
// enables it for experiments.
static uint32_t handoff_threshold(eim_ctx*) {
  const char* e = std::getenv("EIM_HANDOFF");
  return e ? (uint32_t)std::atoi(e) : 0u;
}

static RoundView round_view(Round& rd) {
  return RoundView{rd.table.as<unsigned long long>(), rd.bits, rd.sizes.as<uint32_t>(), rd.failed.as<uint8_t>(),
                   rd.edges.as<unsigned long long>(),
                   reinterpret_cast<const unsigned int*>(rd.ctl.as<SampleCtl>() + 1), rd.first,
                   philox_key(rd.seed)};
}

// one tier-1 sampler launch over rd's remaining ids, bracketed by events
static void round_kernel(eim_ctx* ctx, const eim_graph* g, Round& rd, cudaStream_t st, bool spare_sm_slot) {
  if (rd.nlaunch >= Round::MAX_LAUNCH) fail(EIM_E_STATE, "too many sampler launches in one round");
  SampleCtl* ctl = rd.ctl.as<SampleCtl>();
  const RoundView R = round_view(rd);
  EIM_CUDA(cudaEventRecord(rd.ev[2 * rd.nlaunch], st));
  if (rd.model == EIM_IC) {
    launch_ic<IC_G, false>(ctx, g, rd.seed, R, rd.count, nullptr, IC_W, ctl, rd.retry.as<uint32_t>(), nullptr,
                           ~0ull, st, spare_sm_slot, 0, handoff_threshold(ctx));
  } else {
    int per_sm = 0;
    EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lt_kernel, 256, 0));
    if (spare_sm_slot && per_sm > 1) per_sm -= 1;
    uint64_t blocks = std::min<uint64_t>((uint64_t)std::max(1, per_sm) * ctx->sm_count, (rd.count + 255) / 256);
    lt_kernel<<<(uint32_t)std::max<uint64_t>(blocks, 1), 256, 0, st>>>(g->view, rd.seed, R, rd.count, ctl);
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
  }
  EIM_CUDA(cudaEventRecord(rd.ev[2 * rd.nlaunch + 1], st));
  rd.nlaunch++;
  rd.stream = st;
  rd.launched = true;
}

// memsets + first tier-1 launch of rd's range on stream st
static void round_start(eim_ctx* ctx, const eim_graph* g, Round& rd, cudaStream_t st, bool spare_sm_slot) {
  const uint64_t count = rd.count;
  rd.table.reserve(8ull << rd.bits, false, st);
  EIM_CUDA(cudaMemsetAsync(rd.table.p, 0, 8ull << rd.bits, st));
  EIM_CUDA(cudaMemsetAsync(rd.failed.p, 0, count, st));
  EIM_CUDA(cudaMemsetAsync(rd.sizes.p, 0, count * sizeof(uint32_t), st));
  EIM_CUDA(cudaMemsetAsync(rd.edges.p, 0, count * sizeof(unsigned long long), st));
  EIM_CUDA(cudaMemsetAsync(rd.ctl.p, 0, sizeof(SampleCtl) + 16, st));
  rd.nlaunch = 0;
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
                  uint64_t count, uint64_t set_base, bool hist, Round& rd, cudaStream_t st, bool spare_sm_slot) {
  if (count == 0) return;
  if (count >= 0x3FFFFFF0ull) fail(EIM_E_INVAL, "at most 2^30 sets per sampler launch");
  if (!rd.ev[0])
    for (cudaEvent_t& e : rd.ev) EIM_CUDA(cudaEventCreate(&e));
  rd.first = first;
  rd.count = count;
  rd.set_base = set_base;
  rd.seed = seed;
  rd.model = model;
  rd.hist = hist;
  rd.sizes.reserve(count * sizeof(uint32_t), false, st);
  rd.failed.reserve(count, false, st);
  rd.edges.reserve(count * sizeof(unsigned long long), false, st);
  rd.fill.reserve(count * sizeof(uint32_t), false, st);
  rd.retry.reserve(2 * count * sizeof(uint32_t), false, st);  // two retry lists (tier 1 -> 2 -> 3)
  rd.excl.reserve((count + 1) * sizeof(uint64_t), false, st);
  rd.ctl.reserve(sizeof(SampleCtl) + 16, false, st);
  // table capacity: >= 4x the expected members (mean set size of earlier
  // rounds, else 64), at least 2^20 slots
  const double mean = ctx->est_mean_size > 0 ? ctx->est_mean_size : 64.0;
  uint32_t bits = 20;
  while (bits < 31 && (double)(1ull << bits) < 4.0 * mean * (double)count) bits++;
  rd.bits = bits;
  round_start(ctx, g, rd, st, spare_sm_slot);
}

void round_cancel(eim_ctx* ctx, Round& rd) {
  if (!rd.launched) return;
  EIM_CUDA(cudaMemsetAsync(round_flags(rd), 0xFF, sizeof(unsigned int), ctx->aux_stream));
  EIM_CUDA(cudaStreamSynchronize(ctx->aux_stream));
  EIM_CUDA(cudaStreamSynchronize(rd.stream));
  rd.launched = false;
}

SampleResult round_finalize(eim_ctx* ctx, const eim_graph* g, Round& rd, uint64_t use) {
  SampleResult res;
  if (!rd.launched || rd.count == 0) return res;
  if (use > rd.count) fail(EIM_E_STATE, "round_finalize beyond the launched range");
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
  for (int attempt = 0;; ++attempt) {
    int counted = 0;
    for (;;) {  // until the tier-1 launches have taken every id (a paused round is resumed here)
      EIM_CUDA(cudaStreamWaitEvent(st, rd.ev[2 * rd.nlaunch - 1], 0));
      EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl), cudaMemcpyDeviceToHost, st));
      EIM_CUDA(cudaStreamSynchronize(st));
      if (h->ticket >= rd.count || h->arena_fail) break;
      round_resume(ctx, g, rd, st);
    }
    res.kernel_ms += elapsed(counted);
    res.launches += rd.nlaunch - counted;
    counted = rd.nlaunch;
    bool table_full = h->arena_fail != 0;
    // retry tiers over the ids a tier gave up: tier 2 = a whole SM (1024
    // threads) per sample with a larger shared-memory ring (the long chains
    // handed off by tier 1, and ring overflows); tier 3 = global-memory ring
    // of capacity >= n, which cannot overflow
    uint32_t* lists[2] = {rd.retry.as<uint32_t>(), rd.retry.as<uint32_t>() + rd.count};
    if (!table_full && h->retry_count > 0)  // a pause that arrived after the last id was taken
      EIM_CUDA(cudaMemsetAsync(round_flags(rd) + 1, 0, sizeof(unsigned int), st));
    for (uint32_t tier = 1; !table_full && h->retry_count > 0; ++tier) {
      if (tier > 2) fail(EIM_E_CUDA, "tier-3 sampler failed with a ring of capacity n");
      const uint64_t nretry = h->retry_count;
      res.tier2 += nretry;
      uint32_t* in = lists[(tier - 1) & 1];
      uint32_t* out = lists[tier & 1];
      EIM_CUDA(cudaMemsetAsync(ctl, 0, sizeof(SampleCtl), st));
      if (rd.nlaunch >= Round::MAX_LAUNCH) fail(EIM_E_STATE, "too many sampler launches in one round");
      EIM_CUDA(cudaEventRecord(rd.ev[2 * rd.nlaunch], st));
      if (tier == 1) {
        launch_ic<IC_G2, false>(ctx, g, rd.seed, round_view(rd), nretry, in, IC_W2, ctl, out, nullptr,
                                ctx->sm_count, st, false, 1, 0);
      } else {
        uint32_t W3 = 1;
        while (W3 < g->view.n) W3 <<= 1;
        uint64_t slots = std::min<uint64_t>(nretry, std::max<uint64_t>(1, (1ull << 30) / (4ull * W3)));
        slots = std::min<uint64_t>(slots, (uint64_t)ctx->sm_count);
        ctx->tier_queue.reserve(slots * (uint64_t)W3 * 4, false, st);
        launch_ic<IC_G3, true>(ctx, g, rd.seed, round_view(rd), nretry, in, W3, ctl, out,
                               ctx->tier_queue.as<uint32_t>(), slots, st, false, 2, 0);
      }
      EIM_CUDA(cudaEventRecord(rd.ev[2 * rd.nlaunch + 1], st));
      rd.nlaunch++;
      EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl), cudaMemcpyDeviceToHost, st));
      EIM_CUDA(cudaStreamSynchronize(st));
      res.kernel_ms += elapsed(counted);
      res.launches += rd.nlaunch - counted;
      counted = rd.nlaunch;
      table_full = h->arena_fail != 0;
    }
    if (table_full) {  // rare: redo the whole range with a 4x larger table
      if (attempt >= 4 || rd.bits >= 31) fail(EIM_E_NOMEM, "membership table overflow");
      rd.bits += 2;
      round_start(ctx, g, rd, st, false);
      continue;
    }
    break;
  }
  rd.launched = false;
  if (use == 0) return res;
  // ---- sizes -> offsets (sample-id order) -> arena placement -> scatter + histogram
  unsigned long long* d_cursor = reinterpret_cast<unsigned long long*>(ctx->ctl.as<SampleCtl>() + 1);
  unsigned long long* h_cursor = reinterpret_cast<unsigned long long*>(h + 1);
  uint64_t* excl = rd.excl.as<uint64_t>();
  ensure_sets(ctx, rd.first + use - rd.set_base);
  sizes_to_offsets_kernel<<<grid_for(ctx, use + 1, 256), 256, 0, st>>>(rd.sizes.as<uint32_t>(), use, excl);
  EIM_CUDA(cudaGetLastError());
  size_t tmp = 0, tmp2 = 0;
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, excl, excl, use + 1, st));
  unsigned long long* d_edges_sum = reinterpret_cast<unsigned long long*>(ctl) + 2;  // retry_count slot, unused now
  EIM_CUDA(cub::DeviceReduce::Sum(nullptr, tmp2, rd.edges.as<unsigned long long>(), d_edges_sum, use, st));
  ctx->scratch.reserve(std::max<size_t>(std::max(tmp, tmp2), 1 << 20), false, st);
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(ctx->scratch.p, tmp, excl, excl, use + 1, st));
  EIM_CUDA(cub::DeviceReduce::Sum(ctx->scratch.p, tmp2, rd.edges.as<unsigned long long>(), d_edges_sum, use, st));
  EIM_CUDA(cudaMemcpyAsync(&h->ticket, excl + use, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaMemcpyAsync(&h->edges, d_edges_sum, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaMemcpyAsync(h_cursor, d_cursor, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  const uint64_t total = h->ticket, cursor = h_cursor[0];
  res.edges = h->edges;
  ctx->arena.reserve((cursor + total) * sizeof(uint32_t), true, st);
  const uint64_t set_index0 = rd.first - rd.set_base;
  place_sets_kernel<<<grid_for(ctx, use, 256), 256, 0, st>>>(excl, rd.sizes.as<uint32_t>(), use, cursor, set_index0,
                                                              ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>());
  EIM_CUDA(cudaGetLastError());
  EIM_CUDA(cudaMemsetAsync(rd.fill.p, 0, use * sizeof(uint32_t), st));
  const uint64_t nslots = 1ull << rd.bits;
  scatter_kernel<<<grid_for(ctx, nslots, 256), 256, 0, st>>>(
      rd.table.as<unsigned long long>(), nslots, rd.failed.as<uint8_t>(), ctx->set_start.as<uint64_t>(), set_index0,
      (uint32_t)use, rd.fill.as<uint32_t>(), ctx->arena.as<uint32_t>(),
      rd.hist ? ctx->C_total.as<uint32_t>() : nullptr);
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches += 6;
  h_cursor[0] = cursor + total;
  h_cursor[1] = cursor + total;
  EIM_CUDA(cudaMemcpyAsync(d_cursor, h_cursor, 2 * sizeof(uint64_t), cudaMemcpyHostToDevice, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  ctx->est_mean_size = std::max(1.0, (double)total / (double)use);
  return res;
}

SampleResult sample_range(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed,
                          uint64_t first, uint64_t count, uint64_t set_base, bool hist) {
  if (count == 0) return SampleResult{};
  Round& rd = ctx->rounds[0];
  round_launch(ctx, g, model, seed, first, count, set_base, hist, rd, ctx->stream, false);
  return round_finalize(ctx, g, rd, count);
}

}  // namespace eim
