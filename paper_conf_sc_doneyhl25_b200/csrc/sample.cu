// sample.cu -- RRR-set samplers (Alg. 2, P:107 for IC; P:134-140 for LT).
//
// IC, tier 1 (ic_tier1): one warp per sample id (ids handed out by a launch
//   ticket).  The BFS queue Q and an open-addressing visited hash
//   live in shared memory.  The frontier is expanded in batches of up to 32
//   queued vertices: their in-rows are merged into one space of Philox quads
//   (4 consecutive edge ids share one Philox4x32-10 call, reading R1), and
//   the 32 lanes sweep that space, so small rows do not idle the warp and a
//   hub row is split evenly.  An edge into u is live iff its draw <= T_u
//   (R2).  in_nbr[e] is read only for live edges.  Newly visited vertices are
//   appended with a warp ballot (no atomics on the queue tail).  A set that
//   outgrows the shared-memory queue is abandoned and its id is pushed onto
//   a retry list: the keyed randomness makes the redo exact.
// IC, tier k >= 2 (ic_tierk): the same warp routine with the hash and queue
//   in global memory (generation-tagged 64-bit slots, so no clearing), with
//   capacities growing x16 per tier until they cover n.
// LT, tier 1 (lt_tier1): one thread per reverse walk (the walk is
//   sequential); the path lives in shared memory and is also the
//   visited set.  Tier k: path + generation hash in global memory.
// Every finished set reserves its arena range with one atomic (the arena is
// append-only; set i is (set_start[i], set_len[i])) and bumps the coverage
// histogram C (Alg. 2 l.25).  Member order inside a set is not canonical;
// eim_sample_rrr sorts on export.
#include <cub/cub.cuh>

#include "eim_internal.h"
#include "philox.cuh"

namespace eim {

namespace {

constexpr unsigned FULL = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t hash_slot(uint32_t v, uint32_t bits) {
  return (v * 0x9E3779B1u) >> (32u - bits);
}

// Shared-memory visited table: u32 slots holding v+1 (0 = empty).
struct SmemTable {
  uint32_t* h;
  uint32_t bits;
  __device__ __forceinline__ bool insert(uint32_t v) const {
    const uint32_t key = v + 1u, mask = (1u << bits) - 1u;
    uint32_t i = hash_slot(v, bits);
    for (;;) {
      uint32_t old = atomicCAS(&h[i], 0u, key);
      if (old == 0u) return true;
      if (old == key) return false;
      i = (i + 1u) & mask;
    }
  }
  __device__ __forceinline__ void clear(int lane) const {
    uint4* p = reinterpret_cast<uint4*>(h);
    for (uint32_t i = lane; i < (1u << bits) / 4u; i += 32u) p[i] = make_uint4(0, 0, 0, 0);
  }
};

// Global-memory visited table: 64-bit slots (gen << 32 | v+1); a slot whose
// generation differs from the current sample's is free.
struct GenTable {
  unsigned long long* h;
  uint32_t bits;
  uint32_t gen;
  __device__ __forceinline__ bool insert(uint32_t v) const {
    const unsigned long long want = ((unsigned long long)gen << 32) | (unsigned long long)(v + 1u);
    const uint32_t mask = (1u << bits) - 1u;
    uint32_t i = hash_slot(v, bits);
    unsigned long long cur = __ldcg(&h[i]);
    for (;;) {
      if ((uint32_t)(cur >> 32) != gen) {
        unsigned long long prev = atomicCAS(&h[i], cur, want);
        if (prev == cur) return true;
        cur = prev;
        continue;
      }
      if (cur == want) return false;
      i = (i + 1u) & mask;
      cur = __ldcg(&h[i]);
    }
  }
};

// Group barrier: a warp uses __syncwarp, larger groups a named barrier
// (ids 1..15; id 0 is __syncthreads).
template <int G>
__device__ __forceinline__ void gsync(int gi) {
  if constexpr (G == 32) {
    __syncwarp();
  } else {
    asm volatile("bar.sync %0, %1;" ::"r"(gi + 1), "r"(G) : "memory");
  }
}

// Per-group control block and frontier-batch row descriptors (shared memory).
struct GroupCtl {
  uint32_t tail, flag, gen, pad;
  unsigned long long s, start;
  uint32_t wsum[16];
  uint32_t pad2[8];
};
template <int G>
struct GroupRows {
  unsigned long long q0[G];  // first Philox quad of the row
  uint32_t qend[G];          // inclusive scan of quad counts
  uint32_t nq[G];            // quads of the row
  uint32_t T[G];             // IC threshold of the row's vertex
  uint8_t wlo[G], whi[G];    // first / last valid word in the first / last quad
};

template <int G>
__device__ __forceinline__ uint32_t group_incl_scan(uint32_t x, int gtid, int gi, GroupCtl& gc,
                                                    uint32_t& total) {
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

// One IC RRR set by a group of G threads (Alg. 2 l.5-20).  The queue Q is
// also the member list.  Frontier batches of up to G queued vertices have
// their rows merged into one quad space swept by the whole group; there is no
// per-level barrier beyond one per batch.  Returns false when the set
// outgrows qcap or (cap_quads > 0) the sample exceeds cap_quads Philox quads:
// the caller then re-queues the id for a larger tier.
template <int G, class Tab>
__device__ __forceinline__ bool ic_group_sample(const GraphView& g, const PhiloxKey& K, uint64_t s,
                                                const Tab& tab, uint32_t* queue, uint32_t qcap,
                                                GroupRows<G>& rw, GroupCtl& gc, int gtid, int gi,
                                                uint32_t cap_quads, unsigned long long& se) {
  if (gtid == 0) {
    const uint32_t root = draw_root(s, g.n, K);
    tab.insert(root);
    queue[0] = root;
    gc.tail = 1;
    gc.flag = 0;
  }
  gsync<G>(gi);
  uint32_t head = 0, quads_done = 0;
  se = 0;
  for (;;) {
    const uint32_t tail = *(volatile uint32_t*)&gc.tail;
    const uint32_t flag = *(volatile uint32_t*)&gc.flag;
    if (flag || head >= tail) return flag == 0;
    const uint32_t nb = min((uint32_t)G, tail - head);
    uint32_t nq = 0;
    if (gtid < nb) {
      const uint32_t u = queue[head + gtid];
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
    gsync<G>(gi);
    head += nb;
    quads_done += total;
    if (cap_quads && quads_done > cap_quads) {
      gsync<G>(gi);  // everyone is past the reads of this batch's control words
      return false;
    }
    int r = -1;
    uint32_t qe = 0, qb = 0, nq_r = 0, T_r = 0, wlo_r = 0, whi_r = 0;
    unsigned long long q0_r = 0;
    for (uint32_t base = 0; base < total; base += G) {
      const uint32_t j = base + gtid;
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
        const unsigned long long q = q0_r + li;
        const uint4 w = philox_at(q, s, TAG_EDGE, K);
        uint32_t m = 0xFu;
        if (li == 0) m &= 0xFu << wlo_r;
        if (li == nq_r - 1) m &= 0xFu >> (3u - whi_r);
        uint32_t live = (w.x <= T_r ? 1u : 0u) | (w.y <= T_r ? 2u : 0u) | (w.z <= T_r ? 4u : 0u) |
                        (w.w <= T_r ? 8u : 0u);
        live &= m;
        while (live) {
          const int i = __ffs(live) - 1;
          live &= live - 1;
          const uint32_t v = g.nbr[(q << 2) + i];
          if (*(volatile uint32_t*)&gc.tail >= qcap) {
            gc.flag = 1;
          } else if (tab.insert(v)) {
            const uint32_t pos = atomicAdd(&gc.tail, 1u);
            if (pos < qcap) queue[pos] = v;
            else gc.flag = 1;
          }
        }
      }
    }
    gsync<G>(gi);
  }
}

// Group-cooperative IC sampler.  GLOBAL = false: hash + queue in shared
// memory (tiers 1 and 2); GLOBAL = true: generation-tagged hash + queue in
// global memory, one slot per group (last tiers, capacity up to n).
template <int G, bool GLOBAL>
__global__ void __launch_bounds__(512) ic_group_kernel(GraphView g, uint64_t seed, uint64_t first, uint64_t count,
                                                       const unsigned long long* ids, ArenaView A, SampleCtl* ctl,
                                                       unsigned long long* retry_out, uint32_t hbits, uint32_t qcap,
                                                       uint32_t cap_quads, unsigned long long* gtabs,
                                                       uint32_t* gqueues, uint32_t* gens) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int gi = threadIdx.x / G, gtid = threadIdx.x % G;
  const size_t tab_bytes = GLOBAL ? 0 : ((size_t)4 << hbits) + (size_t)4 * qcap;
  unsigned char* base = smem_raw + (size_t)gi * (sizeof(GroupCtl) + sizeof(GroupRows<G>) + tab_bytes);
  GroupCtl& gc = *reinterpret_cast<GroupCtl*>(base);
  GroupRows<G>& rw = *reinterpret_cast<GroupRows<G>*>(base + sizeof(GroupCtl));
  const uint64_t slot = (uint64_t)blockIdx.x * (blockDim.x / G) + gi;
  uint32_t* queue;
  SmemTable stab{nullptr, hbits};
  unsigned long long* gh = nullptr;
  if constexpr (GLOBAL) {
    gh = gtabs + (slot << hbits);
    queue = gqueues + slot * (uint64_t)qcap;
  } else {
    stab.h = reinterpret_cast<uint32_t*>(base + sizeof(GroupCtl) + sizeof(GroupRows<G>));
    queue = stab.h + (1u << hbits);
    for (uint32_t i = gtid; i < (1u << hbits) / 4u; i += G) reinterpret_cast<uint4*>(stab.h)[i] = make_uint4(0, 0, 0, 0);
  }
  const PhiloxKey K = philox_key(seed);
  unsigned long long edges_acc = 0;
  gsync<G>(gi);
  for (;;) {
    if (gtid == 0) {
      gc.s = atomicAdd(&ctl->ticket, 1ull);
      if constexpr (GLOBAL) {
        uint32_t gen = gens[slot] + 1u;
        if (gen == 0u) gen = 1u;
        gens[slot] = gen;
        gc.gen = gen;
      }
    }
    gsync<G>(gi);
    const unsigned long long t = gc.s;
    if (t >= count) break;
    const uint64_t s = ids ? ids[t] : first + t;
    unsigned long long se = 0;
    bool ok;
    if constexpr (GLOBAL) {
      const uint32_t gen = gc.gen;
      if (gen == 1u) {  // fresh (or wrapped) generation counter: clear this slot's table once
        for (uint64_t i = gtid; i < (1ull << hbits); i += G) gh[i] = 0ull;
        __threadfence_block();
        gsync<G>(gi);
      }
      GenTable tab{gh, hbits, gen};
      ok = ic_group_sample<G>(g, K, s, tab, queue, qcap, rw, gc, gtid, gi, cap_quads, se);
    } else {
      ok = ic_group_sample<G>(g, K, s, stab, queue, qcap, rw, gc, gtid, gi, cap_quads, se);
    }
    const uint32_t size = gc.tail;
    if (gtid == 0) {
      unsigned long long start = ~0ull;
      if (ok) {
        const unsigned long long st = atomicAdd(A.cursor, (unsigned long long)size);
        if (st + size <= A.cap) {
          start = st;
          A.set_start[s - A.set_base] = st;
          A.set_len[s - A.set_base] = size;
          atomicMax(A.valid_end, st + size);
        } else {
          atomicAdd(&ctl->arena_fail, 1ull);
        }
      }
      if (start == ~0ull) retry_out[atomicAdd(&ctl->retry_count, 1ull)] = s;
      gc.start = start;
    }
    gsync<G>(gi);
    const unsigned long long start = gc.start;
    if (start != ~0ull) {
      for (uint32_t i = gtid; i < size; i += G) {
        const uint32_t v = queue[i];
        A.elems[start + i] = v;
        if (A.C) atomicAdd(&A.C[v], 1u);
      }
      edges_acc += se;
    }
    if constexpr (!GLOBAL) {
      for (uint32_t i = gtid; i < (1u << hbits) / 4u; i += G) reinterpret_cast<uint4*>(stab.h)[i] = make_uint4(0, 0, 0, 0);
    }
    gsync<G>(gi);
  }
  // per-thread examined-edge sums
  for (int o = 16; o > 0; o >>= 1) edges_acc += __shfl_xor_sync(FULL, edges_acc, o);
  if ((threadIdx.x & 31) == 0 && edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

// ---------------------------------------------------------------- LT
// Reverse LT walk (R3-R5): at u with d^-(u) > 0, tau_u is the
// LT-tagged draw of u and the chosen in-neighbour is position
// floor(tau * d / 2^32) of u's row (the prefix-scan choice under WC weights);
// the walk stops when d^-(u) = 0 or the chosen vertex is already in the set.
__device__ __forceinline__ uint32_t lt_next(const GraphView& g, const PhiloxKey& K, uint64_t s,
                                            uint32_t u, bool& has) {
  const unsigned long long e0 = g.off[u], e1 = g.off[u + 1];
  if (e1 == e0) {
    has = false;
    return 0;
  }
  has = true;
  const uint4 w = philox_at((uint64_t)(u >> 2), s, TAG_LT, K);
  const uint32_t tau = word_of(w, u & 3u);
  const unsigned long long j = __umul64hi((unsigned long long)tau << 32, e1 - e0);
  return g.nbr[e0 + j];
}

__device__ __forceinline__ void lt_commit(const ArenaView& A, SampleCtl* ctl, unsigned long long* retry_out,
                                          uint64_t s, bool ok, uint32_t L, const uint32_t* path,
                                          uint32_t stride, unsigned long long steps,
                                          unsigned long long& edges_acc) {
  bool fail = !ok;
  if (ok) {
    unsigned long long start = atomicAdd(A.cursor, (unsigned long long)L);
    if (start + L <= A.cap) {
      for (uint32_t i = 0; i < L; ++i) {
        uint32_t v = path[(size_t)i * stride];
        A.elems[start + i] = v;
        if (A.C) atomicAdd(&A.C[v], 1u);
      }
      A.set_start[s - A.set_base] = start;
      A.set_len[s - A.set_base] = L;
      atomicMax(A.valid_end, start + L);
      edges_acc += steps;
    } else {
      fail = true;
      atomicAdd(&ctl->arena_fail, 1ull);
    }
  }
  if (fail) {
    unsigned long long p = atomicAdd(&ctl->retry_count, 1ull);
    retry_out[p] = s;
  }
}

template <int P>
__global__ void __launch_bounds__(128) lt_tier1_kernel(GraphView g, uint64_t seed, uint64_t first,
                                                       uint64_t count, const unsigned long long* ids,
                                                       ArenaView A, SampleCtl* ctl,
                                                       unsigned long long* retry_out) {
  extern __shared__ __align__(16) uint32_t path_smem[];
  uint32_t* path = path_smem + threadIdx.x;  // [i * blockDim + tid]
  const uint32_t stride = blockDim.x;
  const PhiloxKey K = philox_key(seed);
  unsigned long long edges_acc = 0;
  for (;;) {
    const unsigned long long t = atomicAdd(&ctl->ticket, 1ull);
    if (t >= count) break;
    const uint64_t s = ids ? ids[t] : first + t;
    uint32_t u = draw_root(s, g.n, K);
    path[0] = u;
    uint32_t L = 1;
    unsigned long long steps = 0;
    bool ok = true;
    for (;;) {
      bool has;
      const uint32_t v = lt_next(g, K, s, u, has);
      if (!has) break;
      ++steps;
      bool seen = false;
      for (uint32_t i = 0; i < L; ++i) seen |= (path[i * stride] == v);
      if (seen) break;
      if (L == P) {
        ok = false;
        break;
      }
      path[L * stride] = v;
      ++L;
      u = v;
    }
    lt_commit(A, ctl, retry_out, s, ok, L, path, stride, steps, edges_acc);
  }
  if (edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

__global__ void __launch_bounds__(128) lt_tierk_kernel(GraphView g, uint64_t seed, uint64_t count,
                                                       const unsigned long long* ids, ArenaView A,
                                                       SampleCtl* ctl, unsigned long long* retry_out,
                                                       unsigned long long* tabs, uint32_t tbits,
                                                       uint32_t* queues, uint32_t qcap, uint32_t* gens) {
  const uint64_t slot = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long* h = tabs + (slot << tbits);
  uint32_t* path = queues + slot * (uint64_t)qcap;
  const PhiloxKey K = philox_key(seed);
  unsigned long long edges_acc = 0;
  for (;;) {
    const unsigned long long t = atomicAdd(&ctl->ticket, 1ull);
    if (t >= count) break;
    const uint64_t s = ids[t];
    uint32_t gen = gens[slot] + 1u;
    if (gen == 0u) gen = 1u;
    gens[slot] = gen;
    if (gen == 1u)
      for (uint64_t i = 0; i < (1ull << tbits); ++i) h[i] = 0ull;
    GenTable tab{h, tbits, gen};
    uint32_t u = draw_root(s, g.n, K);
    tab.insert(u);
    path[0] = u;
    uint32_t L = 1;
    unsigned long long steps = 0;
    bool ok = true;
    for (;;) {
      bool has;
      const uint32_t v = lt_next(g, K, s, u, has);
      if (!has) break;
      ++steps;
      if (!tab.insert(v)) break;
      if (L == qcap) {
        ok = false;
        break;
      }
      path[L++] = v;
      u = v;
    }
    lt_commit(A, ctl, retry_out, s, ok, L, path, 1, steps, edges_acc);
  }
  if (edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

constexpr int LT_P = 64;                          // path capacity per walker (tier 1)
constexpr int LT_THREADS = 128;

// IC tier table: group size, groups per block, log2 hash slots, queue capacity, work cap.
struct IcTier {
  int G, NG;
  uint32_t hbits, qcap, cap_quads;
  bool global;
};
constexpr IcTier IC_T1{32, 8, 9, 256, 2048, false};     // warp per sample, light samples
constexpr IcTier IC_T2{128, 4, 12, 2048, 0, false};     // 4 warps per sample, heavy samples

template <int G, bool GLOBAL>
size_t ic_smem_per_group(uint32_t hbits, uint32_t qcap) {
  return sizeof(GroupCtl) + sizeof(GroupRows<G>) + (GLOBAL ? 0 : ((size_t)4 << hbits) + (size_t)4 * qcap);
}

}  // namespace

// ------------------------------------------------------------------ host
void arena_reset(eim_ctx* ctx) {
  ctx->arena.reserve(sizeof(uint32_t) * (1u << 22), false, ctx->stream);
  ctx->ctl.reserve(sizeof(SampleCtl) + 2 * sizeof(unsigned long long), false, ctx->stream);
  // ctl layout: [SampleCtl][cursor][valid_end]
  EIM_CUDA(cudaMemsetAsync(ctx->ctl.p, 0, sizeof(SampleCtl) + 2 * sizeof(unsigned long long), ctx->stream));
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

static ArenaView arena_view(eim_ctx* ctx, uint64_t set_base, bool hist) {
  ArenaView A;
  unsigned long long* tail = reinterpret_cast<unsigned long long*>(ctx->ctl.as<SampleCtl>() + 1);
  A.elems = ctx->arena.as<uint32_t>();
  A.cursor = tail;
  A.valid_end = tail + 1;
  A.cap = ctx->arena.bytes / sizeof(uint32_t);
  A.set_start = ctx->set_start.as<uint64_t>();
  A.set_len = ctx->set_len.as<uint32_t>();
  A.set_base = set_base;
  A.C = hist ? ctx->C_total.as<uint32_t>() : nullptr;
  return A;
}

template <int G, bool GLOBAL>
static void launch_ic(eim_ctx* ctx, const eim_graph* g, uint64_t seed, uint64_t first, uint64_t count,
                      const unsigned long long* ids, const ArenaView& A, SampleCtl* ctl,
                      unsigned long long* retry_out, uint32_t hbits, uint32_t qcap, uint32_t cap, int NG,
                      uint64_t max_groups) {
  const size_t smem = ic_smem_per_group<G, GLOBAL>(hbits, qcap) * NG;
  auto kern = ic_group_kernel<G, GLOBAL>;
  EIM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 0;
  EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, G * NG, smem));
  if (per_sm < 1) fail(EIM_E_CUDA, "sampler tier does not fit on an SM");
  uint64_t blocks = (uint64_t)per_sm * ctx->sm_count;
  blocks = std::min<uint64_t>(blocks, (count + NG - 1) / NG);
  blocks = std::min<uint64_t>(blocks, std::max<uint64_t>(1, max_groups / NG));
  blocks = std::max<uint64_t>(blocks, 1);
  unsigned long long* tabs = GLOBAL ? ctx->tier_tab.as<unsigned long long>() : nullptr;
  uint32_t* queues = GLOBAL ? ctx->tier_queue.as<uint32_t>() : nullptr;
  uint32_t* gens = GLOBAL ? ctx->tier_gen.as<uint32_t>() : nullptr;
  kern<<<(uint32_t)blocks, G * NG, smem, ctx->stream>>>(g->view, seed, first, count, ids, A, ctl, retry_out, hbits,
                                                         qcap, cap, tabs, queues, gens);
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches++;
}

SampleResult sample_range(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed,
                          uint64_t first, uint64_t count, uint64_t set_base, bool hist) {
  SampleResult res;
  if (count == 0) return res;
  cudaStream_t st = ctx->stream;
  ensure_sets(ctx, first + count - set_base);
  ctx->retry_a.reserve(count * sizeof(unsigned long long), false, st);
  ctx->retry_b.reserve(count * sizeof(unsigned long long), false, st);
  SampleCtl* ctl = ctx->ctl.as<SampleCtl>();
  unsigned long long* tail = reinterpret_cast<unsigned long long*>(ctl + 1);
  SampleCtl* h = static_cast<SampleCtl*>(ctx->h_pinned);
  unsigned long long* h_tail = reinterpret_cast<unsigned long long*>(h + 1);
  unsigned long long* retry_in = ctx->retry_a.as<unsigned long long>();
  unsigned long long* retry_out = ctx->retry_b.as<unsigned long long>();
  uint32_t nbits = 1;
  while ((1ull << nbits) < (uint64_t)g->view.n) nbits++;

  auto read_ctl = [&]() {
    EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl) + 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    res.edges += h->edges;
  };
  auto grow_if_needed = [&]() {
    if (!h->arena_fail) return;
    // successful reservations form a prefix [0, valid_end): keep it, grow, rewind the cursor
    const uint64_t valid = h_tail[1];
    const uint64_t cap = ctx->arena.bytes / sizeof(uint32_t);
    const uint64_t want = std::max<uint64_t>(cap * 2, valid * 2 + 4096ull * h->retry_count);
    ctx->arena.reserve(want * sizeof(uint32_t), true, st);
    EIM_CUDA(cudaMemcpyAsync(tail, &h_tail[1], sizeof(unsigned long long), cudaMemcpyHostToDevice, st));
  };

  // ---- tier 1 over the contiguous id range
  EIM_CUDA(cudaMemsetAsync(ctl, 0, sizeof(SampleCtl), st));
  ArenaView A = arena_view(ctx, set_base, hist);
  EIM_CUDA(cudaEventRecord(ctx->ev0, st));
  if (model == EIM_IC) {
    launch_ic<32, false>(ctx, g, seed, first, count, nullptr, A, ctl, retry_out, IC_T1.hbits, IC_T1.qcap,
                         IC_T1.cap_quads, IC_T1.NG, ~0ull);
  } else {
    const size_t smem = (size_t)LT_P * LT_THREADS * sizeof(uint32_t);
    int per_sm = 0;
    EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lt_tier1_kernel<LT_P>, LT_THREADS, smem));
    uint64_t blocks = (uint64_t)std::max(1, per_sm) * ctx->sm_count;
    blocks = std::min<uint64_t>(blocks, (count + LT_THREADS - 1) / LT_THREADS);
    lt_tier1_kernel<LT_P><<<(uint32_t)blocks, LT_THREADS, smem, st>>>(g->view, seed, first, count, nullptr, A, ctl,
                                                                      retry_out);
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
  }
  EIM_CUDA(cudaEventRecord(ctx->ev1, st));
  res.launches = 1;
  read_ctl();
  float ms = 0;
  EIM_CUDA(cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1));
  res.kernel_ms = ms;

  // ---- retry tiers over the re-queued ids
  int tier = 1;
  uint32_t qbits = (model == EIM_IC) ? 8 : 6;  // log2 capacity of the tier that failed
  while (h->retry_count > 0) {
    const uint64_t nretry = h->retry_count;
    res.tier2 += nretry;
    grow_if_needed();
    std::swap(retry_in, retry_out);
    EIM_CUDA(cudaMemsetAsync(ctl, 0, sizeof(SampleCtl), st));
    A = arena_view(ctx, set_base, hist);
    ++tier;
    if (model == EIM_IC && tier == 2) {
      launch_ic<128, false>(ctx, g, seed, 0, nretry, retry_in, A, ctl, retry_out, IC_T2.hbits, IC_T2.qcap,
                            IC_T2.cap_quads, IC_T2.NG, ~0ull);
      qbits = 11;
    } else {
      // global-memory tiers: capacity x16 per tier until it covers n
      qbits = std::min(std::max(qbits + 4, 16u), nbits);
      const uint64_t qcap = 1ull << qbits;
      const uint32_t tbits = qbits + 1;
      const uint64_t per_slot = (8ull << tbits) + 4ull * qcap;
      const uint64_t budget = 1ull << 30;
      uint64_t slots = std::min<uint64_t>(nretry, std::max<uint64_t>(1, budget / per_slot));
      slots = std::min<uint64_t>(slots, (uint64_t)ctx->sm_count * (model == EIM_IC ? 2 : 64));
      ctx->tier_tab.reserve(slots * (8ull << tbits), false, st);
      ctx->tier_queue.reserve(slots * qcap * 4, false, st);
      ctx->tier_gen.reserve(slots * 4, false, st);
      EIM_CUDA(cudaMemsetAsync(ctx->tier_gen.p, 0, slots * 4, st));
      if (model == EIM_IC) {
        launch_ic<512, true>(ctx, g, seed, 0, nretry, retry_in, A, ctl, retry_out, tbits, (uint32_t)qcap, 0, 1, slots);
      } else {
        const uint32_t group = (uint32_t)std::min<uint64_t>(128, slots);
        const uint32_t blocks = (uint32_t)((slots + group - 1) / group);
        lt_tierk_kernel<<<blocks, group, 0, st>>>(g->view, seed, nretry, retry_in, A, ctl, retry_out,
                                                  ctx->tier_tab.as<unsigned long long>(), tbits,
                                                  ctx->tier_queue.as<uint32_t>(), (uint32_t)qcap,
                                                  ctx->tier_gen.as<uint32_t>());
        EIM_CUDA(cudaGetLastError());
        ctx->kernel_launches++;
      }
    }
    read_ctl();
    if (h->retry_count == nretry && !h->arena_fail && qbits >= nbits && tier > 3)
      fail(EIM_E_CUDA, "sampler made no progress at full capacity");
  }
  return res;
}

}  // namespace eim
