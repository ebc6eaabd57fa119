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

// Per-warp staging of one frontier batch (row descriptors).
struct RowStage {
  unsigned long long e0[32], e1[32], q0[32];
  uint32_t T[32], qend[32];
};

__device__ __forceinline__ void commit_set(const ArenaView& A, SampleCtl* ctl, unsigned long long* retry_out,
                                           uint64_t s, const uint32_t* queue, uint32_t size, int lane,
                                           bool ok, unsigned long long sample_edges,
                                           unsigned long long& edges_acc) {
  bool arena_fail = false;
  if (ok) {
    unsigned long long start = 0;
    if (lane == 0) start = atomicAdd(A.cursor, (unsigned long long)size);
    start = __shfl_sync(FULL, start, 0);
    if (start + size <= A.cap) {
      for (uint32_t i = lane; i < size; i += 32u) {
        uint32_t v = queue[i];
        A.elems[start + i] = v;
        if (A.C) atomicAdd(&A.C[v], 1u);
      }
      if (lane == 0) {
        A.set_start[s - A.set_base] = start;
        A.set_len[s - A.set_base] = size;
        atomicMax(A.valid_end, start + size);
      }
      edges_acc += sample_edges;
    } else {
      arena_fail = true;
    }
  }
  if (lane == 0 && (!ok || arena_fail)) {
    unsigned long long p = atomicAdd(&ctl->retry_count, 1ull);
    retry_out[p] = s;
    if (arena_fail) atomicAdd(&ctl->arena_fail, 1ull);
  }
}

// One IC RRR set by one warp.  Returns false on queue overflow.
template <class Table>
__device__ __forceinline__ bool ic_sample_warp(const GraphView& g, const PhiloxKey& K, uint64_t s,
                                               const Table& tab, uint32_t* queue, uint32_t qcap,
                                               RowStage& rs, int lane, uint32_t& size_out,
                                               unsigned long long& edges_out) {
  const unsigned lt_mask = (1u << lane) - 1u;
  uint32_t root = 0;
  if (lane == 0) {
    root = draw_root(s, g.n, K);
    tab.insert(root);
    queue[0] = root;
  }
  __syncwarp();
  uint32_t head = 0, tail = 1;
  unsigned long long my_edges = 0;
  while (head < tail) {
    const uint32_t nb = min(32u, tail - head);
    uint32_t nq = 0;
    if (lane < nb) {
      const uint32_t u = queue[head + lane];
      const unsigned long long e0 = g.off[u], e1 = g.off[u + 1];
      rs.e0[lane] = e0;
      rs.e1[lane] = e1;
      rs.T[lane] = g.thr[u];
      rs.q0[lane] = e0 >> 2;
      if (e1 > e0) nq = (uint32_t)(((e1 - 1) >> 2) - (e0 >> 2) + 1);
      my_edges += e1 - e0;
    }
    uint32_t incl = nq;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t t = __shfl_up_sync(FULL, incl, o);
      if (lane >= o) incl += t;
    }
    if (lane < nb) rs.qend[lane] = incl;
    const uint32_t total = __shfl_sync(FULL, incl, 31);
    head += nb;
    __syncwarp();
    // lane-private cursor into the batch's rows
    int r = 0;
    uint32_t qend_r = rs.qend[0];
    uint32_t qbeg_r = 0;
    unsigned long long e0_r = rs.e0[0], e1_r = rs.e1[0], q0_r = rs.q0[0];
    uint32_t T_r = rs.T[0];
    bool overflow = false;
    for (uint32_t base = 0; base < total; base += 32u) {
      const uint32_t j = base + lane;
      const bool valid = j < total;
      uint32_t live = 0;
      unsigned long long eb = 0;
      if (valid) {
        if (j >= qend_r) {
          do {
            ++r;
            qbeg_r = qend_r;
            qend_r = rs.qend[r];
          } while (j >= qend_r);
          e0_r = rs.e0[r];
          e1_r = rs.e1[r];
          q0_r = rs.q0[r];
          T_r = rs.T[r];
        }
        const unsigned long long q = q0_r + (j - qbeg_r);
        const uint4 w = philox_at(q, s, TAG_EDGE, K);
        eb = q << 2;
        // edge eb+i is in the row iff e0 <= eb+i < e1
        live |= (eb + 0 >= e0_r && eb + 0 < e1_r && w.x <= T_r) ? 1u : 0u;
        live |= (eb + 1 >= e0_r && eb + 1 < e1_r && w.y <= T_r) ? 2u : 0u;
        live |= (eb + 2 >= e0_r && eb + 2 < e1_r && w.z <= T_r) ? 4u : 0u;
        live |= (eb + 3 >= e0_r && eb + 3 < e1_r && w.w <= T_r) ? 8u : 0u;
      }
      if (__ballot_sync(FULL, live != 0u) == 0u) continue;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        bool ins = false;
        uint32_t v = 0;
        if ((live >> i) & 1u) {
          v = g.nbr[eb + i];
          ins = tab.insert(v);
        }
        const unsigned bal = __ballot_sync(FULL, ins);
        if (bal) {
          const uint32_t pos = tail + __popc(bal & lt_mask);
          if (ins && pos < qcap) queue[pos] = v;
          tail += __popc(bal);
        }
      }
      if (tail > qcap) {
        overflow = true;
        break;
      }
    }
    if (overflow) {
      size_out = 0;
      return false;
    }
    __syncwarp();
  }
  // warp-reduce the examined-edge count
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) my_edges += __shfl_xor_sync(FULL, my_edges, o);
  edges_out = my_edges;
  size_out = tail;
  return true;
}

template <int HBITS>
__global__ void __launch_bounds__(256) ic_tier1_kernel(GraphView g, uint64_t seed, uint64_t first,
                                                       uint64_t count, const unsigned long long* ids,
                                                       ArenaView A, SampleCtl* ctl,
                                                       unsigned long long* retry_out) {
  constexpr uint32_t H = 1u << HBITS;
  constexpr uint32_t Q = H / 2;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char* base = smem_raw + (size_t)warp * (H * 4 + Q * 4 + sizeof(RowStage));
  SmemTable tab{reinterpret_cast<uint32_t*>(base), HBITS};
  uint32_t* queue = reinterpret_cast<uint32_t*>(base + H * 4);
  RowStage& rs = *reinterpret_cast<RowStage*>(base + H * 4 + Q * 4);
  const PhiloxKey K = philox_key(seed);
  tab.clear(lane);
  __syncwarp();
  unsigned long long edges_acc = 0;
  for (;;) {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(&ctl->ticket, 1ull);
    t = __shfl_sync(FULL, t, 0);
    if (t >= count) break;
    const uint64_t s = ids ? ids[t] : first + t;
    uint32_t size = 0;
    unsigned long long se = 0;
    const bool ok = ic_sample_warp(g, K, s, tab, queue, Q, rs, lane, size, se);
    commit_set(A, ctl, retry_out, s, queue, size, lane, ok, se, edges_acc);
    __syncwarp();
    tab.clear(lane);
    __syncwarp();
  }
  if (lane == 0 && edges_acc) atomicAdd(&ctl->edges, edges_acc);
}

__global__ void __launch_bounds__(256) ic_tierk_kernel(GraphView g, uint64_t seed, uint64_t count,
                                                       const unsigned long long* ids, ArenaView A,
                                                       SampleCtl* ctl, unsigned long long* retry_out,
                                                       unsigned long long* tabs, uint32_t tbits,
                                                       uint32_t* queues, uint32_t qcap, uint32_t* gens) {
  __shared__ RowStage stage[8];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint64_t slot = (uint64_t)blockIdx.x * (blockDim.x >> 5) + warp;
  unsigned long long* h = tabs + (slot << tbits);
  uint32_t* queue = queues + slot * (uint64_t)qcap;
  const PhiloxKey K = philox_key(seed);
  unsigned long long edges_acc = 0;
  for (;;) {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(&ctl->ticket, 1ull);
    t = __shfl_sync(FULL, t, 0);
    if (t >= count) break;
    const uint64_t s = ids[t];
    uint32_t gen = 0;
    if (lane == 0) {
      gen = gens[slot] + 1u;
      if (gen == 0u) gen = 1u;  // (wrap after 2^32 samples: cleared below)
      gens[slot] = gen;
    }
    gen = __shfl_sync(FULL, gen, 0);
    if (gen == 1u) {  // fresh or wrapped generation counter: clear the table once
      for (uint64_t i = lane; i < (1ull << tbits); i += 32) h[i] = 0ull;
      __syncwarp();
      __threadfence_block();
    }
    GenTable tab{h, tbits, gen};
    uint32_t size = 0;
    unsigned long long se = 0;
    const bool ok = ic_sample_warp(g, K, s, tab, queue, qcap, stage[warp], lane, size, se);
    commit_set(A, ctl, retry_out, s, queue, size, lane, ok, se, edges_acc);
    __syncwarp();
  }
  if (lane == 0 && edges_acc) atomicAdd(&ctl->edges, edges_acc);
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

constexpr int IC_HBITS = 10;                      // 1024 hash slots, queue 512 per warp
constexpr int IC_WARPS = 8;
constexpr size_t IC_SMEM_PER_WARP = (1u << IC_HBITS) * 4 + (1u << (IC_HBITS - 1)) * 4 + sizeof(RowStage);
constexpr int LT_P = 64;                          // path capacity per walker (tier 1)
constexpr int LT_THREADS = 128;

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

  // tier 1
  EIM_CUDA(cudaMemsetAsync(ctl, 0, sizeof(SampleCtl), st));
  ArenaView A = arena_view(ctx, set_base, hist);
  unsigned long long* retry_in = ctx->retry_a.as<unsigned long long>();
  unsigned long long* retry_out = ctx->retry_b.as<unsigned long long>();
  EIM_CUDA(cudaEventRecord(ctx->ev0, st));
  if (model == EIM_IC) {
    const size_t smem = IC_SMEM_PER_WARP * IC_WARPS;
    EIM_CUDA(cudaFuncSetAttribute(ic_tier1_kernel<IC_HBITS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, ic_tier1_kernel<IC_HBITS>, IC_WARPS * 32, smem));
    uint32_t blocks = (uint32_t)std::max(1, per_sm) * ctx->sm_count;
    uint64_t need = (count + IC_WARPS - 1) / IC_WARPS;
    if (need < blocks) blocks = (uint32_t)need;
    ic_tier1_kernel<IC_HBITS><<<blocks, IC_WARPS * 32, smem, st>>>(g->view, seed, first, count, nullptr, A, ctl, retry_out);
  } else {
    const size_t smem = (size_t)LT_P * LT_THREADS * sizeof(uint32_t);
    int per_sm = 0;
    EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lt_tier1_kernel<LT_P>, LT_THREADS, smem));
    uint32_t blocks = (uint32_t)std::max(1, per_sm) * ctx->sm_count;
    uint64_t need = (count + LT_THREADS - 1) / LT_THREADS;
    if (need < blocks) blocks = (uint32_t)need;
    lt_tier1_kernel<LT_P><<<blocks, LT_THREADS, smem, st>>>(g->view, seed, first, count, nullptr, A, ctl, retry_out);
  }
  EIM_CUDA(cudaGetLastError());
  EIM_CUDA(cudaEventRecord(ctx->ev1, st));
  ctx->kernel_launches++;
  res.launches = 1;
  EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl) + 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  float ms = 0;
  EIM_CUDA(cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1));
  res.kernel_ms = ms;
  res.edges += h->edges;

  uint32_t qbits = (model == EIM_IC) ? (IC_HBITS - 1) : 6;  // log2 capacity of the tier that failed
  uint32_t nbits = 1;
  while ((1ull << nbits) < (uint64_t)g->view.n) nbits++;
  while (h->retry_count > 0) {
    const uint64_t nretry = h->retry_count;
    res.tier2 += nretry;
    if (h->arena_fail) {
      // grow the arena, keeping [0, valid_end) (successful reservations form a prefix)
      const uint64_t valid = h_tail[1];
      const uint64_t cap = ctx->arena.bytes / sizeof(uint32_t);
      const uint64_t want = std::max<uint64_t>(cap * 2, valid * 2 + 4096ull * nretry);
      ctx->arena.reserve(want * sizeof(uint32_t), true, st);
      EIM_CUDA(cudaMemcpyAsync(tail, &h_tail[1], sizeof(unsigned long long), cudaMemcpyHostToDevice, st));
    }
    std::swap(retry_in, retry_out);
    // next tier: capacity x16 until it covers n (a set has at most n members)
    qbits = std::min(qbits + 4, nbits);
    const uint64_t qcap = 1ull << qbits;
    const uint32_t tbits = qbits + 1;
    const uint64_t per_slot = (8ull << tbits) + 4ull * qcap;
    const uint64_t budget = 1ull << 30;
    uint64_t slots = std::min<uint64_t>(nretry, std::max<uint64_t>(1, budget / per_slot));
    slots = std::min<uint64_t>(slots, (uint64_t)ctx->sm_count * 64);
    const uint32_t max_group = (model == EIM_IC) ? 8 : 128;  // slots (warps / threads) per block
    const uint32_t group = (uint32_t)std::min<uint64_t>(max_group, slots);
    const uint32_t blocks = (uint32_t)((slots + group - 1) / group);
    slots = (uint64_t)blocks * group;
    ctx->tier_tab.reserve(slots * (8ull << tbits), false, st);
    ctx->tier_queue.reserve(slots * qcap * 4, false, st);
    ctx->tier_gen.reserve(slots * 4, false, st);
    EIM_CUDA(cudaMemsetAsync(ctx->tier_gen.p, 0, slots * 4, st));
    EIM_CUDA(cudaMemsetAsync(ctl, 0, sizeof(SampleCtl), st));
    A = arena_view(ctx, set_base, hist);
    if (model == EIM_IC)
      ic_tierk_kernel<<<blocks, group * 32, 0, st>>>(g->view, seed, nretry, retry_in, A, ctl, retry_out,
                                              ctx->tier_tab.as<unsigned long long>(), tbits,
                                              ctx->tier_queue.as<uint32_t>(), (uint32_t)qcap,
                                              ctx->tier_gen.as<uint32_t>());
    else
      lt_tierk_kernel<<<blocks, group, 0, st>>>(g->view, seed, nretry, retry_in, A, ctl, retry_out,
                                              ctx->tier_tab.as<unsigned long long>(), tbits,
                                              ctx->tier_queue.as<uint32_t>(), (uint32_t)qcap,
                                              ctx->tier_gen.as<uint32_t>());
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
    EIM_CUDA(cudaMemcpyAsync(h, ctl, sizeof(SampleCtl) + 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    res.edges += h->edges;
    if (h->retry_count == nretry && !h->arena_fail && qbits >= nbits)
      fail(EIM_E_CUDA, "sampler made no progress at full capacity");
  }
  return res;
}

}  // namespace eim
