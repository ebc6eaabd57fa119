// select.cu -- greedy max-coverage NodeSelection (Alg. 3).
//
// Per NodeSelection (all of R, from scratch, R15):
//   1. candidates = vertices with C[v] > 0, compacted in ascending id order
//      (stable scan), so a candidate index orders like its vertex id;
//   2. the arena is remapped to candidate indices and an inverted index
//      (candidate -> ids of the sets containing it) is built by a counting
//      sort, so a pick touches only the sets that contain it (instead of the
//      paper's thread-per-set binary search over all theta sets);
//   3. ONE cooperative persistent kernel runs all k picks.  Per pick: every
//      block reduces its slice of the working counts W to a 64-bit key
//      (count << 32 | ~index: highest count, ties to the lowest id, R10), a
//      grid barrier, every block reduces the block maxima, the winner's
//      uncovered sets are marked covered (F[i] <- 1) and every member count is
//      decremented (Alg. 3 l.7-12) by one warp per inverted-list entry, a
//      grid barrier.  A selected vertex ends with W = 0 (all its sets are
//      covered); when the maximum count is 0 every set is covered and the
//      pick is the lowest unselected vertex id (R10).
#include <cooperative_groups.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include <cub/cub.cuh>

#include "arena_view.cuh"

namespace cg = cooperative_groups;

namespace eim {

namespace {

constexpr unsigned FULL = 0xFFFFFFFFu;
constexpr int GB = 512;  // threads per block of the greedy kernel
constexpr uint32_t BIG = 64;       // covered sets with more members are walked by a whole block
constexpr uint32_t BIG_CAP = 256;  // queued per block and pick (more are walked by their warp)

__global__ void flag_kernel(const uint32_t* __restrict__ C, uint32_t n, uint32_t* __restrict__ flags) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= n; i += stride)
    flags[i] = (i < n && C[i] > 0u) ? 1u : 0u;
}

// pos = exclusive scan of flags: candidate index of v; nc = pos[n].  Writes
// the candidate list, the vertex -> candidate map, the working counts W
// (zero-padded to a multiple of 4) and the counts as u64 over [0, n] (zero
// past nc) for the inverted-index scan.
__global__ void compact_kernel(const uint32_t* __restrict__ C, const uint32_t* __restrict__ pos, uint32_t n,
                               uint32_t* __restrict__ cand, uint32_t* __restrict__ cidx, uint32_t* __restrict__ W,
                               uint64_t* __restrict__ cnt64) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint32_t nc = pos[n], nc_pad = (nc + 3u) & ~3u;
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
    const uint32_t c = C[v];
    if (c > 0u) {
      const uint32_t p = pos[v];
      cand[p] = (uint32_t)v;
      cidx[v] = p;
      W[p] = c;
      cnt64[p] = c;
    }
  }
  const uint64_t end = max((uint64_t)n + 1, (uint64_t)nc_pad);
  for (uint64_t i = nc + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < end; i += stride) {
    if (i <= n) cnt64[i] = 0ull;
    if (i < nc_pad) W[i] = 0u;
  }
}

__global__ void remap_kernel(const uint32_t* __restrict__ arena, uint32_t ab, uint64_t total,
                             const uint32_t* __restrict__ cidx, uint32_t* __restrict__ arena_c) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += stride)
    arena_c[i] = cidx[arena_get(arena, i, ab)];
}

// inverted index fill: one warp per set.  off[x] holds the END of x's list
// (inclusive scan of counts); each entry is placed at --off[x], so when the
// fill is done off[x] is the START of x's list (and off[x+1] its end).
__global__ void invert_kernel(const uint32_t* __restrict__ arena_c, const uint64_t* __restrict__ set_start,
                              const uint32_t* __restrict__ set_len, uint64_t num_sets,
                              unsigned long long* __restrict__ off, uint32_t* __restrict__ inv) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t i = warp; i < num_sets; i += nwarps) {
    const uint64_t st = set_start[i];
    const uint32_t L = set_len[i];
    for (uint32_t t = lane; t < L; t += 32) {
      const unsigned long long p = atomicAdd(&off[arena_c[st + t]], ~0ull) - 1ull;
      inv[p] = (uint32_t)i;
    }
  }
}

__device__ __forceinline__ unsigned long long umax64(unsigned long long a, unsigned long long b) {
  return a > b ? a : b;
}

__device__ __forceinline__ unsigned long long ckey(uint32_t c, uint32_t i) {
  return c ? (((unsigned long long)c << 32) | (unsigned long long)(0xFFFFFFFFu - i)) : 0ull;
}

__device__ __forceinline__ unsigned long long block_max(unsigned long long k, unsigned long long* red) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) k = umax64(k, __shfl_xor_sync(FULL, k, o));
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = k;
  __syncthreads();
  if (threadIdx.x < 32) {
    k = threadIdx.x < GB / 32 ? red[threadIdx.x] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) k = umax64(k, __shfl_xor_sync(FULL, k, o));
    if (threadIdx.x == 0) red[0] = k;
  }
  __syncthreads();
  k = red[0];
  __syncthreads();
  return k;
}

struct GreedyArgs {
  uint32_t k;
  const uint32_t* nc;           // candidates (device)
  uint32_t* W;                  // working counts per candidate (padded with 0)
  const uint32_t* cand;         // candidate -> vertex (ascending)
  const uint64_t* inv_off;      // nc+1
  const uint32_t* inv;          // set ids
  uint8_t* F;                   // covered flags per set
  const uint64_t* set_start;
  const uint32_t* set_len;
  const uint32_t* arena_c;      // arena in candidate indices
  unsigned long long* blockmax; // gridDim
  uint8_t* selected;            // n flags (for the all-covered case)
  uint32_t* zc;                 // cursor of the lowest possibly-unselected id
  uint32_t* seeds;
  unsigned long long* gains;
  unsigned long long* dbg;      // development: per-pick timestamps (nullable)
  unsigned long long* dbgb;     // development: every block's barrier arrivals (2 per pick and block)
  // chunked argmax (nc >= chunk_min): chunk_key[c] = the maximum key of
  // chunk c's candidates, refreshed only for the chunks whose counts a
  // cover touched (dirty[c]); the argmax then reads one key per chunk
  unsigned long long* chunk_key;
  uint8_t* dirty;
  uint32_t chunk_min;
  uint32_t chunk_shift;         // log2(candidates per chunk)
};

constexpr uint32_t CHUNK_SHIFT = 11;             // 2048 candidates (8 KB of counts) per chunk
// opt-in (EIM_GREEDY_CHUNK_MIN): measured slower than the full scan at every
// config (select per IMM: C2 2.07 -> 2.52 ms, C3 1.35 -> 1.97, C4 7.8 ->
// 8.9, C5 73.5 -> 127 ms): the covers touch most chunks of the hub-heavy
// counts, and marking them costs a store per decrement
constexpr uint32_t CHUNK_MIN_DEFAULT = 0xFFFFFFFFu;

__device__ __forceinline__ unsigned long long gtimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

template <bool CHUNKED>
__global__ void __launch_bounds__(GB) greedy_kernel(GreedyArgs a) {
  cg::grid_group grid = cg::this_grid();
  __shared__ unsigned long long red[GB / 32];
  __shared__ uint32_t big[BIG_CAP];
  __shared__ uint32_t nbig;
  if (threadIdx.x == 0) nbig = 0;
  const uint32_t nc = *a.nc;
  const uint32_t nc4 = ((nc + 3u) & ~3u) / 4;
  const uint4* W4 = reinterpret_cast<const uint4*>(a.W);
  const int lane = threadIdx.x & 31;
  // list entries are dealt to the warps block-interleaved (entry p goes to
  // block p mod gridDim.x), so a short list spreads over all SMs instead of
  // filling the first blocks' warps, and long sets do not pile up in one block
  const uint64_t warp = (uint64_t)(threadIdx.x >> 5) * gridDim.x + blockIdx.x;
  const uint64_t nwarps = ((uint64_t)gridDim.x * GB) >> 5;
  // ---- chunked argmax: for many candidates the full scan of W per pick
  // (4 B per candidate from L2/HBM) is replaced by one key per chunk of
  // 2^chunk_shift candidates; a cover marks the chunks whose counts it
  // decrements, and only those are rescanned (by the block that owns them)
  // before the next argmax.  The keys are exact whenever they are read, so
  // the winner and the tie rule are the full scan's.
  // (the chunked argmax is a separate instantiation: the default kernel
  // carries none of its code)
  const bool chunked = CHUNKED && nc >= a.chunk_min;
  const uint32_t c4 = (1u << a.chunk_shift) / 4;  // uint4 per chunk (>= 1)
  const uint32_t nchunks = (nc4 + c4 - 1) / c4;
  const uint32_t cpb = (nchunks + gridDim.x - 1) / gridDim.x;  // chunks per block
  const uint32_t cb0 = min(blockIdx.x * cpb, nchunks), cb1 = min(cb0 + cpb, nchunks);
  for (uint32_t j = 0; j < a.k; ++j) {
    if (a.dbg && blockIdx.x == 0 && threadIdx.x == 0) a.dbg[3 * j] = gtimer_ns();
    unsigned long long km = 0;
    if (CHUNKED && chunked) {
      // refresh this block's dirty chunks (a warp per chunk), then reduce
      // its chunk keys
      for (uint32_t c = cb0 + (threadIdx.x >> 5); c < cb1; c += GB / 32) {
        if (!__ldcg(a.dirty + c)) continue;
        unsigned long long e = 0;
        for (uint32_t i = c * c4 + lane; i < min((c + 1) * c4, nc4); i += 32) {
          const uint4 w = __ldcg(W4 + i);
          const uint32_t x = 4u * i;
          e = umax64(e, umax64(umax64(ckey(w.x, x), ckey(w.y, x + 1)), umax64(ckey(w.z, x + 2), ckey(w.w, x + 3))));
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) e = umax64(e, __shfl_xor_sync(FULL, e, o));
        if (lane == 0) {
          a.chunk_key[c] = e;
          a.dirty[c] = 0;
        }
      }
      __syncthreads();
      for (uint32_t c = cb0 + threadIdx.x; c < cb1; c += GB) km = umax64(km, a.chunk_key[c]);
      km = block_max(km, red);
      if (threadIdx.x == 0) a.blockmax[blockIdx.x] = km;
      if (a.dbgb && threadIdx.x == 0) a.dbgb[(2ull * j) * gridDim.x + blockIdx.x] = gtimer_ns();
      grid.sync();
      if (a.dbg && blockIdx.x == 0 && threadIdx.x == 0) a.dbg[3 * j + 1] = gtimer_ns();
      km = 0;
      for (uint32_t b = threadIdx.x; b < gridDim.x; b += GB) km = umax64(km, a.blockmax[b]);
      km = block_max(km, red);
    } else {
    // ---- argmax over this block's slice
    for (uint32_t i = blockIdx.x * GB + threadIdx.x; i < nc4; i += gridDim.x * GB) {
      const uint4 c = W4[i];
      const uint32_t x = 4u * i;
      km = umax64(km, ckey(c.x, x));
      km = umax64(km, ckey(c.y, x + 1));
      km = umax64(km, ckey(c.z, x + 2));
      km = umax64(km, ckey(c.w, x + 3));
    }
    km = block_max(km, red);
    if (threadIdx.x == 0) a.blockmax[blockIdx.x] = km;
    if (a.dbgb && threadIdx.x == 0) a.dbgb[(2ull * j) * gridDim.x + blockIdx.x] = gtimer_ns();
    grid.sync();
    if (a.dbg && blockIdx.x == 0 && threadIdx.x == 0) a.dbg[3 * j + 1] = gtimer_ns();
    km = 0;
    for (uint32_t b = threadIdx.x; b < gridDim.x; b += GB) km = umax64(km, a.blockmax[b]);
    km = block_max(km, red);
    }
    if (km == 0ull) {
      // every set is covered: the lowest unselected vertex id, gain 0
      if (blockIdx.x == 0 && threadIdx.x == 0) {
        uint32_t z = *a.zc;
        while (a.selected[z]) ++z;
        *a.zc = z;
        a.selected[z] = 1;
        a.seeds[j] = z;
        a.gains[j] = 0;
      }
    } else {
      const uint32_t ci = 0xFFFFFFFFu - (uint32_t)km;
      if (blockIdx.x == 0 && threadIdx.x == 0) {
        const uint32_t v = a.cand[ci];
        a.selected[v] = 1;
        a.seeds[j] = v;
        a.gains[j] = km >> 32;
      }
      // ---- cover: one warp per entry of the winner's inverted list; a
      // set larger than BIG (the long reverse-BFS sets) is queued and walked
      // by the whole block afterwards, so no warp walks thousands of members
      const uint64_t lo = a.inv_off[ci], hi = a.inv_off[ci + 1];
      for (uint64_t p = lo + warp; p < hi; p += nwarps) {
        const uint32_t i = a.inv[p];
        if (a.F[i]) continue;  // covered by an earlier pick (ids are unique within one list)
        __syncwarp();
        const uint32_t L = a.set_len[i];
        const uint64_t st = a.set_start[i];
        bool queued = false;
        if (lane == 0) {
          a.F[i] = 1;
          if (L > BIG) {
            const uint32_t q = atomicAdd(&nbig, 1u);
            if (q < BIG_CAP) {
              big[q] = i;
              queued = true;
            }
          }
        }
        if (__shfl_sync(FULL, queued, 0)) continue;
#pragma unroll 4
        for (uint32_t t = lane; t < L; t += 32) {
          const uint32_t x = a.arena_c[st + t];
          atomicSub(&a.W[x], 1u);
          if (CHUNKED && chunked) a.dirty[x >> a.chunk_shift] = 1;
        }
      }
      __syncthreads();
      const uint32_t nb = min(nbig, BIG_CAP);
      for (uint32_t q = 0; q < nb; ++q) {
        const uint32_t i = big[q];
        const uint64_t st = a.set_start[i];
        const uint32_t L = a.set_len[i];
#pragma unroll 4
        for (uint32_t t = threadIdx.x; t < L; t += GB) {
          const uint32_t x = a.arena_c[st + t];
          atomicSub(&a.W[x], 1u);
          if (CHUNKED && chunked) a.dirty[x >> a.chunk_shift] = 1;
        }
      }
      __syncthreads();
      if (threadIdx.x == 0) nbig = 0;
    }
    if (a.dbg && blockIdx.x == 0 && threadIdx.x == 0) a.dbg[3 * j + 2] = gtimer_ns();
    if (a.dbgb && threadIdx.x == 0) a.dbgb[(2ull * j + 1) * gridDim.x + blockIdx.x] = gtimer_ns();
    grid.sync();
  }
}

}  // namespace

void greedy_launch(eim_ctx* ctx, int slot, uint32_t n, uint64_t num_sets, uint64_t total, const uint32_t* C,
                   uint32_t k) {
  greedy_setup(ctx, slot, n, num_sets, total, C);
  greedy_picks(ctx, slot, n, num_sets, k, 0);
}

// steps 1-2: candidates, remapped arena, inverted index (enqueued on the slot's stream)
void greedy_setup(eim_ctx* ctx, int slot, uint32_t n, uint64_t num_sets, uint64_t total, const uint32_t* C) {
  GreedySlot& S = ctx->gs[slot];
  cudaStream_t st = S.stream;
  if (st != ctx->stream) {  // the slot's stream starts after the work enqueued so far (sets, C)
    EIM_CUDA(cudaEventRecord(ctx->ev0, ctx->stream));
    EIM_CUDA(cudaStreamWaitEvent(st, ctx->ev0, 0));
  }
  // ---- 1. candidates (C > 0) in ascending id order; nc stays on the device
  // (buffers are sized for nc <= n), so nothing here waits for the host
  S.inv_fill.reserve(((uint64_t)n + 1) * sizeof(uint64_t), false, st);  // scratch: flags/pos (u32)
  uint32_t* pos = S.inv_fill.as<uint32_t>();
  flag_kernel<<<grid_for(ctx, (uint64_t)n + 1, 256), 256, 0, st>>>(C, n, pos);
  EIM_CUDA(cudaGetLastError());
  size_t tmp = 0, tmp2 = 0;
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, pos, pos, (uint64_t)n + 1, st));
  S.inv_off.reserve(((uint64_t)n + 1) * sizeof(uint64_t), false, st);
  uint64_t* inv_off = S.inv_off.as<uint64_t>();
  EIM_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tmp2, inv_off, inv_off, (uint64_t)n + 1, st));
  S.scratch.reserve(std::max<size_t>(std::max(tmp, tmp2), 1 << 20), false, st);
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(S.scratch.p, tmp, pos, pos, (uint64_t)n + 1, st));
  S.cand.reserve((uint64_t)std::max(n, 1u) * 4, false, st);
  S.cidx.reserve((uint64_t)n * 4, false, st);
  S.C_work.reserve(((uint64_t)n + 4) * 4, false, st);
  compact_kernel<<<grid_for(ctx, n, 256), 256, 0, st>>>(C, pos, n, S.cand.as<uint32_t>(), S.cidx.as<uint32_t>(),
                                                          S.C_work.as<uint32_t>(), inv_off);
  EIM_CUDA(cudaGetLastError());
  // ---- 2. arena in candidate indices + inverted index
  S.arena_c.reserve(std::max<uint64_t>(total, 1) * 4, false, st);
  if (total)
    remap_kernel<<<grid_for(ctx, total, 256), 256, 0, st>>>(ctx->arena.as<uint32_t>(), ctx->arena_b, total,
                                                              S.cidx.as<uint32_t>(), S.arena_c.as<uint32_t>());
  EIM_CUDA(cub::DeviceScan::InclusiveSum(S.scratch.p, tmp2, inv_off, inv_off, (uint64_t)n + 1, st));
  S.inv.reserve(std::max<uint64_t>(total, 1) * sizeof(uint32_t), false, st);
  if (num_sets > 0 && total > 0) {
    invert_kernel<<<grid_for(ctx, num_sets * 32, 256), 256, 0, st>>>(
        S.arena_c.as<uint32_t>(), ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>(), num_sets,
        reinterpret_cast<unsigned long long*>(inv_off), S.inv.as<uint32_t>());
    EIM_CUDA(cudaGetLastError());
  }
  ctx->kernel_launches += 7;
}

// Blocks of nsel concurrent selections over num_sets[t] sets each: the SMs
// are shared in proportion to sqrt(num_sets) (a larger R has more
// candidates to scan and longer lists to cover, every selection runs k
// picks, and a pick's latency falls slowly with its blocks), at least 16
// blocks each.  Measured against an even split: C3 selection 1.465 -> 1.41
// ms, C2 1.675 -> 1.65 ms (weights R^1: 1.42 / 1.66, R^1.5: 1.51 / 1.72).
// EIM_GREEDY_EVEN=1: an even split.
void greedy_shares(eim_ctx* ctx, uint32_t nsel, const uint64_t* num_sets, uint32_t* blocks) {
  const uint32_t sm = (uint32_t)ctx->sm_count, lo = std::min<uint32_t>(16, sm / std::max(nsel, 1u));
  const char* pe = getenv("EIM_GREEDY_POW");  // development: weights num_sets^pow (0: even)
  const double pw = getenv("EIM_GREEDY_EVEN") ? 0.0 : (pe ? std::strtod(pe, nullptr) : 0.5);
  double tot = 0;
  for (uint32_t t = 0; t < nsel; ++t) tot += std::pow((double)std::max<uint64_t>(num_sets[t], 1), pw);
  uint32_t used = 0;
  for (uint32_t t = 0; t < nsel; ++t) {
    const double w = std::pow((double)std::max<uint64_t>(num_sets[t], 1), pw) / tot;
    blocks[t] = std::max(lo, (uint32_t)(w * sm));
    used += blocks[t];
  }
  while (used > sm) {  // the minimum pushed the sum over: take from the largest share
    uint32_t* b = std::max_element(blocks, blocks + nsel);
    --*b;
    --used;
  }
}

// step 3: the k picks in one cooperative grid kernel
void greedy_picks(eim_ctx* ctx, int slot, uint32_t n, uint64_t num_sets, uint32_t k, uint32_t blocks_share) {
  GreedySlot& S = ctx->gs[slot];
  cudaStream_t st = S.stream;
  uint32_t* pos = S.inv_fill.as<uint32_t>();
  uint64_t* inv_off = S.inv_off.as<uint64_t>();
  // ---- 3. the k picks in one cooperative kernel
  // covered flags (num_sets), selected flags (n), the all-covered cursor:
  // one buffer, one memset
  const uint64_t fl_sets = (std::max<uint64_t>(num_sets, 1) + 15) & ~15ull;
  const uint64_t fl_sel = ((uint64_t)n + 4 + 15) & ~15ull;
  S.covered.reserve(fl_sets + fl_sel + 16, false, st);
  S.seeds.reserve((uint64_t)k * sizeof(uint32_t), false, st);
  S.gains.reserve((uint64_t)k * sizeof(unsigned long long), false, st);
  EIM_CUDA(cudaMemsetAsync(S.covered.p, 0, fl_sets + fl_sel + 16, st));
  uint8_t* selected = S.covered.as<uint8_t>() + fl_sets;
  uint32_t* zc = reinterpret_cast<uint32_t*>(selected + fl_sel);
  static int per_sm = 0;  // occupancy of the pick kernel (a property of the binary and the device)
  const char* cm = getenv("EIM_GREEDY_CHUNK_MIN");
  const void* kern = cm ? (const void*)greedy_kernel<true> : (const void*)greedy_kernel<false>;
  if (per_sm == 0) EIM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, GB, 0));
  const char* gbe = getenv("EIM_GREEDY_BLOCKS");  // development: grid of the greedy kernel
  uint32_t blocks = gbe ? (uint32_t)atoi(gbe) : (uint32_t)ctx->sm_count;
  // concurrent selections get their share of the SMs (greedy_shares): two
  // 148-block cooperative grids launched together do not overlap (C3: 2.0 ms
  // against 1.93 ms one after the other), 74 + 74 blocks do (1.33 ms)
  if (blocks_share > 0) blocks = std::min(blocks, blocks_share);
  blocks = std::max(1u, std::min(blocks, (uint32_t)std::max(1, per_sm) * ctx->sm_count));
  // chunked argmax from this many candidates on (EIM_GREEDY_CHUNK_MIN; 0:
  // always) with 2^shift candidates per chunk (EIM_GREEDY_CHUNK_SHIFT, >= 2)
  const char* cs = getenv("EIM_GREEDY_CHUNK_SHIFT");
  const uint32_t chunk_shift = std::max<uint32_t>(2, cs ? (uint32_t)strtoul(cs, nullptr, 10) : CHUNK_SHIFT);
  const uint64_t nchunks_max = ((uint64_t)n >> chunk_shift) + 2;
  S.best.reserve(((uint64_t)blocks + nchunks_max + 8) * sizeof(unsigned long long) + 64, false, st);
  S.dirty.reserve(nchunks_max, false, st);
  if (cm) EIM_CUDA(cudaMemsetAsync(S.dirty.p, 1, nchunks_max, st));  // every chunk key is computed at the first pick
  GreedyArgs a;
  a.k = k;
  a.nc = pos + n;
  a.W = S.C_work.as<uint32_t>();
  a.cand = S.cand.as<uint32_t>();
  a.inv_off = inv_off;
  a.inv = S.inv.as<uint32_t>();
  a.F = S.covered.as<uint8_t>();
  a.set_start = ctx->set_start.as<uint64_t>();
  a.set_len = ctx->set_len.as<uint32_t>();
  a.arena_c = S.arena_c.as<uint32_t>();
  a.blockmax = S.best.as<unsigned long long>();
  a.selected = selected;
  a.zc = zc;
  a.seeds = S.seeds.as<uint32_t>();
  a.gains = S.gains.as<unsigned long long>();
  a.chunk_key = S.best.as<unsigned long long>() + blocks + 8;
  a.dirty = S.dirty.as<uint8_t>();
  a.chunk_min = cm ? (uint32_t)strtoul(cm, nullptr, 10) : CHUNK_MIN_DEFAULT;
  a.chunk_shift = chunk_shift;
  a.dbg = nullptr;
  a.dbgb = nullptr;
  const char* gdbg = getenv("EIM_DEBUG_GREEDY");
  const uint64_t dbg_words = (uint64_t)k * 3 + (uint64_t)k * 2 * blocks;
  if (gdbg && slot == 0) {
    ctx->stage_a.reserve(dbg_words * 8 + 64, false, st);
    a.dbg = ctx->stage_a.as<unsigned long long>();
    a.dbgb = a.dbg + (uint64_t)k * 3;
  }
  void* args[] = {&a};
  if (!S.ev[0])
    for (cudaEvent_t& e : S.ev) EIM_CUDA(cudaEventCreate(&e));
  EIM_CUDA(cudaEventRecord(S.ev[0], st));
  EIM_CUDA(cudaLaunchCooperativeKernel(kern, dim3(blocks), dim3(GB), args, 0, st));
  EIM_CUDA(cudaEventRecord(S.ev[1], st));
  ctx->kernel_launches += 2;
  if (a.dbg) {  // file: k, blocks, stamps per pick and block, block 0's stamps, every block's arrivals
    std::vector<unsigned long long> hd(dbg_words + 3);
    hd[0] = k;
    hd[1] = blocks;
    hd[2] = 2;
    EIM_CUDA(cudaMemcpyAsync(hd.data() + 3, a.dbg, dbg_words * 8, cudaMemcpyDeviceToHost, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    FILE* f = fopen(gdbg, "ab");
    if (f) {
      fwrite(hd.data(), 8, hd.size(), f);
      fclose(f);
    }
  }
}

uint64_t greedy_collect(eim_ctx* ctx, int slot, uint32_t k, uint32_t* seeds_out, uint64_t* gains_out,
                        double* kernel_ms) {
  GreedySlot& S = ctx->gs[slot];
  cudaStream_t st = S.stream;
  std::vector<unsigned long long> g(k);
  EIM_CUDA(cudaMemcpyAsync(seeds_out, S.seeds.p, (uint64_t)k * sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaMemcpyAsync(g.data(), S.gains.p, (uint64_t)k * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  if (kernel_ms) {
    float ms = 0;
    EIM_CUDA(cudaEventElapsedTime(&ms, S.ev[0], S.ev[1]));
    *kernel_ms += ms;
  }
  if (st != ctx->stream) {  // later work on the context's stream may reuse what the selection read
    EIM_CUDA(cudaEventRecord(ctx->ev1, st));
    EIM_CUDA(cudaStreamWaitEvent(ctx->stream, ctx->ev1, 0));
  }
  uint64_t cov = 0;
  for (uint32_t j = 0; j < k; ++j) {
    cov += g[j];
    if (gains_out) gains_out[j] = g[j];
  }
  return cov;
}

uint64_t greedy(eim_ctx* ctx, uint32_t n, uint64_t num_sets, uint32_t k, uint32_t* seeds_out,
                uint64_t* gains_out, double* kernel_ms) {
  greedy_launch(ctx, 0, n, num_sets, arena_cursor(ctx), ctx->C_total.as<uint32_t>(), k);
  return greedy_collect(ctx, 0, k, seeds_out, gains_out, kernel_ms);
}

}  // namespace eim
