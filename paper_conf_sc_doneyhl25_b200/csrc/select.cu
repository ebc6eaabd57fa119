// select.cu -- greedy max-coverage NodeSelection (Alg. 3).
//
// Per pick j (two kernels, no host round trip):
//   argmax_kernel: key(x) = C[x] << 32 | (2^32-1-x) maximised over the grid
//     (block reduce + one 64-bit atomicMax per block): highest count, ties to
//     the lowest id (R10).  Already-selected vertices are excluded: the
//     previous pick by index, older picks because their count was replaced by
//     a sentinel.
//   cover_kernel: v = argmax; for every set i in v's inverted list with
//     F[i] = 0: F[i] <- 1 and C[x] -= 1 for each member x (Alg. 3 l.7-12).
// Instead of the paper's thread-per-set binary search over all theta sets
// (P:186), the sets containing v are found through an inverted index
// (vertex -> set ids) built once per NodeSelection by a counting sort on C,
// so a pick touches only the sets that contain v.
#include <cub/cub.cuh>

#include "eim_internal.h"

namespace eim {

namespace {

constexpr unsigned FULL = 0xFFFFFFFFu;

__global__ void count_to_u64_kernel(const uint32_t* __restrict__ C, uint32_t n, uint64_t* __restrict__ out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= n; i += stride)
    out[i] = i < n ? (uint64_t)C[i] : 0ull;
}

// inverted index fill: one warp per set, inv[fill[x]++] = set id
__global__ void invert_kernel(const uint32_t* __restrict__ arena, const uint64_t* __restrict__ set_start,
                              const uint32_t* __restrict__ set_len, uint64_t num_sets,
                              unsigned long long* __restrict__ fill, uint32_t* __restrict__ inv) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t i = warp; i < num_sets; i += nwarps) {
    const uint64_t st = set_start[i];
    const uint32_t L = set_len[i];
    for (uint32_t t = lane; t < L; t += 32) {
      const unsigned long long p = atomicAdd(&fill[arena[st + t]], 1ull);
      inv[p] = (uint32_t)i;
    }
  }
}

__global__ void init_work_kernel(const uint32_t* __restrict__ C, uint32_t n, uint32_t n_pad,
                                 uint32_t* __restrict__ W) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_pad; i += stride)
    W[i] = i < n ? C[i] : SENTINEL;
}

__device__ __forceinline__ unsigned long long vkey(uint32_t c, uint32_t x, uint32_t excl) {
  return (c == SENTINEL || x == excl) ? 0ull : (((unsigned long long)c << 32) | (unsigned long long)(0xFFFFFFFFu - x));
}

__device__ __forceinline__ unsigned long long umax64(unsigned long long a, unsigned long long b) {
  return a > b ? a : b;
}

template <int BLOCK>
__global__ void __launch_bounds__(BLOCK) argmax_kernel(const uint4* __restrict__ W4, uint32_t n4,
                                                       const uint32_t* __restrict__ seeds, uint32_t j,
                                                       unsigned long long* __restrict__ best) {
  const uint32_t excl = j > 0 ? seeds[j - 1] : SENTINEL;
  unsigned long long k = 0;
  const uint32_t stride = gridDim.x * BLOCK;
  for (uint32_t i = blockIdx.x * BLOCK + threadIdx.x; i < n4; i += stride) {
    const uint4 c = W4[i];
    const uint32_t x = i * 4u;
    k = umax64(k, vkey(c.x, x, excl));
    k = umax64(k, vkey(c.y, x + 1, excl));
    k = umax64(k, vkey(c.z, x + 2, excl));
    k = umax64(k, vkey(c.w, x + 3, excl));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) k = umax64(k, __shfl_xor_sync(FULL, k, o));
  __shared__ unsigned long long red[BLOCK / 32];
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = k;
  __syncthreads();
  if (threadIdx.x < 32) {
    k = threadIdx.x < BLOCK / 32 ? red[threadIdx.x] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) k = umax64(k, __shfl_xor_sync(FULL, k, o));
    if (threadIdx.x == 0 && k) atomicMax(&best[j], k);
  }
}

__global__ void cover_kernel(uint32_t j, const unsigned long long* __restrict__ best,
                             uint32_t* __restrict__ seeds, unsigned long long* __restrict__ gains,
                             uint32_t* __restrict__ W, const uint64_t* __restrict__ inv_off,
                             const uint32_t* __restrict__ inv, uint8_t* __restrict__ F,
                             const uint64_t* __restrict__ set_start, const uint32_t* __restrict__ set_len,
                             const uint32_t* __restrict__ arena) {
  const unsigned long long key = best[j];
  const uint32_t v = 0xFFFFFFFFu - (uint32_t)key;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    seeds[j] = v;
    gains[j] = key >> 32;
    if (j > 0) W[seeds[j - 1]] = SENTINEL;  // its sets are all covered: nobody else touches it
  }
  // one warp per entry of v's inverted list: the covered sets are
  // decremented in parallel across the whole grid
  const int lane = threadIdx.x & 31;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const uint64_t lo = inv_off[v], hi = inv_off[v + 1];
  for (uint64_t p = lo + warp; p < hi; p += nwarps) {
    const uint32_t i = inv[p];
    if (F[i]) continue;  // covered by an earlier pick (set ids are unique within v's list)
    __syncwarp();
    if (lane == 0) F[i] = 1;
    const uint64_t st = set_start[i];
    const uint32_t L = set_len[i];
    for (uint32_t t = lane; t < L; t += 32) atomicSub(&W[arena[st + t]], 1u);
  }
}

}  // namespace

uint64_t greedy(eim_ctx* ctx, uint32_t n, uint64_t num_sets, uint32_t k, uint32_t* seeds_out,
                uint64_t* gains_out) {
  cudaStream_t st = ctx->stream;
  const uint32_t n_pad = (n + 3u) & ~3u;
  // ---- inverted index: inv_off = exclusive scan of C_total, then scatter set ids
  ctx->inv_off.reserve(((uint64_t)n + 1) * sizeof(uint64_t), false, st);
  ctx->inv_fill.reserve(((uint64_t)n + 1) * sizeof(uint64_t), false, st);
  uint64_t* inv_off = ctx->inv_off.as<uint64_t>();
  count_to_u64_kernel<<<grid_for(ctx, (uint64_t)n + 1, 256), 256, 0, st>>>(ctx->C_total.as<uint32_t>(), n, inv_off);
  EIM_CUDA(cudaGetLastError());
  size_t tmp = 0;
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, inv_off, inv_off, (uint64_t)n + 1, st));
  ctx->scratch.reserve(std::max<size_t>(tmp, 1 << 20), false, st);
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(ctx->scratch.p, tmp, inv_off, inv_off, (uint64_t)n + 1, st));
  EIM_CUDA(cudaMemcpyAsync(ctx->inv_fill.p, inv_off, ((uint64_t)n + 1) * sizeof(uint64_t), cudaMemcpyDeviceToDevice, st));
  EIM_CUDA(cudaMemcpyAsync(ctx->h_pinned, inv_off + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  const uint64_t total = *static_cast<uint64_t*>(ctx->h_pinned);
  ctx->inv.reserve(std::max<uint64_t>(total, 1) * sizeof(uint32_t), false, st);
  if (num_sets > 0) {
    invert_kernel<<<grid_for(ctx, num_sets * 32, 256), 256, 0, st>>>(
        ctx->arena.as<uint32_t>(), ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>(), num_sets,
        ctx->inv_fill.as<unsigned long long>(), ctx->inv.as<uint32_t>());
    EIM_CUDA(cudaGetLastError());
  }
  // ---- working counts, covered flags, per-pick argmax slots
  ctx->C_work.reserve((uint64_t)n_pad * sizeof(uint32_t), false, st);
  ctx->covered.reserve(std::max<uint64_t>(num_sets, 1), false, st);
  ctx->best.reserve((uint64_t)k * sizeof(unsigned long long), false, st);
  ctx->seeds.reserve((uint64_t)k * sizeof(uint32_t), false, st);
  ctx->gains.reserve((uint64_t)k * sizeof(unsigned long long), false, st);
  uint32_t* W = ctx->C_work.as<uint32_t>();
  init_work_kernel<<<grid_for(ctx, n_pad, 256), 256, 0, st>>>(ctx->C_total.as<uint32_t>(), n, n_pad, W);
  EIM_CUDA(cudaGetLastError());
  EIM_CUDA(cudaMemsetAsync(ctx->covered.p, 0, std::max<uint64_t>(num_sets, 1), st));
  EIM_CUDA(cudaMemsetAsync(ctx->best.p, 0, (uint64_t)k * sizeof(unsigned long long), st));
  ctx->kernel_launches += 5;
  const uint32_t n4 = n_pad / 4;
  constexpr int AB = 256;
  const uint32_t ablocks = grid_for(ctx, n4, AB, 8);
  const uint32_t cblocks = (uint32_t)ctx->sm_count * 8;
  for (uint32_t j = 0; j < k; ++j) {
    argmax_kernel<AB><<<ablocks, AB, 0, st>>>(reinterpret_cast<const uint4*>(W), n4, ctx->seeds.as<uint32_t>(), j,
                                              ctx->best.as<unsigned long long>());
    cover_kernel<<<cblocks, 256, 0, st>>>(j, ctx->best.as<unsigned long long>(), ctx->seeds.as<uint32_t>(),
                                          ctx->gains.as<unsigned long long>(), W, inv_off, ctx->inv.as<uint32_t>(),
                                          ctx->covered.as<uint8_t>(), ctx->set_start.as<uint64_t>(),
                                          ctx->set_len.as<uint32_t>(), ctx->arena.as<uint32_t>());
  }
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches += 2ull * k;
  std::vector<unsigned long long> g(k);
  EIM_CUDA(cudaMemcpyAsync(seeds_out, ctx->seeds.p, (uint64_t)k * sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaMemcpyAsync(g.data(), ctx->gains.p, (uint64_t)k * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  uint64_t cov = 0;
  for (uint32_t j = 0; j < k; ++j) {
    cov += g[j];
    if (gains_out) gains_out[j] = g[j];
  }
  return cov;
}

}  // namespace eim
