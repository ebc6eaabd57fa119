// arena.cu -- the RRR arena R with per-set (start, length) (Fig. 2):
// coverage histogram C, canonical export (sets in sample-id order,
// each ascending) and appending sets received from other ranks.
#include <cub/cub.cuh>

#include "arena_view.cuh"

namespace eim {

namespace {

constexpr unsigned FULL_MASK = 0xFFFFFFFFu;

// One warp per set: C[x] += d for every member x (sets have no duplicates);
// d = 1 adds sets [lo, hi) to the histogram, d = -1 removes them.
__global__ void hist_kernel(const uint32_t* __restrict__ arena, uint32_t ab, const uint64_t* __restrict__ set_start,
                            const uint32_t* __restrict__ set_len, uint64_t lo, uint64_t hi,
                            uint32_t* __restrict__ C, uint32_t d) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t i = lo + warp; i < hi; i += nwarps) {
    const uint64_t st = set_start[i];
    const uint32_t L = set_len[i];
    for (uint32_t t = lane; t < L; t += 32) atomicAdd(&C[arena_get(arena, st + t, ab)], d);
  }
}

// Examined in-edges (IC: sum of d^-(v) over the members -- every member was
// expanded once) or walk steps (LT: |set| - 1, plus the final step unless
// the walk ended at a vertex without in-edges) of sets [lo, hi).
__global__ void set_edges_kernel(const uint32_t* __restrict__ arena, uint32_t ab, const uint64_t* __restrict__ set_start,
                                 const uint32_t* __restrict__ set_len, uint64_t lo, uint64_t hi,
                                 const uint64_t* __restrict__ off, bool ic, unsigned long long* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  unsigned long long e = 0;
  for (uint64_t i = lo + warp; i < hi; i += nwarps) {
    const uint64_t st = set_start[i];
    const uint32_t L = set_len[i];
    unsigned long long s = 0;
    bool sink = false;
    for (uint32_t t = lane; t < L; t += 32) {
      const uint32_t v = arena_get(arena, st + t, ab);
      const uint64_t d = off[v + 1] - off[v];
      s += d;
      sink |= d == 0;
    }
    const bool any_sink = __any_sync(FULL_MASK, sink);  // i is warp-uniform
    if (ic) e += s;
    else if (lane == 0) e += (unsigned long long)L - (any_sink ? 1u : 0u);
  }
  for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(FULL_MASK, e, o);
  if (lane == 0 && e) atomicAdd(out, e);
}

__global__ void len_to_u64_kernel(const uint32_t* __restrict__ len, uint64_t lo, uint64_t count,
                                  uint64_t* __restrict__ out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= count; i += stride)
    out[i] = i < count ? (uint64_t)len[lo + i] : 0ull;
}

// One warp per set: copy arena[set_start[lo+i] ..] to out[offsets[i] ..].
__global__ void gather_kernel(const uint32_t* __restrict__ arena, uint32_t ab, const uint64_t* __restrict__ set_start,
                              const uint32_t* __restrict__ set_len, uint64_t lo, uint64_t count,
                              const uint64_t* __restrict__ offsets, uint32_t* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t i = warp; i < count; i += nwarps) {
    const uint64_t src = set_start[lo + i], dst = offsets[i];
    const uint32_t L = set_len[lo + i];
    for (uint32_t t = lane; t < L; t += 32) out[dst + t] = arena_get(arena, src + t, ab);
  }
}

// Append canonical sets: members go to arena[base_elem + offsets[i] ..].
__global__ void place_kernel(const uint64_t* __restrict__ offsets, uint64_t count, uint64_t base_set,
                             uint64_t base_elem, uint64_t* __restrict__ set_start,
                             uint32_t* __restrict__ set_len) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
    set_start[base_set + i] = base_elem + offsets[i];
    set_len[base_set + i] = (uint32_t)(offsets[i + 1] - offsets[i]);
  }
}

// Append encoded: arena element base + j <- members[j].
__global__ void put_kernel(const uint32_t* __restrict__ members, uint64_t total, uint32_t* arena, uint32_t ab,
                           uint64_t base) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < total; j += stride)
    arena_put(arena, base + j, ab, members[j]);
}

}  // namespace

void hist_sets(eim_ctx* ctx, uint64_t lo, uint64_t hi, int sign) {
  if (hi <= lo) return;
  hist_kernel<<<grid_for(ctx, (hi - lo) * 32, 256), 256, 0, ctx->stream>>>(
      ctx->arena.as<uint32_t>(), ctx->arena_b, ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>(), lo, hi,
      ctx->C_total.as<uint32_t>(), sign < 0 ? 0xFFFFFFFFu : 1u);
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches++;
}

void drop_sets(eim_ctx* ctx, const eim_graph* g, bool ic, uint64_t keep, uint64_t R, uint64_t* edges) {
  *edges = 0;
  if (R <= keep) return;
  if (!g->view.off) fail(EIM_E_STATE, "drop_sets needs the plain offsets of the graph");
  cudaStream_t st = ctx->stream;
  hist_sets(ctx, keep, R, -1);
  unsigned long long* d = reinterpret_cast<unsigned long long*>(static_cast<char*>(ctx->h_pinned) + 2048);
  ctx->stage_a.reserve(64, false, st);
  unsigned long long* dd = ctx->stage_a.as<unsigned long long>();
  EIM_CUDA(cudaMemsetAsync(dd, 0, sizeof(unsigned long long), st));
  set_edges_kernel<<<grid_for(ctx, (R - keep) * 32, 256), 256, 0, st>>>(
      ctx->arena.as<uint32_t>(), ctx->arena_b, ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>(), keep, R,
      g->view.off, ic, dd);
  EIM_CUDA(cudaGetLastError());
  EIM_CUDA(cudaMemcpyAsync(d, dd, sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaMemcpyAsync(d + 1, ctx->set_start.as<uint64_t>() + keep, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  ctx->kernel_launches += 2;
  *edges = d[0];
  ctx->arena_used = d[1];  // the dropped sets were appended after every kept one
}

// Compacts sets [lo, lo+count) (set indices) into stage_a (offsets, u64) and
// stage_b (members).  Returns the member total.  sort: ascending within sets.
static uint64_t compact_sets(eim_ctx* ctx, uint64_t lo, uint64_t count, bool sort, uint64_t** d_offsets,
                             uint32_t** d_members, uint64_t sort_cap = UINT64_MAX) {
  cudaStream_t st = ctx->stream;
  ctx->stage_a.reserve((count + 1) * sizeof(uint64_t), false, st);
  uint64_t* offs = ctx->stage_a.as<uint64_t>();
  len_to_u64_kernel<<<grid_for(ctx, count + 1, 256), 256, 0, st>>>(ctx->set_len.as<uint32_t>(), lo, count, offs);
  EIM_CUDA(cudaGetLastError());
  size_t tmp = 0;
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, offs, offs, count + 1, st));
  ctx->scratch.reserve(std::max<size_t>(tmp, 1 << 20), false, st);
  EIM_CUDA(cub::DeviceScan::ExclusiveSum(ctx->scratch.p, tmp, offs, offs, count + 1, st));
  uint64_t total = 0;
  EIM_CUDA(cudaMemcpyAsync(ctx->h_pinned, offs + count, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  total = *static_cast<uint64_t*>(ctx->h_pinned);
  if (total > sort_cap) {  // the members are not wanted (capacity exceeded): offsets only
    *d_offsets = offs;
    *d_members = nullptr;
    return total;
  }
  ctx->stage_b.reserve(std::max<uint64_t>(total, 1) * sizeof(uint32_t), false, st);
  uint32_t* out = ctx->stage_b.as<uint32_t>();
  if (count > 0) {
    gather_kernel<<<grid_for(ctx, count * 32, 256), 256, 0, st>>>(
        ctx->arena.as<uint32_t>(), ctx->arena_b, ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>(), lo,
        count, offs, out);
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
  }
  ctx->kernel_launches += 1;
  if (sort && total > 0) {
    if (total > (uint64_t)INT32_MAX || count > (uint64_t)INT32_MAX)
      fail(EIM_E_CAPACITY, "export larger than 2^31 members is not supported");
    ctx->stage_c.reserve(total * sizeof(uint32_t), false, st);
    uint32_t* sorted = ctx->stage_c.as<uint32_t>();
    size_t tmp2 = 0;
    EIM_CUDA(cub::DeviceSegmentedSort::SortKeys(nullptr, tmp2, out, sorted, (int)total, (int)count, offs,
                                                 offs + 1, st));
    ctx->scratch.reserve(std::max<size_t>(tmp2, 1 << 20), false, st);
    EIM_CUDA(cub::DeviceSegmentedSort::SortKeys(ctx->scratch.p, tmp2, out, sorted, (int)total, (int)count,
                                                 offs, offs + 1, st));
    ctx->kernel_launches += 2;
    out = sorted;
  }
  *d_offsets = offs;
  *d_members = out;
  return total;
}

uint64_t export_sets(eim_ctx* ctx, uint64_t count, uint64_t** d_offsets, uint32_t** d_members, uint64_t members_cap) {
  // members that will not be copied out (more than members_cap) need no sort
  return compact_sets(ctx, 0, count, true, d_offsets, d_members, members_cap);
}

uint64_t compact_range(eim_ctx* ctx, uint64_t lo, uint64_t count, uint64_t** d_offsets, uint32_t** d_members) {
  return compact_sets(ctx, lo, count, false, d_offsets, d_members);
}

void append_sets(eim_ctx* ctx, uint64_t base, uint64_t count, const uint64_t* d_offsets,
                 const uint32_t* d_members, uint64_t total) {
  cudaStream_t st = ctx->stream;
  if (count == 0) return;
  ensure_sets(ctx, base + count);
  uint64_t cur = arena_cursor(ctx);
  arena_ensure(ctx, cur + total);
  if (total && ctx->arena_b == 32)
    EIM_CUDA(cudaMemcpyAsync(ctx->arena.as<uint32_t>() + cur, d_members, total * sizeof(uint32_t),
                             cudaMemcpyDeviceToDevice, st));
  else if (total) {
    put_kernel<<<grid_for(ctx, total, 256), 256, 0, st>>>(d_members, total, ctx->arena.as<uint32_t>(), ctx->arena_b,
                                                          cur);
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches++;
  }
  place_kernel<<<grid_for(ctx, count, 256), 256, 0, st>>>(d_offsets, count, base, cur,
                                                           ctx->set_start.as<uint64_t>(), ctx->set_len.as<uint32_t>());
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches++;
  ctx->arena_used = cur + total;
}

}  // namespace eim
