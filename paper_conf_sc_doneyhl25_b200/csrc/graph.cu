// graph.cu -- device reverse-CSR store (CSC of offsets, in-neighbours,
// weights).  Weights are never stored: under weighted cascade every in-edge of
// v shares p = 1/d^-(v), so one integer threshold per vertex,
// T_v = floor((2^32-1)/d), decides liveness as draw <= T_v (reading R2).
#include "eim_internal.h"

namespace eim {

namespace {

__global__ void validate_kernel(const uint64_t* __restrict__ off, const uint32_t* __restrict__ nbr,
                                uint32_t n, uint64_t m, unsigned int* bad) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t v = tid; v < n; v += stride)
    if (off[v] > off[v + 1]) atomicOr(bad, 1u);
  // in_neighbors < n, four per thread-iteration
  const uint64_t m4 = m / 4;
  const uint4* nbr4 = reinterpret_cast<const uint4*>(nbr);
  unsigned int flag = 0;
  for (uint64_t i = tid; i < m4; i += stride) {
    uint4 x = nbr4[i];
    flag |= (x.x >= n) | (x.y >= n) | (x.z >= n) | (x.w >= n);
  }
  for (uint64_t i = m4 * 4 + tid; i < m; i += stride) flag |= nbr[i] >= n;
  if (__any_sync(0xFFFFFFFFu, flag) && (threadIdx.x & 31) == 0) atomicOr(bad, 2u);
}

__global__ void threshold_kernel(const uint64_t* __restrict__ off, uint32_t n, uint32_t* __restrict__ thr) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
    const uint64_t d = off[v + 1] - off[v];
    thr[v] = (d == 0 || d > 0xFFFFFFFFull) ? 0u : 0xFFFFFFFFu / (uint32_t)d;
  }
}

}  // namespace

void graph_validate_and_thresholds(eim_ctx* ctx, eim_graph* g) {
  cudaStream_t st = ctx->stream;
  unsigned int* d_bad = reinterpret_cast<unsigned int*>(ctx->scratch.p);
  EIM_CUDA(cudaMemsetAsync(d_bad, 0, sizeof(unsigned int), st));
  const GraphView& v = g->view;
  // the u4 path reads nbr in 16-byte units: the allocation is 16-byte aligned
  validate_kernel<<<ctx->sm_count * 8, 256, 0, st>>>(v.off, v.nbr, v.n, v.m, d_bad);
  EIM_CUDA(cudaGetLastError());
  threshold_kernel<<<grid_for(ctx, v.n, 256), 256, 0, st>>>(v.off, v.n, const_cast<uint32_t*>(v.thr));
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches += 2;
  unsigned int* h = static_cast<unsigned int*>(ctx->h_pinned);
  uint64_t* h64 = reinterpret_cast<uint64_t*>(static_cast<char*>(ctx->h_pinned) + 64);
  EIM_CUDA(cudaMemcpyAsync(h, d_bad, sizeof(unsigned int), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaMemcpyAsync(h64, v.off, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaMemcpyAsync(h64 + 1, v.off + v.n, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  if (h64[0] != 0) fail(EIM_E_INVAL, "in_offsets[0] != 0");
  if (h64[1] != v.m) fail(EIM_E_INVAL, "in_offsets[n] != m");
  if (*h & 1u) fail(EIM_E_INVAL, "in_offsets is not non-decreasing");
  if (*h & 2u) fail(EIM_E_INVAL, "an in_neighbors entry is >= n");
}

}  // namespace eim
