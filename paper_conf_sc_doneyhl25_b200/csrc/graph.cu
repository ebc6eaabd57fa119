// graph.cu -- device reverse-CSR store (CSC of offsets, in-neighbours,
// weights).  Weights are never stored: under weighted cascade every in-edge of
// v shares p = 1/d^-(v), so one integer threshold per vertex,
// T_v = floor((2^32-1)/d), decides liveness as draw <= T_v (reading R2).


#include "graph_view.cuh"

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

// Any edge u -> v with u != v?  A warp per row; stops early once found.
template <class GV>
__global__ void proper_edge_kernel(GV g, uint32_t n, unsigned int* found) {
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t v = warp; v < n; v += nwarps) {
    if (*(volatile unsigned int*)found) return;
    unsigned int f = 0;
    const uint64_t e1 = g_off(g, v + 1);
    for (uint64_t e = g_off(g, v) + lane; e < e1 && !f; e += 32) f = g_nbr(g, e) != (uint32_t)v;
    if (__any_sync(0xFFFFFFFFu, f)) {
      if (lane == 0) atomicOr(found, 1u);
      return;
    }
  }
}

// Log encoding (layout R24): container i holds stream bits
// [32 i, 32 i + 32); one thread per container ORs in the values that overlap
// it, so no two threads write the same word.  Containers past the data (the
// padding) are zero.
template <class T>
__global__ void log_encode_kernel(const T* __restrict__ x, uint64_t count, uint32_t b, uint32_t* __restrict__ w,
                                  uint64_t nwords) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t data_words = (count * b + 31) / 32;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nwords; i += stride) {
    uint32_t word = 0;
    if (i < data_words) {
      const uint64_t t0 = 32 * i;
      const uint64_t j0 = t0 / b, j1 = min((t0 + 31) / b, count - 1);
      for (uint64_t j = j0; j <= j1; ++j) {
        const int64_t sh = (int64_t)(j * b) - (int64_t)t0;  // value j starts at bit sh of this word
        const uint64_t v = (uint64_t)x[j];
        word |= (uint32_t)(sh >= 0 ? (v << sh) : (v >> -sh));
      }
    }
    w[i] = word;
  }
}

__global__ void max_of_kernel(const uint32_t* __restrict__ x, uint64_t count, unsigned int* out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  uint32_t m = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) m = max(m, x[i]);
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(0xFFFFFFFFu, m, o));
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}

// LT cumulative weights (R25): one warp per row, inclusive scan of
// w = x + 1 in 64 bits; cum = scan - 1.  A row whose sum exceeds 2^32
// (sum p > 1) raises *bad (LT is then rejected on this graph).
__global__ void lt_cum_kernel(const uint64_t* __restrict__ off, const uint32_t* __restrict__ x, uint32_t n,
                              uint32_t* __restrict__ cum, unsigned int* bad) {
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t v = warp; v < n; v += nwarps) {
    const uint64_t e0 = off[v], e1 = off[v + 1];
    unsigned long long carry = 0;
    for (uint64_t b = e0; b < e1; b += 32) {
      const uint64_t e = b + lane;
      unsigned long long s = e < e1 ? (unsigned long long)x[e] + 1ull : 0ull;
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long t = __shfl_up_sync(0xFFFFFFFFu, s, o);
        if (lane >= (uint32_t)o) s += t;
      }
      s += carry;
      if (e < e1) {
        if (s > (1ull << 32)) atomicOr(bad, 1u);
        cum[e] = s > (1ull << 32) ? 0xFFFFFFFFu : (uint32_t)(s - 1ull);
      }
      carry = __shfl_sync(0xFFFFFFFFu, s, 31);
    }
  }
}

}  // namespace

void graph_attach_weights(eim_ctx* ctx, eim_graph* g, const uint32_t* h_x) {
  cudaStream_t st = ctx->stream;
  const uint64_t m = g->view.m, m4 = (m + 3) / 4 * 4 + 4;
  EIM_CUDA(cudaMallocAsync(&g->d_x, m4 * sizeof(uint32_t), st));
  EIM_CUDA(cudaMallocAsync(&g->d_cum, std::max<uint64_t>(m, 1) * sizeof(uint32_t), st));
  EIM_CUDA(cudaMemsetAsync(g->d_x, 0, m4 * sizeof(uint32_t), st));
  if (m) EIM_CUDA(cudaMemcpyAsync(g->d_x, h_x, m * sizeof(uint32_t), cudaMemcpyHostToDevice, st));
  ctx->scratch.reserve(1 << 20, false, st);
  unsigned int* d_bad = reinterpret_cast<unsigned int*>(ctx->scratch.p);
  EIM_CUDA(cudaMemsetAsync(d_bad, 0, sizeof(unsigned int), st));
  lt_cum_kernel<<<grid_for(ctx, (uint64_t)g->view.n * 32, 256), 256, 0, st>>>(
      g->view.off, static_cast<const uint32_t*>(g->d_x), g->view.n, static_cast<uint32_t*>(g->d_cum), d_bad);
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches++;
  unsigned int* h = static_cast<unsigned int*>(ctx->h_pinned);
  EIM_CUDA(cudaMemcpyAsync(h, d_bad, sizeof(unsigned int), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  g->lt_ok = *h == 0;
  g->weighted = true;
  g->wview = WeightedGraphView{g->view.n, m, g->view.off, g->view.nbr, static_cast<const uint32_t*>(g->d_x),
                               static_cast<const uint32_t*>(g->d_cum)};
  g->bytes += (m4 + std::max<uint64_t>(m, 1)) * sizeof(uint32_t);
}

uint32_t bit_width(uint64_t x) {
  uint32_t b = 0;
  while (b < 64 && (x >> b) != 0) b++;
  return b;
}

void graph_log_encode(eim_ctx* ctx, eim_graph* g) {
  cudaStream_t st = ctx->stream;
  const uint32_t n = g->view.n;
  const uint64_t m = g->view.m;
  // n_b = bit_width(x_max) (R19): offsets top out at m; neighbours at their max
  ctx->scratch.reserve(1 << 20, false, st);
  unsigned int* d_max = reinterpret_cast<unsigned int*>(ctx->scratch.p);
  EIM_CUDA(cudaMemsetAsync(d_max, 0, sizeof(unsigned int), st));
  if (m) max_of_kernel<<<grid_for(ctx, m, 256), 256, 0, st>>>(g->view.nbr, m, d_max);
  EIM_CUDA(cudaGetLastError());
  unsigned int* h = static_cast<unsigned int*>(ctx->h_pinned);
  EIM_CUDA(cudaMemcpyAsync(h, d_max, sizeof(unsigned int), cudaMemcpyDeviceToHost, st));
  EIM_CUDA(cudaStreamSynchronize(st));
  const uint32_t boff = bit_width(m), bnbr = bit_width(*h);
  const uint64_t woff = ((uint64_t)(n + 1) * boff + 31) / 32 + 2, wnbr = (m * bnbr + 31) / 32 + 2;
  EIM_CUDA(cudaMallocAsync(&g->d_offw, woff * sizeof(uint32_t), st));
  EIM_CUDA(cudaMallocAsync(&g->d_nbrw, wnbr * sizeof(uint32_t), st));
  log_encode_kernel<uint64_t><<<grid_for(ctx, woff, 256), 256, 0, st>>>(g->view.off, (uint64_t)n + 1, boff,
                                                                        static_cast<uint32_t*>(g->d_offw), woff);
  EIM_CUDA(cudaGetLastError());
  if (bnbr)
    log_encode_kernel<uint32_t><<<grid_for(ctx, wnbr, 256), 256, 0, st>>>(g->view.nbr, m, bnbr,
                                                                          static_cast<uint32_t*>(g->d_nbrw), wnbr);
  else
    EIM_CUDA(cudaMemsetAsync(g->d_nbrw, 0, wnbr * sizeof(uint32_t), st));
  EIM_CUDA(cudaGetLastError());
  ctx->kernel_launches += 3;
  g->pview = PackedGraphView{n, m, static_cast<const uint32_t*>(g->d_offw), static_cast<const uint32_t*>(g->d_nbrw),
                             boff, bnbr};
  g->packed = true;
  const uint64_t wbytes = g->weighted ? g->bytes - ((uint64_t)(n + 1) * sizeof(uint64_t) +
                                                    std::max<uint64_t>(m, 4) * sizeof(uint32_t) + (uint64_t)n * sizeof(uint32_t))
                                      : 0;
  if (g->weighted)  // the probabilities stay 32-bit next to the packed offsets and neighbours
    g->pwview = PackedWeightedGraphView{n, m, g->pview, static_cast<const uint32_t*>(g->d_x),
                                        static_cast<const uint32_t*>(g->d_cum)};
  // the plain store is gone: only the packed view may be used from here on
  EIM_CUDA(cudaFreeAsync(g->d_off, st));
  EIM_CUDA(cudaFreeAsync(g->d_nbr, st));
  EIM_CUDA(cudaFreeAsync(g->d_thr, st));
  g->d_off = g->d_nbr = g->d_thr = nullptr;
  g->view.off = nullptr;
  g->view.nbr = nullptr;
  g->view.thr = nullptr;
  g->bytes = (woff + wnbr) * sizeof(uint32_t) + wbytes;
  EIM_CUDA(cudaStreamSynchronize(st));
}

// Source elimination needs a graph on which some set can be non-empty (R22).
bool graph_has_proper_edge(eim_ctx* ctx, const eim_graph* g) {
  if (g->proper_edge < 0) {
    cudaStream_t st = ctx->stream;
    ctx->scratch.reserve(1 << 20, false, st);
    unsigned int* d = reinterpret_cast<unsigned int*>(ctx->scratch.p);
    EIM_CUDA(cudaMemsetAsync(d, 0, sizeof(unsigned int), st));
    const uint32_t grid = grid_for(ctx, (uint64_t)g->view.n * 32, 256);
    with_graph_view(g, [&](const auto& gv) { proper_edge_kernel<<<grid, 256, 0, st>>>(gv, g->view.n, d); });
    EIM_CUDA(cudaGetLastError());
    ctx->kernel_launches += 1;
    unsigned int* h = static_cast<unsigned int*>(ctx->h_pinned);
    EIM_CUDA(cudaMemcpyAsync(h, d, sizeof(unsigned int), cudaMemcpyDeviceToHost, st));
    EIM_CUDA(cudaStreamSynchronize(st));
    const_cast<eim_graph*>(g)->proper_edge = *h ? 1 : 0;
  }
  return g->proper_edge == 1;
}

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
