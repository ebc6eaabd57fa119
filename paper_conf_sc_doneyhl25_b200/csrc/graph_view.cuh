// graph_view.cuh -- device accessors of the graph stores, so every kernel
// that walks the reverse CSR is written once and instantiated for the plain
// store (GraphView: u64 offsets, u32 neighbours, u32 thresholds), the
// log-encoded store (PackedGraphView, layout R24), the store with
// general edge probabilities (WeightedGraphView, R25) and both at once
// (PackedWeightedGraphView).
#pragma once
#include "eim_internal.h"

namespace eim {

// read-only path (ld.global.nc): the store never changes while a kernel runs,
// and the loads may be issued ahead of the membership-table atomics
__device__ __forceinline__ uint64_t g_off(const GraphView& g, uint64_t v) { return __ldg(g.off + v); }
__device__ __forceinline__ uint32_t g_nbr(const GraphView& g, uint64_t e) { return __ldg(g.nbr + e); }
__device__ __forceinline__ uint32_t g_thr(const GraphView& g, uint32_t v, uint64_t /*d*/) { return g.thr[v]; }

// Value j of a log-encoded array (R24): bits [j b, (j+1) b) of the
// little-endian bit stream; b <= 32 spans at most two containers.
__device__ __forceinline__ uint32_t log_decode32(const uint32_t* __restrict__ w, uint64_t j, uint32_t b) {
  const uint64_t t = j * b;
  const uint64_t i = t >> 5;
  const uint32_t x = __funnelshift_r(__ldg(w + i), __ldg(w + i + 1), (uint32_t)t & 31u);
  return b >= 32 ? x : x & ((1u << b) - 1u);
}

// b <= 64: up to three containers.
__device__ __forceinline__ uint64_t log_decode64(const uint32_t* __restrict__ w, uint64_t j, uint32_t b) {
  const uint64_t t = j * b;
  const uint64_t i = t >> 5;
  const uint32_t sh = (uint32_t)t & 31u;
  uint64_t x = (((uint64_t)__ldg(w + i + 1) << 32) | __ldg(w + i)) >> sh;
  if (b + sh > 64) x |= (uint64_t)__ldg(w + i + 2) << (64 - sh);
  return b >= 64 ? x : x & ((1ull << b) - 1ull);
}

__device__ __forceinline__ uint64_t g_off(const PackedGraphView& g, uint64_t v) {
  return g.boff <= 32 ? (uint64_t)log_decode32(g.offw, v, g.boff) : log_decode64(g.offw, v, g.boff);
}
__device__ __forceinline__ uint32_t g_nbr(const PackedGraphView& g, uint64_t e) { return log_decode32(g.nbrw, e, g.bnbr); }
// weighted cascade: T_v = floor((2^32-1)/d), as graph.cu stores it for the plain store (R2)
__device__ __forceinline__ uint32_t g_thr(const PackedGraphView&, uint32_t, uint64_t d) {
  return (d == 0 || d > 0xFFFFFFFFull) ? 0u : 0xFFFFFFFFu / (uint32_t)d;
}

__device__ __forceinline__ uint64_t g_off(const WeightedGraphView& g, uint64_t v) { return __ldg(g.off + v); }
__device__ __forceinline__ uint32_t g_nbr(const WeightedGraphView& g, uint64_t e) { return __ldg(g.nbr + e); }
__device__ __forceinline__ uint32_t g_thr(const WeightedGraphView&, uint32_t, uint64_t) { return 0u; }

__device__ __forceinline__ uint64_t g_off(const PackedWeightedGraphView& g, uint64_t v) { return g_off(g.p, v); }
__device__ __forceinline__ uint32_t g_nbr(const PackedWeightedGraphView& g, uint64_t e) { return g_nbr(g.p, e); }
__device__ __forceinline__ uint32_t g_thr(const PackedWeightedGraphView&, uint32_t, uint64_t) { return 0u; }

// L2 prefetch of in_nbr[e] (no register result, so the sweep does not wait)
__device__ __forceinline__ void l2_prefetch(const void* p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }
__device__ __forceinline__ void g_prefetch_nbr(const GraphView& g, uint64_t e) { l2_prefetch(g.nbr + e); }
__device__ __forceinline__ void g_prefetch_nbr(const WeightedGraphView& g, uint64_t e) { l2_prefetch(g.nbr + e); }
__device__ __forceinline__ void g_prefetch_nbr(const PackedGraphView& g, uint64_t e) {
  l2_prefetch(g.nbrw + ((e * g.bnbr) >> 5));
}
__device__ __forceinline__ void g_prefetch_nbr(const PackedWeightedGraphView& g, uint64_t e) { g_prefetch_nbr(g.p, e); }

// ---- IC liveness of the 4 edges of Philox quad q (words w): edge 4q+i is
// live iff w_i <= its threshold.  Weighted cascade: one threshold T per row.
template <class GV>
__device__ __forceinline__ uint32_t quad_live_mask(const GV&, uint64_t, uint32_t T, const uint4& w) {
  return (w.x <= T ? 1u : 0u) | (w.y <= T ? 2u : 0u) | (w.z <= T ? 4u : 0u) | (w.w <= T ? 8u : 0u);
}
template <class GV>
__device__ __forceinline__ bool quad_any_live(const GV&, uint64_t, uint32_t T, const uint4& w) {
  return min(min(w.x, w.y), min(w.z, w.w)) <= T;
}
// general probabilities: the quad's 4 thresholds in one 16-byte load
__device__ __forceinline__ uint32_t quad_live_mask_x(const uint32_t* x, uint64_t q, const uint4& w) {
  const uint4 t = __ldg(reinterpret_cast<const uint4*>(x) + q);
  return (w.x <= t.x ? 1u : 0u) | (w.y <= t.y ? 2u : 0u) | (w.z <= t.z ? 4u : 0u) | (w.w <= t.w ? 8u : 0u);
}
__device__ __forceinline__ uint32_t quad_live_mask(const WeightedGraphView& g, uint64_t q, uint32_t, const uint4& w) {
  return quad_live_mask_x(g.x, q, w);
}
__device__ __forceinline__ bool quad_any_live(const WeightedGraphView& g, uint64_t q, uint32_t, const uint4& w) {
  return quad_live_mask_x(g.x, q, w) != 0u;
}
__device__ __forceinline__ uint32_t quad_live_mask(const PackedWeightedGraphView& g, uint64_t q, uint32_t,
                                                   const uint4& w) {
  return quad_live_mask_x(g.x, q, w);
}
__device__ __forceinline__ bool quad_any_live(const PackedWeightedGraphView& g, uint64_t q, uint32_t, const uint4& w) {
  return quad_live_mask_x(g.x, q, w) != 0u;
}

// ---- LT choice in row [e0, e1) for threshold tau: the offset j of the
// chosen in-edge, or ~0 when no in-neighbour is chosen.  Weighted cascade
// (R4): j = floor(tau d / 2^32).
template <class GV>
__device__ __forceinline__ uint64_t lt_choose(const GV&, uint64_t e0, uint64_t e1, uint32_t tau) {
  return __umul64hi((unsigned long long)tau << 32, e1 - e0);
}
// general weights (R25): first e with cum_e >= tau (binary search; cum is
// strictly increasing within the row)
__device__ __forceinline__ uint64_t lt_choose_cum(const uint32_t* cum, uint64_t e0, uint64_t e1, uint32_t tau) {
  if (cum[e1 - 1] < tau) return ~0ull;
  uint64_t lo = e0, hi = e1 - 1;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (cum[mid] >= tau) hi = mid;
    else lo = mid + 1;
  }
  return lo - e0;
}
__device__ __forceinline__ uint64_t lt_choose(const WeightedGraphView& g, uint64_t e0, uint64_t e1, uint32_t tau) {
  return lt_choose_cum(g.cum, e0, e1, tau);
}
__device__ __forceinline__ uint64_t lt_choose(const PackedWeightedGraphView& g, uint64_t e0, uint64_t e1,
                                              uint32_t tau) {
  return lt_choose_cum(g.cum, e0, e1, tau);
}

}  // namespace eim
