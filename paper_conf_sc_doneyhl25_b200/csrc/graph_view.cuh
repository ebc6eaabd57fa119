// graph_view.cuh -- device accessors of the two graph stores, so every
// kernel that walks the reverse CSR is written once and instantiated for the
// plain store (GraphView: u64 offsets, u32 neighbours, u32 thresholds) and
// the log-encoded store (PackedGraphView, layout R24).
#pragma once
#include "eim_internal.h"

namespace eim {

__device__ __forceinline__ uint64_t g_off(const GraphView& g, uint64_t v) { return g.off[v]; }
__device__ __forceinline__ uint32_t g_nbr(const GraphView& g, uint64_t e) { return g.nbr[e]; }
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

}  // namespace eim
