// arena_view.cuh -- element access to the RRR arena R, plain (b = 32)
// or log-encoded (b < 32, layout R24).  Encoded writes OR the
// element's bits into one or two zeroed containers with atomicOr, so writers
// of neighbouring elements never lose each other's bits.
#pragma once
#include "graph_view.cuh"

namespace eim {

__device__ __forceinline__ uint32_t arena_get(const uint32_t* __restrict__ a, uint64_t j, uint32_t b) {
  return b == 32 ? a[j] : log_decode32(a, j, b);
}

__device__ __forceinline__ void arena_put(uint32_t* a, uint64_t j, uint32_t b, uint32_t v) {
  if (b == 32) {
    a[j] = v;
    return;
  }
  const uint64_t t = j * b;
  const uint64_t i = t >> 5;
  const uint32_t sh = (uint32_t)t & 31u;
  atomicOr(a + i, v << sh);
  if (sh + b > 32) atomicOr(a + i + 1, v >> (32 - sh));
}

}  // namespace eim
