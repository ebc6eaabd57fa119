// philox.cuh -- device Philox4x32-10 and the counter layout of reading R1
// (DESIGN.md §3): key = (lo32 seed, hi32 seed); counter =
// (lo32 q, hi32 q, lo32 s, (hi32 s & 0x3FFFFFFF) | tag << 30).
// Tags: EDGE (q = e >> 2, word e & 3), ROOT (q = 0, words 0,1 = r64),
// LT (q = u >> 2, word u & 3).
#pragma once
#include <stdint.h>

namespace eim {

enum : uint32_t { TAG_EDGE = 0u, TAG_ROOT = 1u, TAG_LT = 2u };

// Round keys for one seed: 10 rounds, key bumped by the Weyl constants
// between rounds.  Kept in registers by the caller (loop invariant).
struct PhiloxKey {
  uint32_t k0[10], k1[10];
};

__host__ __device__ __forceinline__ PhiloxKey philox_key(uint64_t seed) {
  PhiloxKey K;
  uint32_t a = (uint32_t)seed, b = (uint32_t)(seed >> 32);
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    K.k0[r] = a;
    K.k1[r] = b;
    a += 0x9E3779B9u;
    b += 0xBB67AE85u;
  }
  return K;
}

__device__ __forceinline__ uint4 philox(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                        const PhiloxKey& K) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    uint32_t lo0 = 0xD2511F53u * c0;
    uint32_t hi0 = __umulhi(0xD2511F53u, c0);
    uint32_t lo1 = 0xCD9E8D57u * c2;
    uint32_t hi1 = __umulhi(0xCD9E8D57u, c2);
    uint32_t n0 = hi1 ^ c1 ^ K.k0[r];
    uint32_t n2 = hi0 ^ c3 ^ K.k1[r];
    c0 = n0;
    c1 = lo1;
    c2 = n2;
    c3 = lo0;
  }
  return make_uint4(c0, c1, c2, c3);
}

// Counter words 2,3 for sample s and a tag.
__device__ __forceinline__ uint32_t ctr_hi(uint64_t s, uint32_t tag) {
  return ((uint32_t)(s >> 32) & 0x3FFFFFFFu) | (tag << 30);
}

__device__ __forceinline__ uint4 philox_at(uint64_t q, uint64_t s, uint32_t tag, const PhiloxKey& K) {
  return philox((uint32_t)q, (uint32_t)(q >> 32), (uint32_t)s, ctr_hi(s, tag), K);
}

__device__ __forceinline__ uint32_t word_of(const uint4& w, uint32_t i) {
  return i == 0 ? w.x : (i == 1 ? w.y : (i == 2 ? w.z : w.w));
}

// Alg. 2 l.6 root: floor(r64 * n / 2^64).
__device__ __forceinline__ uint32_t draw_root(uint64_t s, uint32_t n, const PhiloxKey& K) {
  uint4 w = philox_at(0, s, TAG_ROOT, K);
  uint64_t r64 = (uint64_t)w.x | ((uint64_t)w.y << 32);
  return (uint32_t)__umul64hi(r64, (uint64_t)n);
}

}  // namespace eim
