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

// 32x32 -> 64 product as one wide multiply (IMAD.WIDE.U32).  Written as
// inline PTX so the compiler cannot split it into IMAD.HI + IMAD or
// strength-reduce a loop-carried operand into separate halves.
__device__ __forceinline__ uint64_t mulw(uint32_t a, uint32_t b) {
  uint64_t r;
  asm("mul.wide.u32 %0, %1, %2;" : "=l"(r) : "r"(a), "r"(b));
  return r;
}

__device__ __forceinline__ uint4 philox(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                        const PhiloxKey& K) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint64_t p0 = mulw(0xD2511F53u, c0), p1 = mulw(0xCD9E8D57u, c2);
    const uint32_t n0 = (uint32_t)(p1 >> 32) ^ c1 ^ K.k0[r];
    const uint32_t n2 = (uint32_t)(p0 >> 32) ^ c3 ^ K.k1[r];
    c0 = n0;
    c1 = (uint32_t)p1;
    c2 = n2;
    c3 = (uint32_t)p0;
  }
  return make_uint4(c0, c1, c2, c3);
}

// Counter words 2,3 for sample s and a tag.
__device__ __forceinline__ uint32_t ctr_hi(uint64_t s, uint32_t tag) {
  return ((uint32_t)(s >> 32) & 0x3FFFFFFFu) | (tag << 30);
}

// EDGE draws of one sample with the quad's high word fixed: counter
// (c0, c1, s_lo, ctr_hi(s, EDGE)) with only c0 varying.  In round 0 the
// product M1*c2 and the word hi1^c1^k0 are constants, and so is round 1's
// product M0*c0, so a call needs 18 instead of 20 wide multiplies.  The
// result is exactly philox(c0, c1, c2, c3, K).
struct EdgeConsts {
  uint32_t x0;  // round 0: c3 ^ k1[0]
  uint32_t a;   // round 1 input word 0: hi(M1*c2) ^ c1 ^ k0[0]
  uint32_t y1;  // round 1: lo(M1*c2) ^ k0[1]
  uint32_t z1;  // round 1: hi(M0*a) ^ k1[1]
  uint32_t l1;  // round 1 output word 3: lo(M0*a)
};

__device__ __forceinline__ EdgeConsts edge_consts(uint32_t c1, uint32_t c2, uint32_t c3, const PhiloxKey& K) {
  EdgeConsts E;
  const uint32_t lo1 = 0xCD9E8D57u * c2, hi1 = __umulhi(0xCD9E8D57u, c2);
  E.x0 = c3 ^ K.k1[0];
  E.a = hi1 ^ c1 ^ K.k0[0];
  E.y1 = lo1 ^ K.k0[1];
  E.z1 = __umulhi(0xD2511F53u, E.a) ^ K.k1[1];
  E.l1 = 0xD2511F53u * E.a;
  return E;
}

__device__ __forceinline__ uint4 philox_edge(uint32_t c0, const EdgeConsts& E, const PhiloxKey& K) {
  // round 0: (a, lo(M1*c2), hi(M0*c0) ^ c3 ^ k1[0], lo(M0*c0))
  const uint64_t q0 = mulw(0xD2511F53u, c0);
  const uint32_t r0c2 = (uint32_t)(q0 >> 32) ^ E.x0;
  // round 1
  const uint64_t q1 = mulw(0xCD9E8D57u, r0c2);
  uint32_t x0 = (uint32_t)(q1 >> 32) ^ E.y1;
  uint32_t x1 = (uint32_t)q1;
  uint32_t x2 = (uint32_t)q0 ^ E.z1;
  uint32_t x3 = E.l1;
#pragma unroll
  for (int r = 2; r < 10; ++r) {
    const uint64_t p0 = mulw(0xD2511F53u, x0), p1 = mulw(0xCD9E8D57u, x2);
    x0 = (uint32_t)(p1 >> 32) ^ x1 ^ K.k0[r];
    x2 = (uint32_t)(p0 >> 32) ^ x3 ^ K.k1[r];
    x1 = (uint32_t)p1;
    x3 = (uint32_t)p0;
  }
  return make_uint4(x0, x1, x2, x3);
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
