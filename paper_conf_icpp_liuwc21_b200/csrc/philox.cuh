// philox.cuh — counter-based random weights in registers.
//
// The paper materialises two n x d random matrices L, G per iteration with
// Thrust (Sec 3.1; Eq. 4, L and G at P:L195-211) — 16 B of HBM
// traffic per element (write + read).  Here every weight is recomputed from
// (seed, t, particle, dim) by Philox4x32-10 in registers: 0 B of HBM.
// One call yields the 4 weights of one float4 of dimensions for one tag.
//
// Stream layout (reading 6):
//   word(tag, t, i, j) = Philox4x32-10(ctr = {j>>2, i, t, tag}, key = {seed lo, seed hi})[j&3]
//   tags: R1 = 0 (l_ij of Eq. 1), R2 = 1 (g_ij), X0 = 2, V0 = 3 (init, t = 0)
//   U(w) = (w >> 8) * 2^-24  in [0, 1 - 2^-24]  (reading 5)
#pragma once
#include <cstdint>

namespace fastpso {

enum : uint32_t { kTagR1 = 0, kTagR2 = 1, kTagX0 = 2, kTagV0 = 3 };

constexpr uint32_t kPhiloxW0 = 0x9E3779B9u, kPhiloxW1 = 0xBB67AE85u;  // Weyl key bumps

struct PhiloxKey {
  uint32_t k0, k1;
  __device__ __forceinline__ uint32_t rk0(int r) const { return k0 + (uint32_t)r * kPhiloxW0; }
  __device__ __forceinline__ uint32_t rk1(int r) const { return k1 + (uint32_t)r * kPhiloxW1; }
};

// Philox4x32-10 (Salmon et al., SC'11): 10 rounds of two 32x32->64 products;
// the key is bumped by the Weyl constants between rounds.
template <class K>
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, const K& key) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint32_t lo0 = 0xD2511F53u * c.x;
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x);
    const uint32_t lo1 = 0xCD9E8D57u * c.z;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z);
    c = make_uint4(hi1 ^ c.y ^ key.rk0(r), lo1, hi0 ^ c.w ^ key.rk1(r), lo0);
  }
  return c;
}

// 24-bit uniform: exact conversion (w >> 8 < 2^24) times an exact power of 2.
__device__ __forceinline__ float u01(uint32_t w) {
  return __uint2float_rn(w >> 8) * 0x1p-24f;
}

__device__ __forceinline__ float4 u01x4(uint4 w) {
  return make_float4(u01(w.x), u01(w.y), u01(w.z), u01(w.w));
}

// The 24-bit integers m = w >> 8 of one call, as exact floats (U = m 2^-24).
__device__ __forceinline__ float4 raw24x4(uint4 w) {
  return make_float4(__uint2float_rn(w.x >> 8), __uint2float_rn(w.y >> 8),
                     __uint2float_rn(w.z >> 8), __uint2float_rn(w.w >> 8));
}

// m of float4 q (dims 4q..4q+3) of particle i at iteration t.
template <class K>
__device__ __forceinline__ float4 raw24x4(const K& key, uint32_t tag, uint32_t t, uint32_t i,
                                          uint32_t q) {
  return raw24x4(philox4x32_10(make_uint4(q, i, t, tag), key));
}

// --- Philox for a thread that owns a fixed float4 slot q over many rows ---
// With the counter {q, i, t, tag}, the products of rounds 1-3 that involve
// only q, t and the tag do not change from row to row.  PhiloxIter holds the
// per-kernel values (t), PhiloxSlot the per-(slot, tag) ones; philox_slot_row
// then evaluates the same 10 rounds with the row-independent products taken
// from them -- bit for bit philox4x32_10({q, i, t, tag}).  Round by round
// (M0, M1 the multipliers, rk the round keys):
//   r0: c = {hi(M1 t) ^ i ^ rk0(0), lo(M1 t), hi(M0 q) ^ tag ^ rk1(0), lo(M0 q)}
//   r1: M0 c.x depends on the row (shared by both tags); M1 c.z on (q, tag) only
//   r2: M0 c.x on (q, tag) only; M1 c.z on the row (shared by both tags)
//   r3..r9: everything depends on the row.
struct PhiloxIter {
  uint32_t a0;  // hi(M1 t) ^ rk0(0)
  uint32_t b0;  // lo(M1 t)
};
struct PhiloxSlot {
  uint32_t w1;  // lo(M0 q) ^ rk1(1)       (r1: c.z = hi(M0 c.x) ^ c.w ^ rk1(1))
  uint32_t p2;  // lo(M1 c1.z) ^ rk0(2)    (r2: c.x = hi(M1 c2.z) ^ c2.y ^ rk0(2))
  uint32_t q2;  // hi(M0 c2.x) ^ rk1(2)    (r2: c.z = hi(M0 c2.x) ^ c2.w ^ rk1(2))
  uint32_t r2;  // lo(M0 c2.x)             (r2: c.w)
};
template <class K>
__device__ __forceinline__ PhiloxIter philox_iter(const K& key, uint32_t t) {
  return PhiloxIter{__umulhi(0xCD9E8D57u, t) ^ key.rk0(0), 0xCD9E8D57u * t};
}
template <class K>
__device__ __forceinline__ PhiloxSlot philox_slot(const K& key, const PhiloxIter& it, uint32_t q,
                                                  uint32_t tag) {
  const uint32_t lo0 = 0xD2511F53u * q, hi0 = __umulhi(0xD2511F53u, q);
  const uint32_t c1z = hi0 ^ tag ^ key.rk1(0);           // round-0 output .z
  const uint32_t c2x = __umulhi(0xCD9E8D57u, c1z) ^ it.b0 ^ key.rk0(1);  // round-1 output .x
  const uint32_t c2y = 0xCD9E8D57u * c1z;                // round-1 output .y
  return PhiloxSlot{lo0 ^ key.rk1(1), c2y ^ key.rk0(2), __umulhi(0xD2511F53u, c2x) ^ key.rk1(2),
                    0xD2511F53u * c2x};
}
// Rounds 0-2 of the row part, shared by the two tags of one float4: returns
// {round-1 lo(M0 c.x), round-2 hi/lo(M1 c.z)} through out-parameters.
__device__ __forceinline__ void philox_row_shared(const PhiloxIter& it, const PhiloxSlot& s0,
                                                  uint32_t i, uint32_t& lo0r1, uint32_t& hi1r2,
                                                  uint32_t& lo1r2) {
  const uint32_t c1x = it.a0 ^ i;                         // round-0 output .x
  lo0r1 = 0xD2511F53u * c1x;                              // round-1 output .w
  const uint32_t c2z = __umulhi(0xD2511F53u, c1x) ^ s0.w1;  // round-1 output .z (tag-free)
  hi1r2 = __umulhi(0xCD9E8D57u, c2z);
  lo1r2 = 0xCD9E8D57u * c2z;                              // round-2 output .y
}
template <class K>
__device__ __forceinline__ uint4 philox_slot_row(const K& key, const PhiloxSlot& s, uint32_t lo0r1,
                                                 uint32_t hi1r2, uint32_t lo1r2) {
  uint4 c = make_uint4(hi1r2 ^ s.p2, lo1r2, s.q2 ^ lo0r1, s.r2);  // after round 2
#pragma unroll
  for (int r = 3; r < 10; ++r) {
    const uint32_t lo0 = 0xD2511F53u * c.x;
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x);
    const uint32_t lo1 = 0xCD9E8D57u * c.z;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z);
    c = make_uint4(hi1 ^ c.y ^ key.rk0(r), lo1, hi0 ^ c.w ^ key.rk1(r), lo0);
  }
  return c;
}

// The 4 uniforms of float4 q (dims 4q..4q+3) of particle i at iteration t.
template <class K>
__device__ __forceinline__ float4 uniforms4(const K& key, uint32_t tag, uint32_t t,
                                            uint32_t i, uint32_t q) {
  return u01x4(philox4x32_10(make_uint4(q, i, t, tag), key));
}

}  // namespace fastpso
