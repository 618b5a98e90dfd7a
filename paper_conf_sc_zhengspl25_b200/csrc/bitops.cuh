// bitops.cuh -- bit-parallel building blocks of the replay kernels: the
// Alg. 2 window count over 32 rounds at once (bit-sliced), the ">= k"
// compare, Alg. 3's sample-and-hold as a carry chain, and predicated ORs of
// compare results into 32-bit masks.  Shared by kernels_stream.cu and
// kernels_walk.cu.
#pragma once

#include <cstdint>

namespace magus {

// ---- Alg. 2, bit-parallel: bit i of the result = (#events at positions
// i-H .. i-1 >= k), positions < 0 coming from the previous word Ep. ----
// count (bit-sliced, NB bits) >= k  <=>  no borrow out of count - k; km[j] =
// all-ones where bit j of k is set (k < 2^NB always: k <= H + 1)
template <int NB>
__device__ __forceinline__ uint32_t ge_k(const uint32_t* c, const uint32_t* km) {
  uint32_t b = 0;
#pragma unroll
  for (int j = 0; j < NB; ++j) b = (~c[j] & km[j]) | (~c[j] & b) | (km[j] & b);  // maj: 1 LOP3
  return ~b;
}
__device__ __forceinline__ void fa(uint32_t a, uint32_t b, uint32_t c, uint32_t& s, uint32_t& cy) {
  s = a ^ b ^ c;
  cy = (a & b) | (c & (a ^ b));
}
// Bit-sliced count of the H events before each of the 32 positions
// (positions < 0 come from the previous word Ep): c[0..NBITS) per position.
template <int H>
struct Window {  // compile-time H <= 32: ripple-carry counter, 6 bits
  static constexpr int NBITS = 6;
  static __device__ __forceinline__ void count(uint32_t E, uint32_t Ep, int, uint32_t* c) {
#pragma unroll
    for (int l = 0; l < 6; ++l) c[l] = 0;
#pragma unroll
    for (int j = 1; j <= H; ++j) {
      uint32_t b = __funnelshift_lc(Ep, E, j);  // clamps: j = 32 -> Ep
#pragma unroll
      for (int l = 0; l < 6; ++l) {
        const uint32_t t = c[l] & b;
        c[l] ^= b;
        b = t;
      }
    }
  }
};
template <>
struct Window<10> {  // the paper's H = 10 (P@24182): carry-save tree, 16 LOP3
  static constexpr int NBITS = 4;
  static __device__ __forceinline__ void count(uint32_t E, uint32_t Ep, int, uint32_t* c) {
    uint32_t s[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) s[j] = __funnelshift_l(Ep, E, j + 1);
    uint32_t a0, a1, b0, b1, c0, c1, d0, d1, f1, f2, g2;
    fa(s[0], s[1], s[2], a0, a1);
    fa(s[3], s[4], s[5], b0, b1);
    fa(s[6], s[7], s[8], c0, c1);
    fa(a0, b0, c0, d0, d1);
    c[0] = d0 ^ s[9];
    const uint32_t e1 = d0 & s[9];
    fa(a1, b1, c1, f1, f2);
    fa(d1, e1, f1, c[1], g2);
    c[2] = f2 ^ g2;
    c[3] = f2 & g2;
  }
};
template <>
struct Window<0> {  // runtime H <= 32
  static constexpr int NBITS = 6;
  static __device__ __forceinline__ void count(uint32_t E, uint32_t Ep, int H, uint32_t* c) {
#pragma unroll
    for (int l = 0; l < 6; ++l) c[l] = 0;
    for (int j = 1; j <= H; ++j) {
      uint32_t b = __funnelshift_lc(Ep, E, j);  // clamps: j = 32 -> Ep
#pragma unroll
      for (int l = 0; l < 6; ++l) {
        const uint32_t t = c[l] & b;
        c[l] ^= b;
        b = t;
      }
    }
  }
};

// ---- Alg. 3 sample-and-hold: D_i = V at the last action <= i, else carry ----
// A carry chain: a "set" (action to min, A & V) generates, a "reset" (action to
// max, A & ~V) kills, every other position propagates.  The carries of
// x + y + cin with x = ~(A & ~V), y = A & V are exactly that (x & y = set,
// x ^ y = no action), so one 33-bit add replaces a 5-step log-depth fill.
__device__ __forceinline__ uint32_t forward_fill(uint32_t A, uint32_t V, uint32_t cin) {
  const uint32_t x = ~(A & ~V), y = A & V;
  const uint64_t sum = (uint64_t)x + (uint64_t)y + (uint64_t)cin;
  const uint32_t cin_bits = (uint32_t)sum ^ x ^ y;                // carry INTO bit i (bit 0: cin)
  return __funnelshift_r(cin_bits, (uint32_t)(sum >> 32), 1);     // carry OUT of bit i
}

// w |= bit if a > b / a < b: one compare + one predicated LOP3 per bit
// (the C form compiles to compare + SEL + a shared IADD3).
__device__ __forceinline__ void or_if_gt(uint32_t& w, double a, double b, uint32_t bit) {
  asm("{\n.reg .pred p;\nsetp.gt.f64 p, %1, %2;\n@p or.b32 %0, %0, %3;\n}"
      : "+r"(w) : "d"(a), "d"(b), "r"(bit));
}
__device__ __forceinline__ void or_if_lt(uint32_t& w, double a, double b, uint32_t bit) {
  asm("{\n.reg .pred p;\nsetp.lt.f64 p, %1, %2;\n@p or.b32 %0, %0, %3;\n}"
      : "+r"(w) : "d"(a), "d"(b), "r"(bit));
}
__device__ __forceinline__ void or_if_eq(uint32_t& w, int a, int b, uint32_t bit) {
  asm("{\n.reg .pred p;\nsetp.eq.s32 p, %1, %2;\n@p or.b32 %0, %0, %3;\n}" : "+r"(w) : "r"(a), "r"(b), "r"(bit));
}
__device__ __forceinline__ void or_if_ne(uint32_t& w, int a, int b, uint32_t bit) {
  asm("{\n.reg .pred p;\nsetp.ne.s32 p, %1, %2;\n@p or.b32 %0, %0, %3;\n}" : "+r"(w) : "r"(a), "r"(b), "r"(bit));
}
__device__ __forceinline__ void or_if_gt(uint32_t& w, float a, float b, uint32_t bit) {
  asm("{\n.reg .pred p;\nsetp.gt.f32 p, %1, %2;\n@p or.b32 %0, %0, %3;\n}"
      : "+r"(w) : "f"(a), "f"(b), "r"(bit));
}

}  // namespace magus
