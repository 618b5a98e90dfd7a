// device_common.cuh -- small device helpers shared by the libmagus kernels.
#pragma once

#include <cstdint>

#include "magus_internal.h"

namespace magus {

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {  // splitmix64 finaliser
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

// Digest multiplier of decision word w.
__device__ __forceinline__ uint64_t digest_mul(int64_t w) { return mix64((uint64_t)w) | 1ULL; }

// Quantised stretch, literal form (model M):
//   r = x * (1/B_l); sigma = r - 1 if r > 1 else 0; cap 2^15; units 2^-24.
__device__ __forceinline__ uint64_t q_literal(float x, double invB) {
  const double r = (double)x * invB;
  if (r > 1.0) {
    double s = r - 1.0;
    if (s > 32768.0) s = 32768.0;
    return (uint64_t)(s * kQScale);
  }
  return 0;
}

// Same quantity, strength-reduced (valid when x > xthr, i.e. RN(x*invB) > 1):
// r24 = RN(x*invB*2^24) = RN(x*invB)*2^24 and RN(r24 - 2^24) = RN(r-1)*2^24
// (power-of-two scaling commutes with round-to-nearest in the normal range).
// s24 is in (0, 2^39], so floor(s24) = bits(RZ(s24 + 2^52)) - bits(2^52):
// an fp64 add instead of the F2I conversion on the slow XU pipe.
__device__ __forceinline__ uint64_t q_scaled(float x, double invB24) {
  double s24 = (double)x * invB24 - kQScale;
  s24 = s24 < kQCapScaled ? s24 : kQCapScaled;  // never NaN here: x > xthr
  return (uint64_t)__double_as_longlong(__dadd_rz(s24, 4503599627370496.0)) - 0x4330000000000000ULL;
}
// Same without the cap, for x <= x_stretch at ratio_max: s24 < (r_max/r_min)
// * 2^24 <= 127 * 2^24 < 2^39 (ratio_max <= 127), so the cap never binds.
__device__ __forceinline__ uint64_t q_scaled_nocap(float x, double invB24) {
  const double s24 = (double)x * invB24 - kQScale;
  return (uint64_t)__double_as_longlong(__dadd_rz(s24, 4503599627370496.0)) - 0x4330000000000000ULL;
}

// Model M finalisation of one (trace, config); fixed fp64
// operation order, compiled with --fmad=false.
__device__ __forceinline__ void finalize_summary(const DevPlatform& p, int64_t T, int64_t events,
                                                 int64_t hi_rounds, int64_t msr, int64_t changes,
                                                 int64_t n_min_dec, int64_t n_min_int, uint64_t q_min,
                                                 uint64_t q_max, uint64_t q_base, uint64_t digest,
                                                 int64_t n_burst_base, int64_t n_burst_magus,
                                                 magus_summary* s, magus_base* b) {
  const int64_t n_max_int = T - n_min_int;
  const double time_max = p.dt * (double)n_max_int + p.cQ * (double)q_max;
  const double time_min = p.dt * (double)n_min_int + p.cQ * (double)q_min;
  const double time = (p.dt * (double)T + p.cQ * (double)(q_min + q_max)) + p.t_sw * (double)changes;
  const double energy = (p.P_max * time_max + p.P_min * time_min) + p.e_sw * (double)changes;
  const double base_time = p.dt * (double)T + p.cQ * (double)q_base;
  if (s) {
    magus_summary o;
    o.n_events = events;
    o.n_hi_rounds = hi_rounds;
    o.n_msr_writes = msr;
    o.n_changes = changes;
    o.n_min_dec = n_min_dec;
    o.n_min_int = n_min_int;
    o.q_min = q_min;
    o.q_max = q_max;
    o.digest = digest;
    o.time_s = time;
    o.energy_j = energy;
    o.slowdown = time / base_time - 1.0;
    o.viol = o.slowdown > p.bound ? 1 : 0;
    o.reserved = 0;
    o.n_burst_base = n_burst_base;
    o.n_burst_magus = n_burst_magus;
    *s = o;
  }
  if (b) {
    magus_base o;
    o.q_base = q_base;
    o.time_s = base_time;
    o.energy_j = p.P_max * base_time;
    o.reserved = 0;
    *b = o;
  }
}

}  // namespace magus
