// precompute.cpp -- host-side validation and per-config constants.
//
// The stream kernel never divides: Alg. 1's "d = delta / L; d > tau_inc"
// (P@20631 lines 3-4) is replaced by "delta > d_inc" where d_inc is the
// largest double whose quotient by L does not exceed tau_inc.  Because
// RN(delta / L) is monotone non-decreasing in delta (L > 0), the two
// predicates agree for every non-NaN double delta (and both are false for
// NaN).  The same holds for the decrease test, Alg. 2's "s/n >= t_hi"
// (-> s >= k) and model M's "x/B > 1" (-> x > xthr, a float threshold).
// Each inversion is an exact search over the ordered bit patterns, so the
// host computes it with the very predicate the paper states.
#include <cmath>
#include <cstdio>
#include <cstring>

#include "magus_internal.h"

namespace magus {
namespace {

// Total order on non-NaN doubles as integers (-0 and +0 share key 0).
int64_t dkey(double d) {
  uint64_t b;
  std::memcpy(&b, &d, 8);
  if (b >> 63) return -(int64_t)(b & 0x7FFFFFFFFFFFFFFFULL);
  return (int64_t)b;
}
double dfromkey(int64_t k) {
  uint64_t b = k >= 0 ? (uint64_t)k : ((uint64_t)(-k) | 0x8000000000000000ULL);
  double d;
  std::memcpy(&d, &b, 8);
  return d;
}

}  // namespace

double invert_inc(double L, double tau_inc) {
  // largest delta with !(delta / L > tau_inc)
  int64_t lo = dkey(-INFINITY), hi = dkey(INFINITY);  // pred(lo) true, pred(hi) false
  while ((uint64_t)hi - (uint64_t)lo > 1) {
    const int64_t mid = lo + (int64_t)(((uint64_t)hi - (uint64_t)lo) / 2);  // range > INT64_MAX
    double d = dfromkey(mid) / L;
    if (!(d > tau_inc)) lo = mid; else hi = mid;
  }
  return dfromkey(lo);
}

double invert_dec(double L, double tau_dec) {
  // smallest delta with !(delta / L < tau_dec)
  int64_t lo = dkey(-INFINITY), hi = dkey(INFINITY);  // dec(lo) true, dec(hi) false
  while ((uint64_t)hi - (uint64_t)lo > 1) {
    const int64_t mid = lo + (int64_t)(((uint64_t)hi - (uint64_t)lo) / 2);
    double d = dfromkey(mid) / L;
    if (d < tau_dec) lo = mid; else hi = mid;
  }
  double r = dfromkey(hi);
  return r == 0.0 ? 0.0 : r;  // canonical +0
}

float stretch_threshold(double invB) {
  // largest float f >= 0 with !((double)f * invB > 1.0)
  uint32_t lo = 0, hi = 0x7F800000u;  // 0 -> true, +inf -> false
  while (hi - lo > 1) {
    uint32_t mid = lo + (hi - lo) / 2;
    float f;
    std::memcpy(&f, &mid, 4);
    double r = (double)f * invB;
    if (!(r > 1.0)) lo = mid; else hi = mid;
  }
  float f;
  std::memcpy(&f, &lo, 4);
  return f;
}

float above_threshold(double theta) {
  // largest float f with !((double)f > theta); -inf when even -FLT_MAX exceeds it
  if (!(theta < (double)3.4028234663852886e38)) return INFINITY;
  int64_t lo = -(int64_t)0x7F800000, hi = 0x7F800000;  // ordered float keys: -inf .. +inf
  auto val = [](int64_t k) {
    uint32_t b = k >= 0 ? (uint32_t)k : ((uint32_t)(-k) | 0x80000000u);
    float f;
    std::memcpy(&f, &b, 4);
    return f;
  };
  if ((double)val(lo) > theta) return -INFINITY;
  while (hi - lo > 1) {
    const int64_t mid = lo + (hi - lo) / 2;
    if (!((double)val(mid) > theta)) lo = mid; else hi = mid;
  }
  return val(lo);
}

bool validate_policy(const magus_policy& p, char* msg, size_t n) {
  if (p.window < 2) { std::snprintf(msg, n, "window %d < 2", p.window); return false; }
  if (p.history < 1 || p.history > 64) {
    std::snprintf(msg, n, "history %d not in [1, 64]", p.history);
    return false;
  }
  if (!(p.deriv_len > 0.0) || !std::isfinite(p.deriv_len)) {
    std::snprintf(msg, n, "deriv_len %g not finite and > 0", p.deriv_len);
    return false;
  }
  if (!std::isfinite(p.tau_inc) || !std::isfinite(p.tau_dec)) {
    std::snprintf(msg, n, "tau_inc / tau_dec must be finite");
    return false;
  }
  if (!(p.t_hi > 0.0)) { std::snprintf(msg, n, "t_hi %g not > 0", p.t_hi); return false; }
  if (p.variant < 0 || p.variant > (MAGUS_VARIANT_CLOSED_LOOP | MAGUS_VARIANT_GRADUAL)) {
    std::snprintf(msg, n, "unknown variant %d", p.variant);
    return false;
  }
  if ((p.variant & MAGUS_VARIANT_GRADUAL) ? p.step < 1 : p.step != 0) {
    std::snprintf(msg, n, "step %d: >= 1 for the gradual variant, else 0", p.step);
    return false;
  }
  if ((p.variant & MAGUS_VARIANT_CLOSED_LOOP) && p.window > 128) {
    std::snprintf(msg, n, "closed-loop variant needs window <= 128");
    return false;
  }
  return true;
}

bool validate_platform(const magus_platform& p, char* msg, size_t n) {
  if (p.ratio_min < 1 || p.ratio_max > 127 || p.ratio_min >= p.ratio_max) {
    std::snprintf(msg, n, "ratio range [%d, %d] invalid", p.ratio_min, p.ratio_max);
    return false;
  }
  const double v[] = {p.dt_s, p.bw_max_mbs, p.beta, p.p_other_w, p.p_unc_min_w, p.p_unc_max_w,
                      p.e_switch_j, p.t_switch_s, p.slowdown_bound, p.burst_mbs};
  for (double d : v)
    if (!std::isfinite(d)) { std::snprintf(msg, n, "platform values must be finite"); return false; }
  if (!(p.dt_s > 0.0) || !(p.bw_max_mbs > 0.0)) {
    std::snprintf(msg, n, "dt_s and bw_max_mbs must be > 0");
    return false;
  }
  if (p.beta < 0.0 || p.p_other_w < 0.0 || p.p_unc_min_w < 0.0 || p.p_unc_max_w < 0.0 ||
      p.e_switch_j < 0.0 || p.t_switch_s < 0.0) {
    std::snprintf(msg, n, "beta, powers, switch costs must be >= 0");
    return false;
  }
  return true;
}

DevPolicy make_dev_policy(const magus_policy& p) {
  DevPolicy d;
  std::memset(&d, 0, sizeof(d));
  d.L = p.deriv_len;
  d.tau_inc = p.tau_inc;
  d.tau_dec = p.tau_dec;
  d.d_inc = invert_inc(p.deriv_len, p.tau_inc);
  d.d_dec = invert_dec(p.deriv_len, p.tau_dec);
  d.t_hi = p.t_hi;
  d.W = p.window;
  d.H = p.history;
  d.variant = p.variant;
  d.step = p.step;
  d.k = p.history + 1;
  for (int s = 0; s <= p.history; ++s)
    if ((double)s / (double)p.history >= p.t_hi) { d.k = s; break; }
  return d;
}

DevPlatform make_dev_platform(const magus_platform& p) {
  DevPlatform d;
  std::memset(&d, 0, sizeof(d));
  d.r_min = p.ratio_min;
  d.r_max = p.ratio_max;
  const double Bmin = (p.bw_max_mbs * (double)p.ratio_min) / (double)p.ratio_max;
  const double Bmax = (p.bw_max_mbs * (double)p.ratio_max) / (double)p.ratio_max;
  d.invB_min = 1.0 / Bmin;
  d.invB_max = 1.0 / Bmax;
  d.invB24_min = d.invB_min * kQScale;  // exact power-of-two scaling
  d.invB24_max = d.invB_max * kQScale;
  d.xthr_min = stretch_threshold(d.invB_min);
  d.xthr_max = stretch_threshold(d.invB_max);
  d.dt = p.dt_s;
  d.cQ = (p.dt_s * p.beta) / kQScale;
  const double span = (double)(p.ratio_max - p.ratio_min);
  d.P_max = (p.p_other_w + p.p_unc_min_w) +
            ((p.p_unc_max_w - p.p_unc_min_w) * (double)(p.ratio_max - p.ratio_min)) / span;
  d.P_min = (p.p_other_w + p.p_unc_min_w) +
            ((p.p_unc_max_w - p.p_unc_min_w) * (double)(p.ratio_min - p.ratio_min)) / span;
  d.e_sw = p.e_switch_j;
  d.t_sw = p.t_switch_s;
  d.bound = p.slowdown_bound;
  d.burst_mbs = p.burst_mbs;
  d.Bmin = Bmin;
  d.Bmax = Bmax;
  d.xburst = above_threshold(p.burst_mbs);
  d.xobs_max = above_threshold(Bmax);
  d.burst_on = (p.burst_mbs > 0.0 && Bmax > p.burst_mbs) ? 1 : 0;
  d.burst_min_keeps = (Bmin > p.burst_mbs) ? 1 : 0;
  return d;
}

}  // namespace magus
