// kernels_ref.cu -- the per-sample replay kernel.
//
// One thread per (trace, config), sequential over all T intervals, in the
// paper's per-round order: Alg. 2 on the H previous events (P@21063), the
// frequent-transition override (Alg. 3 l.9-15), Alg. 1 with the literal fp64
// division d = delta / L (P@20631 l.3), event logging (l.17/22/28/31) and
// the step rule (l.18-25).
//
// Roles: (1) the parity baseline of the stream, sequential, walk and
// speculative kernels (an independent GPU formulation: literal division,
// popc of a history register, per-sample accounting); (2) the last-resort
// fallback (closed-loop configs none of those kernels takes); (3) a literal
// form of the NEXT variants:
//   f3 closed loop  -- Alg. 1 observes the delivered throughput
//                      min(x_t, B(l_t)), which depends on the decision that
//                      governs interval t, so no time segmentation is exact;
//   f4 gradual step -- +-step ratio per event (the contrast of P@35554), so
//                      decisions are multi-level and model M keeps one
//                      (intervals, stretch) pair per level.
#include "device_common.cuh"

namespace magus {

constexpr int kMaxLevels = 128;  // ratios 1..127

// Model M per level (the same formulas as the host, evaluated on the device).
__device__ __forceinline__ double capacity(const DevPlatform& p, double bw_max, int l) {
  return (bw_max * (double)l) / (double)p.r_max;
}

// LITERAL: Alg. 1/2 with the printed fp64 divisions (the parity baseline of
// the stream kernel); otherwise the exact host-inverted thresholds of
// precompute.cpp (delta > d_inc, s >= k), which shortens the dependent chain
// of the sequential variants by two fp64 divisions per round.
template <bool MULTI, bool LITERAL>
__global__ void __launch_bounds__(128)
ref_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
           const DevPolicy* __restrict__ pol, int32_t C, DevPlatform plat, double bw_max,
           double p_lo, double p_span, magus_summary* __restrict__ out, magus_base* __restrict__ base,
           uint32_t* __restrict__ dec, uint8_t* __restrict__ levels) {
  // per-level tables (levels r_min..r_max): 1/B_l, B_l, P_l
  __shared__ double s_invB[kMaxLevels], s_B[kMaxLevels], s_P[kMaxLevels];
  const int nlev = plat.r_max - plat.r_min + 1;
  for (int i = threadIdx.x; i < nlev; i += blockDim.x) {
    const int l = plat.r_min + i;
    const double B = capacity(plat, bw_max, l);
    s_B[i] = B;
    s_invB[i] = 1.0 / B;
    s_P[i] = p_lo + (p_span * (double)(l - plat.r_min)) / (double)(plat.r_max - plat.r_min);
  }
  __syncthreads();

  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= N * C) return;
  const int32_t c = (int32_t)(gid / N);
  const int64_t n = gid - (int64_t)c * N;
  const DevPolicy P = pol[c];
  const int64_t nw = (T + 31) / 32;
  const uint64_t hmask = P.H >= 64 ? ~0ULL : ((1ULL << P.H) - 1ULL);
  const bool closed = (P.variant & MAGUS_VARIANT_CLOSED_LOOP) != 0;
  const bool gradual = (P.variant & MAGUS_VARIANT_GRADUAL) != 0;
  const int lmin = plat.r_min, lmax = plat.r_max;

  uint64_t hist = 0;             // uncore_tune_ls: H zeros (P@24182); bit j = round t-1-j
  int lvl = lmax;                // uncore_freq: starts at max (P@23755)
  int64_t events = 0, hi_rounds = 0, msr = 0, changes = 0, n_min_dec = 0, n_min_int = 0;
  uint64_t q_min = 0, q_max = 0, q_base = 0, digest = 0;
  int64_t b_base = 0, b_magus = 0;  // Sec. 6.3 bursts (model M 4.6)
  const bool bursts = plat.burst_mbs > 0.0;
  uint32_t word = 0;
  int prev = lmax;               // dec[t-1]; dec[-1] := max
  uint8_t ring[kMaxLevels];      // closed loop: level that governed interval t (mod 128)
  uint32_t nl[MULTI ? kMaxLevels : 1];
  uint64_t ql[MULTI ? kMaxLevels : 1];
  if constexpr (MULTI) {
    for (int i = 0; i < nlev; ++i) { nl[i] = 0; ql[i] = 0; }
  }

  // The scan is sequential, but its inputs are not: each 32-step chunk of
  // samples and of their Alg. 1 lags is loaded up front (64 independent
  // coalesced loads), so the dependent chain never waits on memory.
  // (staged through this thread's columns of a shared-memory tile)
  __shared__ float s_x[32][128], s_l[32][128];
  for (int64_t t = 0; t < T; ++t) {
    const int j = (int)(t & 31);
    if (j == 0) {
#pragma unroll 8
      for (int i = 0; i < 32; ++i) {
        const int64_t ti = t + i, tli = ti - P.W + 1;
        s_x[i][threadIdx.x] = ti < T ? x[ti * ld + n] : 0.0f;
        s_l[i][threadIdx.x] = (ti < T && tli >= 0) ? x[tli * ld + n] : 0.0f;
      }
    }
    const float xt = s_x[j][threadIdx.x], xl = s_l[j][threadIdx.x];
    const int leff = prev;       // model M / closed loop: interval t runs at dec[t-1] (R6)
    if (closed) ring[t & (kMaxLevels - 1)] = (uint8_t)leff;
    if (t >= P.W) {              // MDFS rounds start at t = W (reading R5)
      const int64_t tl = t - P.W + 1;
      double yt = (double)xt, yl = (double)xl;
      if (closed) {              // f3: delivered throughput min(x, B(level))
        const double Bt = s_B[leff - lmin], Bl = s_B[ring[tl & (kMaxLevels - 1)] - lmin];
        if (yt > Bt) yt = Bt;
        if (yl > Bl) yl = Bl;
      }
      // Alg. 2: s = sum of the H logged events, f = s / n, f >= t_hi
      const int s = __popcll(hist);
      const bool hi = LITERAL ? ((double)s / (double)P.H) >= P.t_hi : s >= P.k;
      if (hi) { lvl = lmax; ++msr; ++hi_rounds; }
      // Alg. 1: d = (ls[n] - ls[0]) / L
      int p;
      if (LITERAL) {
        const double d = (yt - yl) / P.L;
        p = d > P.tau_inc ? 1 : (d < P.tau_dec ? -1 : 0);
      } else {
        const double D = yt - yl;
        p = D > P.d_inc ? 1 : (D < P.d_dec ? -1 : 0);
      }
      if (p != 0) {
        ++events;
        if (!hi) {
          if (gradual) lvl = p > 0 ? min(lvl + P.step, lmax) : max(lvl - P.step, lmin);  // f4
          else lvl = p > 0 ? lmax : lmin;                                                 // l.18/25
          ++msr;
        }
      }
      hist = ((hist << 1) | (uint64_t)(p != 0)) & hmask;
    }
    const int dmin = lvl == lmin;
    if (levels) levels[((int64_t)c * T + t) * N + n] = (uint8_t)lvl;
    // model M accounting of interval t at level leff
    if constexpr (MULTI) {
      const int li = leff - lmin;
      ++nl[li];
      ql[li] += q_literal(xt, s_invB[li]);
    } else {
      if (leff == lmin) { ++n_min_int; q_min += q_literal(xt, plat.invB_min); }
      else q_max += q_literal(xt, plat.invB_max);
    }
    q_base += q_literal(xt, plat.invB_max);
    if (bursts && (double)xt > plat.burst_mbs) {  // delivered min(x, B_l) > theta
      b_base += plat.Bmax > plat.burst_mbs;
      b_magus += s_B[leff - lmin] > plat.burst_mbs;
    }
    n_min_dec += dmin;
    if (t >= 1 && lvl != prev) ++changes;
    word |= (uint32_t)dmin << (t & 31);
    if ((t & 31) == 31 || t == T - 1) {
      const int64_t w = t >> 5;
      if (dec) dec[((int64_t)c * nw + w) * N + n] = word;
      digest += (uint64_t)word * digest_mul(w);
      word = 0;
    }
    prev = lvl;
  }
  magus_summary* so = out ? out + (int64_t)c * N + n : nullptr;
  magus_base* bo = (base && c == 0) ? base + n : nullptr;
  if constexpr (MULTI) {
    // general model M: energy = sum over levels, ascending
    n_min_int = nl[0];
    q_min = ql[0];
    for (int i = 1; i < nlev; ++i) q_max += ql[i];
    finalize_summary(plat, T, events, hi_rounds, msr, changes, n_min_dec, n_min_int, q_min, q_max,
                     q_base, digest, b_base, b_magus, so, bo);
    if (so) {
      double energy = 0.0;
      for (int i = 0; i < nlev; ++i)
        energy = energy + s_P[i] * (plat.dt * (double)nl[i] + plat.cQ * (double)ql[i]);
      energy = energy + plat.e_sw * (double)changes;
      so->energy_j = energy;
    }
  } else {
    finalize_summary(plat, T, events, hi_rounds, msr, changes, n_min_dec, n_min_int, q_min, q_max,
                     q_base, digest, b_base, b_magus, so, bo);
  }
}

int launch_reference(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
                     const DevPolicy* pol_dev, int32_t C, const DevPlatform& plat, double bw_max,
                     double p_lo, double p_span, bool multi, bool literal, magus_summary* out_summary,
                     magus_base* out_base, uint32_t* out_dec, uint8_t* out_levels) {
  const int64_t total = N * C;
  const unsigned blocks = (unsigned)((total + 127) / 128);
  auto k = multi ? (literal ? ref_kernel<true, true> : ref_kernel<true, false>)
                 : (literal ? ref_kernel<false, true> : ref_kernel<false, false>);
  k<<<blocks, 128, 0, s>>>(x, N, T, ld, pol_dev, C, plat, bw_max, p_lo, p_span, out_summary, out_base,
                           out_dec, out_levels);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
