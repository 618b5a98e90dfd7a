// kernels_ref.cu -- the reference (per-sample) replay kernel.
//
// One thread per (trace, config), sequential over all T intervals, in the
// paper's per-round order: Alg. 2 on the H previous events (P@21063), the
// frequent-transition override (Alg. 3 l.9-15), Alg. 1 with the literal fp64
// division d = delta / L (P@20631 l.3), event logging (l.17/22/28/31) and
// the jump rule (l.18-25).  It is the parity baseline for the stream kernel
// and the general fallback (any W >= 2, H <= 64), not the fast path: at one
// thread per trace it cannot fill the GPU for N ~ 4k.
#include "device_common.cuh"

namespace magus {

__global__ void __launch_bounds__(128)
ref_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
           const DevPolicy* __restrict__ pol, int32_t C, DevPlatform plat,
           magus_summary* __restrict__ out, magus_base* __restrict__ base,
           uint32_t* __restrict__ dec) {
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= N * C) return;
  const int32_t c = (int32_t)(gid / N);
  const int64_t n = gid - (int64_t)c * N;
  const DevPolicy P = pol[c];
  const int64_t nw = (T + 31) / 32;
  const uint64_t hmask = P.H >= 64 ? ~0ULL : ((1ULL << P.H) - 1ULL);

  uint64_t hist = 0;             // uncore_tune_ls: H zeros (P@24182); bit j = round t-1-j
  int freq_min = 0;              // uncore_freq: starts at max (P@23755)
  int64_t events = 0, hi_rounds = 0, msr = 0, changes = 0, n_min_dec = 0, n_min_int = 0;
  uint64_t q_min = 0, q_max = 0, q_base = 0, digest = 0;
  int64_t b_base = 0, b_magus = 0;  // Sec. 6.3 bursts (model M 4.6)
  const bool bursts = plat.burst_mbs > 0.0;
  uint32_t word = 0;
  int prev = 0;                  // dec[t-1] (min = 1); dec[-1] := max

  for (int64_t t = 0; t < T; ++t) {
    const float xt = x[t * ld + n];
    if (t >= P.W) {              // MDFS rounds start at t = W (reading R5)
      const float xl = x[(t - P.W + 1) * ld + n];
      // Alg. 2: s = sum of the H logged events, f = s / n, f >= t_hi
      const int s = __popcll(hist);
      const bool hi = ((double)s / (double)P.H) >= P.t_hi;
      if (hi) { freq_min = 0; ++msr; ++hi_rounds; }
      // Alg. 1: d = (ls[n] - ls[0]) / L
      const double d = ((double)xt - (double)xl) / P.L;
      const int p = d > P.tau_inc ? 1 : (d < P.tau_dec ? -1 : 0);
      if (p != 0) {
        ++events;
        if (!hi) { freq_min = (p < 0); ++msr; }
      }
      hist = ((hist << 1) | (uint64_t)(p != 0)) & hmask;
    }
    const int dmin = freq_min;
    // model M: the interval t runs at dec[t-1] (reading R6)
    if (prev) { ++n_min_int; q_min += q_literal(xt, plat.invB_min); }
    else q_max += q_literal(xt, plat.invB_max);
    q_base += q_literal(xt, plat.invB_max);
    if (bursts && (double)xt > plat.burst_mbs) {  // delivered min(x, B_l) > theta
      b_base += plat.Bmax > plat.burst_mbs;
      b_magus += (prev ? plat.Bmin : plat.Bmax) > plat.burst_mbs;
    }
    n_min_dec += dmin;
    if (t >= 1 && dmin != prev) ++changes;
    word |= (uint32_t)dmin << (t & 31);
    if ((t & 31) == 31 || t == T - 1) {
      const int64_t w = t >> 5;
      if (dec) dec[((int64_t)c * nw + w) * N + n] = word;
      digest += (uint64_t)word * digest_mul(w);
      word = 0;
    }
    prev = dmin;
  }
  finalize_summary(plat, T, events, hi_rounds, msr, changes, n_min_dec, n_min_int, q_min, q_max,
                   q_base, digest, b_base, b_magus, out ? out + (int64_t)c * N + n : nullptr,
                   (base && c == 0) ? base + n : nullptr);
}

int launch_reference(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
                     const DevPolicy* pol_dev, int32_t C, const DevPlatform& plat,
                     magus_summary* out_summary, magus_base* out_base, uint32_t* out_dec) {
  const int64_t total = N * C;
  const int64_t blocks = (total + 127) / 128;
  ref_kernel<<<(unsigned)blocks, 128, 0, s>>>(x, N, T, ld, pol_dev, C, plat, out_summary, out_base,
                                              out_dec);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
