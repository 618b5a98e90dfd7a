// kernels_post.cu -- segment carry resolution, per-config totals, and the
// device build of the synthetic trace generator.
#include "device_common.cuh"
#include "../../gen/magus_gen.h"

namespace magus {

// ---------------------------------------------------------------------------
// Per-config totals: exact integer sums over traces (order-free).
// ---------------------------------------------------------------------------
constexpr int kTotThreads = 256;
constexpr int kTotAcc = kTotAccWords;

__global__ void __launch_bounds__(kTotThreads)
totals_kernel(const magus_summary* __restrict__ sm, const magus_base* __restrict__ base, int64_t N,
              int64_t T, uint64_t* __restrict__ tot) {
  const int32_t c = blockIdx.x;
  uint64_t a[kTotAcc];
#pragma unroll
  for (int i = 0; i < kTotAcc; ++i) a[i] = 0;
  for (int64_t n = threadIdx.x; n < N; n += kTotThreads) {
    const magus_summary& s = sm[(int64_t)c * N + n];
    a[0] += (uint64_t)s.viol;
    a[1] += (uint64_t)s.n_events;
    a[2] += (uint64_t)s.n_hi_rounds;
    a[3] += (uint64_t)s.n_msr_writes;
    a[4] += (uint64_t)s.n_changes;
    a[5] += (uint64_t)s.n_min_dec;
    a[6] += (uint64_t)s.n_min_int;
    a[7] += s.q_min & 0xFFFFFFFFULL;
    a[8] += s.q_min >> 32;
    a[9] += s.q_max & 0xFFFFFFFFULL;
    a[10] += s.q_max >> 32;
    const uint64_t qb = base[n].q_base;
    a[11] += qb & 0xFFFFFFFFULL;
    a[12] += qb >> 32;
    a[13] += (uint64_t)s.n_burst_base;
    a[14] += (uint64_t)s.n_burst_magus;
  }
  __shared__ uint64_t red[kTotThreads / 32][kTotAcc];
#pragma unroll
  for (int i = 0; i < kTotAcc; ++i) {
    uint64_t v = a[i];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xFFFFFFFFu, v, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5][i] = v;
  }
  __syncthreads();
  if (threadIdx.x < kTotAcc) {
    uint64_t v = 0;
    for (int w = 0; w < kTotThreads / 32; ++w) v += red[w][threadIdx.x];
    // accumulators 0..12 -> words 1..13; 13, 14 -> the burst words
    const int word = threadIdx.x < 13 ? 1 + threadIdx.x : MAGUS_TOT_BURST_BASE + (threadIdx.x - 13);
    tot[(int64_t)c * MAGUS_TOT_WORDS + word] = v;
  }
  if (threadIdx.x == 0) {
    tot[(int64_t)c * MAGUS_TOT_WORDS + MAGUS_TOT_N_TRACES] = (uint64_t)N;
    tot[(int64_t)c * MAGUS_TOT_WORDS + MAGUS_TOT_N_STEPS] = (uint64_t)N * (uint64_t)T;
    tot[(int64_t)c * MAGUS_TOT_WORDS + MAGUS_TOT_RESERVED] = 0;
  }
}

int launch_totals(cudaStream_t s, const magus_summary* summary, const magus_base* base, int64_t N,
                  int64_t T, int32_t C, uint64_t* totals) {
  totals_kernel<<<C, kTotThreads, 0, s>>>(summary, base, N, T, totals);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

// ---------------------------------------------------------------------------
// Synthetic traces: one thread per trace, sequential in t, coalesced stores.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(128)
gen_kernel(uint64_t seed, int64_t id0, int64_t N, int64_t T, int64_t ld, int32_t kind,
           float* __restrict__ out) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= N) return;
  mg_state g;
  mg_init(&g, seed, id0 + i, kind);
  for (int64_t t = 0; t < T; ++t) out[t * ld + i] = (float)mg_step(&g);
}

// ---------------------------------------------------------------------------
// Device form of the fleet derivation + sweep choice (api.cu derive_totals /
// choose_best), bit-identical: the same fp64 operations in the same order,
// and a correctly rounded conversion of the 128-bit q sums to double.
// ---------------------------------------------------------------------------
// RN(unsigned 128-bit hi:lo) to double: keep the top 64 bits, fold every
// dropped bit into a sticky LSB (below the rounding position), convert, scale.
__device__ __forceinline__ double u128_to_double_rn(uint64_t hi, uint64_t lo) {
  if (hi == 0) return __ull2double_rn(lo);
  const int s = 64 - __clzll(hi);                     // bits beyond the low 64, 1..64
  const uint64_t top = s == 64 ? hi : ((hi << (64 - s)) | (lo >> s));  // the top 64 bits
  const uint64_t sticky = (s == 64 ? lo : (lo << (64 - s))) != 0 ? 1ULL : 0ULL;
  return ldexp(__ull2double_rn(top | sticky), s);
}
// Q = qhi_sum * 2^32 + qlo_sum as a 128-bit value
__device__ __forceinline__ void limbs_to_u128(uint64_t hi_sum, uint64_t lo_sum, uint64_t& H, uint64_t& L) {
  const uint64_t a = hi_sum << 32;
  L = a + lo_sum;
  H = (hi_sum >> 32) + (L < a ? 1ULL : 0ULL);
}
__device__ void derive_dev(const DevPlatform& p, const uint64_t* w, magus_derived* out) {
  const uint64_t NT = w[MAGUS_TOT_N_STEPS], mint = w[MAGUS_TOT_MIN_INT];
  uint64_t h1, l1, h2, l2, h3, l3;
  limbs_to_u128(w[MAGUS_TOT_QMIN_HI], w[MAGUS_TOT_QMIN_LO], h1, l1);
  limbs_to_u128(w[MAGUS_TOT_QMAX_HI], w[MAGUS_TOT_QMAX_LO], h2, l2);
  limbs_to_u128(w[MAGUS_TOT_QBASE_HI], w[MAGUS_TOT_QBASE_LO], h3, l3);
  const uint64_t ls = l1 + l2, hs = h1 + h2 + (ls < l1 ? 1ULL : 0ULL);  // qmin + qmax
  const double ch = (double)w[MAGUS_TOT_CHANGES];
  const double time_max = p.dt * (double)(NT - mint) + p.cQ * u128_to_double_rn(h2, l2);
  const double time_min = p.dt * (double)mint + p.cQ * u128_to_double_rn(h1, l1);
  const double time = (p.dt * (double)NT + p.cQ * u128_to_double_rn(hs, ls)) + p.t_sw * ch;
  const double energy = (p.P_max * time_max + p.P_min * time_min) + p.e_sw * ch;
  const double base_time = p.dt * (double)NT + p.cQ * u128_to_double_rn(h3, l3);
  const double base_energy = p.P_max * base_time;
  out->energy_j = energy;
  out->time_s = time;
  out->base_energy_j = base_energy;
  out->base_time_s = base_time;
  out->saving = 1.0 - energy / base_energy;
  out->slowdown = time / base_time - 1.0;
  out->n_viol = (int64_t)w[MAGUS_TOT_N_VIOL];
  out->n_traces = (int64_t)w[MAGUS_TOT_N_TRACES];
  const uint64_t uni = w[MAGUS_TOT_BURST_BASE], inter = w[MAGUS_TOT_BURST_MAGUS];
  out->jaccard = uni ? (double)inter / (double)uni : 1.0;
}

// one thread: C <= a few hundred configs, a handful of fp64 ops each
__global__ void sweep_best_kernel(const uint64_t* __restrict__ tot, int32_t C, DevPlatform plat,
                                  SweepResult* __restrict__ res) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  int32_t b = -1, bi = 0;
  magus_derived db, di, dc;
  derive_dev(plat, tot, &di);  // infeasible fallback: argmin (n_viol, energy)
  for (int32_t c = 0; c < C; ++c) {
    derive_dev(plat, tot + (int64_t)c * MAGUS_TOT_WORDS, &dc);
    if (dc.n_viol == 0 && (b < 0 || dc.energy_j < db.energy_j)) { b = c; db = dc; }
    if (c > 0 && (dc.n_viol < di.n_viol || (dc.n_viol == di.n_viol && dc.energy_j < di.energy_j))) {
      bi = c;
      di = dc;
    }
  }
  res->feasible = b >= 0 ? 1 : 0;
  res->best = b >= 0 ? b : bi;
  res->row = b >= 0 ? db : di;
}

int launch_sweep_best(cudaStream_t s, const uint64_t* totals, int32_t C, const DevPlatform& plat,
                      SweepResult* res) {
  sweep_best_kernel<<<1, 32, 0, s>>>(totals, C, plat, res);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

__global__ void digest_table_kernel(unsigned long long* __restrict__ mul, int64_t nw) {
  const int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (w < nw) {  // 16-B rows so the stream kernel can bulk-copy one per stage
    mul[2 * w] = digest_mul(w);
    mul[2 * w + 1] = 0ULL;
  }
}

int launch_digest_table(cudaStream_t s, unsigned long long* mul, int64_t nw) {
  digest_table_kernel<<<(unsigned)((nw + 255) / 256), 256, 0, s>>>(mul, nw);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

// time-chunked generation: rows [t0, t0 + R) into out rows 0..R-1; the phase
// machine of each trace is carried in `state` between chunks (t0 = 0 seeds it)
__global__ void __launch_bounds__(128)
gen_resume_kernel(uint64_t seed, int64_t id0, int64_t N, int64_t t0, int64_t R, int64_t ld,
                  int32_t kind, mg_state* __restrict__ state, float* __restrict__ out) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= N) return;
  mg_state g;
  if (t0 == 0) mg_init(&g, seed, id0 + i, kind);
  else g = state[i];
  for (int64_t t = 0; t < R; ++t) out[t * ld + i] = (float)mg_step(&g);
  state[i] = g;
}

int launch_gen_resume(cudaStream_t s, uint64_t seed, int64_t id0, int64_t N, int64_t t0, int64_t R,
                      int64_t ld, int32_t kind, void* state, float* out) {
  gen_resume_kernel<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(seed, id0, N, t0, R, ld, kind,
                                                                (mg_state*)state, out);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}
size_t gen_state_bytes(int64_t N) { return sizeof(mg_state) * (size_t)N; }

int launch_gen(cudaStream_t s, uint64_t seed, int64_t id0, int64_t N, int64_t T, int64_t ld,
               int32_t kind, float* out) {
  gen_kernel<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(seed, id0, N, T, ld, kind, out);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
