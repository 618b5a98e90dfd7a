// kernels_post.cu -- segment carry resolution, per-config totals, and the
// device build of the synthetic trace generator.
#include "device_common.cuh"
#include "../../gen/magus_gen.h"

namespace magus {

// ---------------------------------------------------------------------------
// Fix-up: one thread per (trace, config) walks that pair's time segments in
// order.  Segment s was scanned under a hypothesis h for dec[t0-1] (max for
// s = 0, where it is the true init value P@23755; min otherwise).  The true
// carry is the last decision of the nearest earlier segment that contains an
// action (Alg. 3 is a sample-and-hold), else max.  Where it differs from h,
// only the segment prefix before its first action changes: its interval
// levels ([t0, a]) and decisions ([t0, a-1]) flip, which moves exactly the
// recorded prefix sums between the min/max accumulators, flips the change at
// a, and rewrites the prefix decision bits.  All sums are integers: exact.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(128)
fixup_kernel(int64_t N, int64_t T, int32_t C, DevPlatform plat, int64_t nseg, int64_t seg_len,
             SegRecords rec, magus_summary* __restrict__ out, magus_base* __restrict__ base,
             uint32_t* __restrict__ dec) {
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= N * C) return;
  const int32_t c = (int32_t)(gid / N);
  const int64_t n = gid - (int64_t)c * N;
  const int64_t nw = (T + 31) / 32;
  uint32_t carry = 0;  // dec[-1] = max
  int64_t ev = 0, hi = 0, msr = 0, ch = 0, mdec = 0, mint = 0;
  uint64_t qmin = 0, qmax = 0, qbase = 0, dig = 0;
  for (int64_t s = 0; s < nseg; ++s) {
    const int64_t r = ((int64_t)c * nseg + s) * N + n;
    const int64_t t0 = s * seg_len;
    const int64_t t1 = (t0 + seg_len < T) ? t0 + seg_len : T;
    const uint32_t fl = rec.flags[r];
    const uint32_t hyp = (fl & kFlagHypMin) ? 1u : 0u;
    const bool seen = (fl & kFlagSeen) != 0;
    ev += rec.ev[r];
    hi += rec.hi[r];
    msr += rec.msr[r];
    qbase += rec.qbase[r];
    int64_t s_ch = rec.ch[r], s_mdec = rec.mdec[r], s_mint = rec.mint[r];
    uint64_t s_qmin = rec.qmin[r], s_qmax = rec.qmax[r], s_dig = rec.dig[r];
    if (carry != hyp) {
      const uint32_t a_rel = rec.apos[r];
      const int64_t n_int = seen ? (int64_t)a_rel + 1 : t1 - t0;
      const int64_t n_dec = seen ? (int64_t)a_rel : t1 - t0;
      const uint64_t pqmin = rec.pqmin[r], pqmax = rec.pqmax[r], pdig = rec.pdig[r];
      if (hyp) {  // assumed min, truly max
        s_mint -= n_int; s_mdec -= n_dec;
        s_qmin -= pqmin; s_qmax += pqmax; s_dig -= pdig;
      } else {    // assumed max, truly min
        s_mint += n_int; s_mdec += n_dec;
        s_qmin += pqmin; s_qmax -= pqmax; s_dig += pdig;
      }
      if (seen) {
        const uint32_t Va = (fl & kFlagVa) ? 1u : 0u;
        s_ch += (int64_t)(Va != carry) - (int64_t)(Va != hyp);
      }
      if (dec) {
        for (int64_t p = t0; p < t0 + n_dec; p += 32) {  // t0 is word aligned
          const int64_t len = t0 + n_dec - p;
          const uint32_t mask = len >= 32 ? ~0u : ((1u << len) - 1u);
          uint32_t* wp = dec + ((int64_t)c * nw + (p >> 5)) * N + n;
          *wp = carry ? (*wp | mask) : (*wp & ~mask);
        }
      }
    }
    ch += s_ch; mdec += s_mdec; mint += s_mint;
    qmin += s_qmin; qmax += s_qmax; dig += s_dig;
    if (seen) carry = (fl & kFlagLastMin) ? 1u : 0u;
  }
  finalize_summary(plat, T, ev, hi, msr, ch, mdec, mint, qmin, qmax, qbase, dig,
                   out ? out + (int64_t)c * N + n : nullptr, (base && c == 0) ? base + n : nullptr);
}

int launch_fixup(cudaStream_t s, int64_t N, int64_t T, int32_t C, const DevPlatform& plat,
                 int64_t nseg, int64_t seg_len, const SegRecords& rec, magus_summary* out_summary,
                 magus_base* out_base, uint32_t* out_dec) {
  const int64_t blocks = (N * C + 127) / 128;
  fixup_kernel<<<(unsigned)blocks, 128, 0, s>>>(N, T, C, plat, nseg, seg_len, rec, out_summary,
                                                out_base, out_dec);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

// ---------------------------------------------------------------------------
// Per-config totals: exact integer sums over traces (order-free).
// ---------------------------------------------------------------------------
constexpr int kTotThreads = 256;
constexpr int kTotAcc = 13;

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
    tot[(int64_t)c * MAGUS_TOT_WORDS + 1 + threadIdx.x] = v;  // words 1..13
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

int launch_gen(cudaStream_t s, uint64_t seed, int64_t id0, int64_t N, int64_t T, int64_t ld,
               int32_t kind, float* out) {
  gen_kernel<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(seed, id0, N, T, ld, kind, out);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
