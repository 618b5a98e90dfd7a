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

int launch_gen(cudaStream_t s, uint64_t seed, int64_t id0, int64_t N, int64_t T, int64_t ld,
               int32_t kind, float* out) {
  gen_kernel<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(seed, id0, N, T, ld, kind, out);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
