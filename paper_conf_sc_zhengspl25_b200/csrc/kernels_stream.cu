// kernels_stream.cu -- the B200 hot path: TMA-staged, bit-parallel,
// time-segmented replay of Alg. 1-3 + model M.
//
// Layout and mapping:
//   * traces are time-major fp32 x[t][ld]; one CTA owns 128 consecutive
//     traces x one time segment [t0, t1) x one config; one consumer thread
//     owns one trace and scans it sequentially.
//   * a producer warp streams [32 steps x 128 traces] boxes (16 KB) into a
//     4-stage shared-memory ring with cp.async.bulk.tensor (TMA) completing
//     on mbarriers; consumer warps release a stage one word later (the Alg. 1
//     lag reaches W-1 <= 32 steps back).
//   * each consumer handles 32 steps at a time ("a word"): per sample it only
//     computes the Alg. 1 predicates (delta vs. host-inverted thresholds,
//     precompute.cpp) and the stretch flag, packed into 32-bit masks.  Alg. 2
//     (count of the H previous events >= k) is a bit-sliced carry-save
//     counter over 32 positions at once; Alg. 3's sample-and-hold of the
//     frequency is a 5-step log-depth forward fill; every counter is a popc.
//   * segments are exact (SURVEY PS3 / DESIGN 6.3): p_t and hi_t depend only
//     on x[t-W-H+1..t], so a segment re-reads a halo of ceil((W+H-1)/32)
//     words; the only carried state is dec[t0-1], which the kernel assumes
//     (hypothesis) and the fix-up kernel (kernels_post.cu) resolves exactly
//     from per-segment prefix records.  All accumulators are integers, so
//     any segmentation gives bit-identical results.
#include <cuda.h>

#include "device_common.cuh"

namespace magus {
namespace {

constexpr int kTraces = 128;
constexpr int kRows = 32;
constexpr int kStages = 4;
constexpr int kStageFloats = kTraces * kRows;           // 16 KB
constexpr int kConsumerWarps = kTraces / 32;
constexpr int kThreads = kTraces + 32;                  // + producer warp
constexpr uint32_t kStageBytes = kStageFloats * 4;
constexpr int kSmemBytes = kStages * kStageFloats * 4;  // 64 KB

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int32_t c0, int32_t c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}

// ---- Alg. 2, bit-parallel: bit i of the result = (#events at positions
// i-H .. i-1 >= k), positions < 0 coming from the previous word Ep. ----
struct KMask {
  uint32_t m[6];
};
__device__ __forceinline__ KMask make_kmask(int k) {
  KMask r;
#pragma unroll
  for (int j = 0; j < 6; ++j) r.m[j] = ((k >> j) & 1) ? ~0u : 0u;
  return r;
}
// count (bit-sliced, NB bits) >= k  <=>  no borrow out of count - k
template <int NB>
__device__ __forceinline__ uint32_t ge_k(const uint32_t* c, const KMask& km) {
  uint32_t b = 0;
#pragma unroll
  for (int j = 0; j < NB; ++j) b = (~c[j] & km.m[j]) | (~c[j] & b) | (km.m[j] & b);  // maj
#pragma unroll
  for (int j = NB; j < 6; ++j) b |= km.m[j];  // k >= 2^NB: always borrows
  return ~b;
}
__device__ __forceinline__ void fa(uint32_t a, uint32_t b, uint32_t c, uint32_t& s, uint32_t& cy) {
  s = a ^ b ^ c;
  cy = (a & b) | (c & (a ^ b));
}
template <int H>
struct Window {  // compile-time H: ripple-carry bit-sliced counter (6 bits, H <= 32)
  static __device__ __forceinline__ uint32_t ge(uint32_t E, uint32_t Ep, int, const KMask& km) {
    uint32_t c[6] = {0, 0, 0, 0, 0, 0};
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
    return ge_k<6>(c, km);
  }
};
template <>
struct Window<10> {  // the paper's H = 10 (P@24182): carry-save tree, 16 LOP3
  static __device__ __forceinline__ uint32_t ge(uint32_t E, uint32_t Ep, int, const KMask& km) {
    uint32_t s[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) s[j] = __funnelshift_l(Ep, E, j + 1);
    uint32_t a0, a1, b0, b1, c0, c1, d0, d1, f1, f2, g2;
    fa(s[0], s[1], s[2], a0, a1);
    fa(s[3], s[4], s[5], b0, b1);
    fa(s[6], s[7], s[8], c0, c1);
    fa(a0, b0, c0, d0, d1);
    uint32_t c[4];
    c[0] = d0 ^ s[9];
    const uint32_t e1 = d0 & s[9];
    fa(a1, b1, c1, f1, f2);
    fa(d1, e1, f1, c[1], g2);
    c[2] = f2 ^ g2;
    c[3] = f2 & g2;
    return ge_k<4>(c, km);
  }
};
template <>
struct Window<0> {  // runtime H <= 32
  static __device__ __forceinline__ uint32_t ge(uint32_t E, uint32_t Ep, int H, const KMask& km) {
    uint32_t c[6] = {0, 0, 0, 0, 0, 0};
    for (int j = 1; j <= H; ++j) {
      uint32_t b = __funnelshift_lc(Ep, E, j);  // clamps: j = 32 -> Ep
#pragma unroll
      for (int l = 0; l < 6; ++l) {
        const uint32_t t = c[l] & b;
        c[l] ^= b;
        b = t;
      }
    }
    return ge_k<6>(c, km);
  }
};

// ---- Alg. 3 sample-and-hold: D_i = V at the last action <= i, else carry ----
__device__ __forceinline__ uint32_t forward_fill(uint32_t A, uint32_t V, uint32_t carry_mask) {
  uint32_t y = V & A, m = A;
  y |= (y << 1) & ~m;  m |= m << 1;
  y |= (y << 2) & ~m;  m |= m << 2;
  y |= (y << 4) & ~m;  m |= m << 4;
  y |= (y << 8) & ~m;  m |= m << 8;
  y |= (y << 16) & ~m; m |= m << 16;
  return y | (carry_mask & ~m);
}

template <int W_T, int H_T>
__global__ void __launch_bounds__(kThreads)
stream_kernel(const __grid_constant__ CUtensorMap tmap, int64_t N, int64_t T,
              const DevPolicy* __restrict__ pol, const int32_t* __restrict__ cidx, DevPlatform plat,
              int64_t nseg, int64_t seg_len, int32_t ngroups, SegRecords rec,
              uint32_t* __restrict__ out_dec, int64_t dec_cstride) {
  extern __shared__ __align__(1024) float sm[];
  __shared__ __align__(8) uint64_t full_bar[kStages];
  __shared__ __align__(8) uint64_t empty_bar[kStages];

  const int32_t g = blockIdx.x % ngroups;
  const int64_t s = (blockIdx.x / ngroups) % nseg;
  const int32_t cl = cidx[blockIdx.x / ((int64_t)ngroups * nseg)];  // global config index
  const int64_t t0 = s * seg_len;
  const int64_t t1 = (t0 + seg_len < T) ? t0 + seg_len : T;
  const DevPolicy P = pol[cl];
  const int W = W_T > 0 ? W_T : P.W;
  const int H = H_T > 0 ? H_T : P.H;
  const int64_t wt0 = t0 >> 5;
  int64_t nhalo = 0;
  if (s > 0) {
    nhalo = (W + H - 1 + 31) / 32;
    if (nhalo > wt0) nhalo = wt0;
  }
  const int64_t w_first = wt0 - nhalo;
  const int64_t nwords = (t1 + 31) / 32 - w_first;

  // zero the ring (the first word's lag reads the "previous" stage), init barriers
  for (int i = threadIdx.x; i < kStages * kStageFloats; i += kThreads) sm[i] = 0.0f;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) {
      mbar_init(&full_bar[i], 1);
      mbar_init(&empty_bar[i], kConsumerWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == kConsumerWarps) {  // ---------------- producer warp ----------------
    if (lane == 0) {
      for (int64_t j = 0; j < nwords; ++j) {
        const int st = (int)(j % kStages);
        if (j >= kStages) mbar_wait(&empty_bar[st], (uint32_t)((j / kStages) - 1) & 1u);
        mbar_expect_tx(&full_bar[st], kStageBytes);
        tma_load_2d(sm + st * kStageFloats, &tmap, &full_bar[st], g * kTraces,
                    (int32_t)((w_first + j) * kRows));
      }
    }
    return;
  }

  // ---------------- consumer: one trace per thread ----------------
  const int tid = threadIdx.x;
  const int64_t n = (int64_t)g * kTraces + tid;
  const double d_inc = P.d_inc, d_dec = P.d_dec;
  const KMask km = make_kmask(P.k);
  const float xthr_min = plat.xthr_min, xthr_max = plat.xthr_max;
  const double invB24_min = plat.invB24_min, invB24_max = plat.invB24_max;
  const bool hyp_min = (s > 0);  // segment 0 starts from the true dec[-1] = max
  uint32_t Eprev = 0, carry = hyp_min ? 1u : 0u, Dlast = 0;
  bool seen = false;
  uint32_t Va = 0;
  int64_t apos = -1;
  uint32_t ev = 0, hi = 0, msr = 0, ch = 0, mdec = 0, mint = 0;
  unsigned long long qmin = 0, qmax = 0, qbase = 0, dig = 0, pqmin = 0, pqmax = 0, pdig = 0;
  uint32_t* dec_out = (out_dec && n < N) ? out_dec + (int64_t)cl * dec_cstride + n : nullptr;

  for (int64_t j = 0; j < nwords; ++j) {
    const int st = (int)(j % kStages);
    mbar_wait(&full_bar[st], (uint32_t)(j / kStages) & 1u);
    const float* cur = sm + st * kStageFloats + tid;
    const float* prv = sm + ((j + kStages - 1) % kStages) * kStageFloats + tid;
    const int64_t w = w_first + j;
    const int64_t p0 = w * 32;

    // ---- per-sample: Alg. 1 predicates + stretch flag, packed ----
    uint32_t incw = 0, decw = 0, smin = 0;
    float wmax = 0.0f;
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      const float xi = cur[i * kTraces];
      float xl;
      if (W_T > 0) {
        xl = (i >= W_T - 1) ? cur[(i - (W_T - 1)) * kTraces] : prv[(i - (W_T - 1) + 32) * kTraces];
      } else {
        const float* b = (i >= W - 1) ? cur : prv + 32 * kTraces;
        xl = b[(i - (W - 1)) * kTraces];
      }
      const double D = (double)xi - (double)xl;  // Alg. 1 l.3 numerator, RN fp64
      if (D > d_inc) incw |= 1u << i;            // <=> RN(D / L) > tau_inc
      if (D < d_dec) decw |= 1u << i;            // <=> RN(D / L) < tau_dec
      if (xi > xthr_min) smin |= 1u << i;        // <=> RN(x / B_min) > 1
      wmax = fmaxf(wmax, xi);
    }
    const uint32_t warm = (p0 >= W) ? 0u : ((W - p0) >= 32 ? ~0u : ((1u << (W - p0)) - 1u));
    const uint32_t incv = incw & ~warm;          // p = +1
    const uint32_t decv = decw & ~warm & ~incv;  // p = -1 (line 4 before line 6)
    const uint32_t E = incv | decv;              // uncore_tune_ls.push_back(1)

    if (w >= wt0) {
      const uint32_t outm = (p0 + 32 <= T) ? ~0u : ((1u << (uint32_t)(T - p0)) - 1u);
      // Alg. 2 + override (l.9-15): hi_t from the H events before t
      const uint32_t HI = Window<H_T>::ge(E, Eprev, H, km) & ~warm;
      const uint32_t act = HI | E;                 // tune_uncore_freq calls
      const uint32_t A = act | warm;               // positions that set the frequency
      const uint32_t V = decv & ~HI;               // ... to min (l.25)
      const uint32_t D = forward_fill(A, V, carry ? ~0u : 0u);
      const uint32_t Lv = (D << 1) | carry;        // interval level = dec[t-1]
      ev += __popc(E & outm);
      hi += __popc(HI & outm);
      msr += __popc(act & outm);
      uint32_t chm = (D ^ Lv) & outm;
      if (p0 == 0) chm &= ~1u;
      ch += __popc(chm);
      const uint32_t Dout = D & outm;
      mdec += __popc(Dout);
      mint += __popc(Lv & outm);
      const uint64_t M = digest_mul(w);
      dig += (unsigned long long)Dout * M;
      if (dec_out) dec_out[w * N] = Dout;
      uint32_t pre_int = 0;
      if (!seen) {
        const uint32_t Am = A & outm;
        uint32_t pre_dec;
        if (Am) {
          const int i = __ffs(Am) - 1;
          seen = true;
          apos = p0 + i;
          Va = (V >> i) & 1u;
          pre_int = (i == 31) ? ~0u : ((2u << i) - 1u);
          pre_dec = (1u << i) - 1u;
        } else {
          pre_int = outm;
          pre_dec = outm;
        }
        pdig += (unsigned long long)pre_dec * M;
      }
      // model M stretch: sparse over the samples that need it
      uint32_t mq = smin & (Lv | pre_int) & outm;
      while (mq) {
        const int i = __ffs(mq) - 1;
        mq &= mq - 1;
        const unsigned long long q = q_scaled(cur[i * kTraces], invB24_min);
        if ((Lv >> i) & 1u) qmin += q;
        if ((pre_int >> i) & 1u) pqmin += q;
      }
      if (wmax > xthr_max) {  // some sample exceeds even the capacity at max
        uint32_t mx = smin & outm;  // x > xthr_max implies x > xthr_min
        while (mx) {
          const int i = __ffs(mx) - 1;
          mx &= mx - 1;
          const float xi = cur[i * kTraces];
          if (xi > xthr_max) {
            const unsigned long long q = q_scaled(xi, invB24_max);
            qbase += q;
            if (!((Lv >> i) & 1u)) qmax += q;
            if ((pre_int >> i) & 1u) pqmax += q;
          }
        }
      }
      carry = D >> 31;
      Dlast = D;
    }
    Eprev = E;
    // release the previous stage (its rows were this word's lag)
    __syncwarp();
    if (j >= 1 && lane == 0) mbar_arrive(&empty_bar[(j - 1) % kStages]);
  }

  if (n < N) {
    const int64_t r = ((int64_t)cl * nseg + s) * N + n;
    const uint32_t last_min = (Dlast >> (uint32_t)((t1 - 1) & 31)) & 1u;
    rec.ev[r] = ev;
    rec.hi[r] = hi;
    rec.msr[r] = msr;
    rec.ch[r] = ch;
    rec.mdec[r] = mdec;
    rec.mint[r] = mint;
    rec.flags[r] = (hyp_min ? kFlagHypMin : 0u) | (seen ? kFlagSeen : 0u) | (Va ? kFlagVa : 0u) |
                   (last_min ? kFlagLastMin : 0u);
    rec.apos[r] = seen ? (uint32_t)(apos - t0) : 0xFFFFFFFFu;
    rec.qmin[r] = qmin;
    rec.qmax[r] = qmax;
    rec.qbase[r] = qbase;
    rec.dig[r] = dig;
    rec.pqmin[r] = pqmin;
    rec.pqmax[r] = pqmax;
    rec.pdig[r] = pdig;
  }
}

typedef void (*stream_fn)(CUtensorMap, int64_t, int64_t, const DevPolicy*, const int32_t*,
                          DevPlatform, int64_t, int64_t, int32_t, SegRecords, uint32_t*, int64_t);

stream_fn pick(int32_t W, int32_t H) {
  if (H == 10) {
    switch (W) {
      case 4: return stream_kernel<4, 10>;
      case 6: return stream_kernel<6, 10>;
      case 10: return stream_kernel<10, 10>;
      case 16: return stream_kernel<16, 10>;
      default: break;
    }
    if (W >= 2 && W <= 33) return stream_kernel<0, 10>;
  }
  if (W >= 2 && W <= 33 && H >= 1 && H <= 32) return stream_kernel<0, 0>;
  return nullptr;
}

}  // namespace

bool stream_supported(int32_t W, int32_t H) { return pick(W, H) != nullptr; }

int stream_ctas_per_sm(int32_t W, int32_t H) {
  stream_fn f = pick(W, H);
  if (!f) return 0;
  cudaFuncSetAttribute((const void*)f, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, (const void*)f, kThreads, kSmemBytes) !=
      cudaSuccess)
    return 0;
  return nb;
}

int launch_stream(cudaStream_t st, const void* tmap, int64_t N, int64_t T,
                  const DevPolicy* pol_dev, const int32_t* cidx_dev, int32_t nc, int32_t W,
                  int32_t H, const DevPlatform& plat, int64_t nseg, int64_t seg_len,
                  const SegRecords& rec, uint32_t* out_dec, int64_t dec_cstride, int* grid_out) {
  stream_fn f = pick(W, H);
  if (!f) return -1;
  cudaFuncSetAttribute((const void*)f, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
  const int32_t ngroups = (int32_t)((N + kTraces - 1) / kTraces);
  const int64_t grid = (int64_t)ngroups * nseg * nc;
  if (grid_out) *grid_out = (int)grid;
  const CUtensorMap* m = reinterpret_cast<const CUtensorMap*>(tmap);
  f<<<(unsigned)grid, kThreads, kSmemBytes, st>>>(*m, N, T, pol_dev, cidx_dev, plat, nseg, seg_len,
                                                  ngroups, rec, out_dec, dec_cstride);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
