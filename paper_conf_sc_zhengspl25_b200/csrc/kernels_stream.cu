// kernels_stream.cu -- the B200 hot path: TMA-staged, bit-parallel,
// time-segmented replay of Alg. 1-3 + model M, in ONE launch per (W, H).
//
// Layout and mapping:
//   * traces are time-major fp32 x[t][ld]; one CTA owns 128 consecutive
//     traces x one time segment [t0, t1) x one config; one consumer thread
//     owns one trace and scans it sequentially.
//   * a producer warp streams [32 steps x 128 traces] boxes (16 KB) into a
//     shared-memory ring with cp.async.bulk.tensor (TMA) completing on
//     mbarriers.  For a compile-time W the Alg. 1 lag x[t-W+1] is kept in
//     registers (each sample is widened to fp64 once), so a stage is released
//     as soon as its word is done (3 stages, 4 CTAs/SM).
//   * each consumer handles 32 steps at a time ("a word"): per sample it only
//     computes the Alg. 1 predicates (delta vs. host-inverted thresholds,
//     precompute.cpp) and the stretch flag, packed into 32-bit masks.  Alg. 2
//     (count of the H previous events >= k) is a bit-sliced carry-save
//     counter over 32 positions at once; Alg. 3's sample-and-hold of the
//     frequency is a 5-step log-depth forward fill; every counter is a popc.
//   * segments are exact (DESIGN 6.3): p_t and hi_t depend only on
//     x[t-W-H+1..t], so a segment re-reads a halo of ceil((W+H-1)/32) words;
//     the only carried state is dec[t0-1].  A segment scans under a
//     hypothesis for it, publishes {has-action, last decision} per trace,
//     and resolves its true carry by a decoupled look-back over earlier
//     segments (CTAs take work tickets in launch order, so every predecessor
//     is already resident: no deadlock).  Only the prefix before the first
//     action depends on the carry; its effect on the counters is a recorded
//     delta, its decision words are stored after the look-back.
//   * all accumulators are integers: per-segment sums are combined with
//     64-bit atomics (order-free, exact), the last segment CTA of each
//     (trace group, config) finalises the fp64 model-M quantities, and the
//     last group of each config writes the config's totals.  Any
//     segmentation gives bit-identical results.
#include <cuda.h>

#include "device_common.cuh"

namespace magus {
namespace {

constexpr int kTraces = 128;
constexpr int kRows = 32;
constexpr int kStageFloats = kTraces * kRows;           // 16 KB
constexpr int kConsumerWarps = kTraces / 32;
constexpr int kThreads = kTraces + 32;                  // + producer warp
constexpr uint32_t kStageBytes = kStageFloats * 4;
constexpr int kTotAcc = 13;

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
// try_wait with a suspend-time hint: a waiting warp is parked by the hardware
// instead of re-issuing the probe (the producer otherwise burns ~20 % of the
// SM's issue slots spinning on the empty barriers).
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity), "r"(0x989680u)
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
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void consumer_sync() {  // the 128 consumer threads only
  asm volatile("bar.sync 1, %0;" ::"n"(kTraces) : "memory");
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
__device__ __forceinline__ void or_if_gt(uint32_t& w, float a, float b, uint32_t bit) {
  asm("{\n.reg .pred p;\nsetp.gt.f32 p, %1, %2;\n@p or.b32 %0, %0, %3;\n}"
      : "+r"(w) : "f"(a), "f"(b), "r"(bit));
}

__device__ __forceinline__ uint32_t tail_mask(int64_t p0, int64_t T) {
  return (p0 + 32 <= T) ? ~0u : ((1u << (uint32_t)(T - p0)) - 1u);
}

#ifndef MAGUS_STAGES_REG
#define MAGUS_STAGES_REG 3
#endif
template <int W_T>
struct Stages {
  // register lag (compile-time W): a stage is free once its word is read;
  // runtime W reads the lag from the previous stage, held one word longer.
  static constexpr int n = W_T > 0 ? MAGUS_STAGES_REG : 4;
  static constexpr int smem = n * kStageFloats * 4;
};

template <int W_T, int H_T>
__global__ void __launch_bounds__(kThreads, W_T > 0 ? (MAGUS_STAGES_REG == 3 ? 4 : 3) : 3)
stream_kernel(const __grid_constant__ CUtensorMap tmap, int64_t N, int64_t T,
              const DevPolicy* __restrict__ pol, const int32_t* __restrict__ cidx, DevPlatform plat,
              int64_t nseg, int64_t seg_len, int32_t ngroups, int32_t nconf, StreamWork wk) {
  constexpr int kStages = Stages<W_T>::n;
  extern __shared__ __align__(1024) float sm[];
  __shared__ __align__(8) uint64_t full_bar[kStages];
  __shared__ __align__(8) uint64_t empty_bar[kStages];
  __shared__ uint32_t sh_ticket, sh_last, sh_last2;
  // per-stage word constants, computed by the producer lane off the critical path
  __shared__ unsigned long long st_mul[kStages];  // digest multiplier mix64(w) | 1
  __shared__ uint32_t st_warm[kStages];           // positions t < W (no MDFS round yet)
  __shared__ uint32_t st_tail[kStages];           // positions t < T
  __shared__ unsigned long long sh_red[kConsumerWarps][kTotAcc];

  if (threadIdx.x == 0) {
    sh_ticket = atomicAdd(wk.ticket, 1u);  // launch-order work ticket
    for (int i = 0; i < kStages; ++i) {
      mbar_init(&full_bar[i], 1);
      mbar_init(&empty_bar[i], kConsumerWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  // zero the ring (the runtime-W path's first word reads a "previous" stage)
  for (int i = threadIdx.x; i < kStages * kStageFloats; i += kThreads) sm[i] = 0.0f;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();

  // ticket -> (segment, config, group), segment-major so that the predecessor
  // segment of the same (config, group) always holds a smaller ticket
  const uint32_t ticket = sh_ticket;
  const int64_t per_seg = (int64_t)ngroups * nconf;
  const int64_t s = ticket / per_seg;
  const int32_t rem = (int32_t)(ticket - s * per_seg);
  const int32_t c = cidx[rem / ngroups];  // global config index
  const int32_t g = rem % ngroups;
  const int64_t t0 = s * seg_len;
  const int64_t t1 = (t0 + seg_len < T) ? t0 + seg_len : T;
  const DevPolicy P = pol[c];
  const int W = W_T > 0 ? W_T : P.W;
  const int H = H_T > 0 ? H_T : P.H;
  const int64_t wt0 = t0 >> 5;
  const int64_t wend = (t1 + 31) >> 5;
  int64_t nhalo = 0;
  if (s > 0) {
    nhalo = (W + H - 1 + 31) / 32;
    if (nhalo > wt0) nhalo = wt0;
  }
  const int64_t w_first = wt0 - nhalo;
  const int64_t nwords = wend - w_first;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == kConsumerWarps) {  // ---------------- producer warp ----------------
    if (lane == 0) {
      int st = 0;
      uint32_t ph = 0;
      for (int64_t j = 0; j < nwords; ++j) {
        if (j >= kStages) mbar_wait(&empty_bar[st], ph ^ 1u);
        const int64_t w = w_first + j, p0 = w * 32;
        st_mul[st] = digest_mul(w);
        st_warm[st] = (p0 >= W) ? 0u : ((W - p0) >= 32 ? ~0u : ((1u << (W - p0)) - 1u));
        st_tail[st] = tail_mask(p0, T);
        mbar_expect_tx(&full_bar[st], kStageBytes);  // arrive: releases the writes above
        tma_load_2d(sm + st * kStageFloats, &tmap, &full_bar[st], g * kTraces,
                    (int32_t)((w_first + j) * kRows));
        if (++st == kStages) { st = 0; ph ^= 1u; }
      }
    }
    return;
  }

  // ---------------- consumer: one trace per thread ----------------
  const int tid = threadIdx.x;
  const int64_t n = (int64_t)g * kTraces + tid;
  const bool valid = n < N;
  const double d_inc = P.d_inc, d_dec = P.d_dec;
  const KMask km = make_kmask(P.k);
  const float xthr_min = plat.xthr_min, xthr_max = plat.xthr_max;
  const double invB24_min = plat.invB24_min, invB24_max = plat.invB24_max;
  const uint32_t hyp = (s > 0) ? 1u : 0u;  // segment 0 starts from the true dec[-1] = max
  uint32_t Eprev = 0, carry = hyp, Dlast = 0;
  bool seen = false;
  uint32_t Va = 0, Dwa = 0, pre_dec_a = 0;
  int64_t apos = -1, wa = -1;
  uint32_t ev = 0, hi = 0, msr = 0, ch = 0, mdec = 0, mint = 0;
  unsigned long long qmin = 0, qmax = 0, qbase = 0, dig = 0, pqmin = 0, pqmax = 0, pdig = 0;
  uint32_t* dec_out = (wk.dec && valid) ? wk.dec + (int64_t)c * wk.dec_cstride + n : nullptr;
  uint32_t* dec_ptr = dec_out ? dec_out + wt0 * N : nullptr;  // advances one word row per word
  double pd[W_T > 1 ? W_T - 1 : 1];  // previous word's last W-1 samples, widened
#pragma unroll
  for (int k = 0; k < (W_T > 1 ? W_T - 1 : 1); ++k) pd[k] = 0.0;

  int st = 0, pst = kStages - 1;
  uint32_t ph = 0;
  for (int64_t j = 0; j < nwords; ++j) {
    mbar_wait(&full_bar[st], ph);
    const float* cur = sm + st * kStageFloats + tid;
    const int64_t w = w_first + j;
    const int64_t p0 = w * 32;

    // ---- per sample: Alg. 1 predicates + stretch flag, packed ----
    uint32_t incw = 0, decw = 0, smin = 0;
    float wmax = 0.0f;
    if constexpr (W_T > 0) {
      double xd[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const float xi = cur[i * kTraces];
        xd[i] = (double)xi;                                    // exact widening, once
        const double xl = (i >= W_T - 1) ? xd[i - (W_T - 1)] : pd[i];
        const double D = xd[i] - xl;                           // Alg. 1 l.3 numerator (RN)
        or_if_gt(incw, D, d_inc, 1u << i);                     // <=> RN(D / L) > tau_inc
        or_if_lt(decw, D, d_dec, 1u << i);                     // <=> RN(D / L) < tau_dec
        or_if_gt(smin, xi, xthr_min, 1u << i);                 // <=> RN(x / B_min) > 1
        wmax = fmaxf(wmax, xi);
      }
#pragma unroll
      for (int k = 0; k < W_T - 1; ++k) pd[k] = xd[32 - (W_T - 1) + k];
    } else {
      const float* prv = sm + pst * kStageFloats + tid;
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const float xi = cur[i * kTraces];
        const float* b = (i >= W - 1) ? cur : prv + 32 * kTraces;
        const float xl = b[(i - (W - 1)) * kTraces];
        const double D = (double)xi - (double)xl;
        if (D > d_inc) incw |= 1u << i;
        if (D < d_dec) decw |= 1u << i;
        if (xi > xthr_min) smin |= 1u << i;
        wmax = fmaxf(wmax, xi);
      }
    }
    const uint32_t warm = st_warm[st];
    const uint32_t incv = incw & ~warm;          // p = +1
    const uint32_t decv = decw & ~warm & ~incv;  // p = -1 (line 4 before line 6)
    const uint32_t E = incv | decv;              // uncore_tune_ls.push_back(1)

    if (w >= wt0) {
      const uint32_t outm = st_tail[st];
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
      const uint64_t M = st_mul[st];
      dig += (unsigned long long)Dout * M;
      uint32_t pre_int = 0;
      if (!seen) {  // prefix: decisions depend on the carry -> stored after the look-back
        const uint32_t Am = A & outm;
        uint32_t pre_dec;
        if (Am) {
          const int i = __ffs(Am) - 1;
          seen = true;
          apos = p0 + i;
          Va = (V >> i) & 1u;
          pre_int = (i == 31) ? ~0u : ((2u << i) - 1u);
          pre_dec = (1u << i) - 1u;
          wa = w;
          Dwa = Dout;
          pre_dec_a = pre_dec;
        } else {
          pre_int = outm;
          pre_dec = outm;
        }
        pdig += (unsigned long long)pre_dec * M;
      } else if (dec_ptr) {
        *dec_ptr = Dout;
      }
      if (dec_ptr) dec_ptr += N;
      // model M stretch: sparse over the samples that need it
      uint32_t mq = smin & (Lv | pre_int) & outm;
      while (mq) {  // order-free integer sums; two independent chains per trip
        const int i1 = 31 - __clz(mq);
        mq ^= 1u << i1;
        const int i2 = mq ? 31 - __clz(mq) : i1;
        const uint32_t m2 = mq ? 1u << i2 : 0u;
        mq ^= m2;
        const unsigned long long q1 = q_scaled(cur[i1 * kTraces], invB24_min);
        const unsigned long long q2 = m2 ? q_scaled(cur[i2 * kTraces], invB24_min) : 0ULL;
        if ((Lv >> i1) & 1u) qmin += q1;
        if ((pre_int >> i1) & 1u) pqmin += q1;
        if (Lv & m2) qmin += q2;
        if (pre_int & m2) pqmin += q2;
      }
      if (wmax > xthr_max) {  // some sample exceeds even the capacity at max
        uint32_t mx = smin & outm;  // x > xthr_max implies x > xthr_min
        while (mx) {
          const int i = 31 - __clz(mx);
          mx ^= 1u << i;
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
    __syncwarp();
    if constexpr (W_T > 0) {
      if (lane == 0) mbar_arrive(&empty_bar[st]);                      // word read: free
    } else {
      if (j >= 1 && lane == 0) mbar_arrive(&empty_bar[pst]);           // lag read: free
    }
    pst = st;
    if (++st == kStages) { st = 0; ph ^= 1u; }
  }

  // ---------------- epilogue: publish, look back, correct ----------------
  const uint32_t last_min = (Dlast >> (uint32_t)((t1 - 1) & 31)) & 1u;
  uint32_t* status = wk.status + ((int64_t)c * nseg) * N + n;
  if (valid) st_release(status + s * N, (wk.epoch << 3) | 1u | (seen ? 2u : 0u) | (last_min << 2));
  uint32_t cin = 0;  // true dec[t0-1]
  if (valid && s > 0) {
    for (int64_t jj = s - 1; jj >= 0; --jj) {
      uint32_t v;
      while (((v = ld_acquire(status + jj * N)) >> 3) != wk.epoch) __nanosleep(32);
      if (v & 2u) { cin = (v >> 2) & 1u; break; }
    }
  }
  if (valid) {
    if (cin != hyp) {
      const int64_t n_int = seen ? apos - t0 + 1 : t1 - t0;
      const int64_t n_dec = seen ? apos - t0 : t1 - t0;
      if (hyp) {  // assumed min, truly max
        mint -= (uint32_t)n_int; mdec -= (uint32_t)n_dec;
        qmin -= pqmin; qmax += pqmax; dig -= pdig;
      } else {    // assumed max, truly min
        mint += (uint32_t)n_int; mdec += (uint32_t)n_dec;
        qmin += pqmin; qmax -= pqmax; dig += pdig;
      }
      if (seen) ch += (uint32_t)((int)(Va != cin) - (int)(Va != hyp));
    }
    if (dec_out) {  // deferred prefix decision words
      const uint32_t fill = cin ? ~0u : 0u;
      const int64_t wlast = seen ? wa : wend;
      for (int64_t w = wt0; w < wlast; ++w) dec_out[w * N] = fill & tail_mask(w * 32, T);
      if (seen) dec_out[wa * N] = (Dwa & ~pre_dec_a) | (fill & pre_dec_a);
    }
    // segment sums -> per-(config, trace) accumulators (exact integer atomics)
    unsigned long long* acc = wk.acc + (int64_t)c * kAccFields * N + n;
    atomicAdd(acc + 0 * N, (unsigned long long)ev);
    atomicAdd(acc + 1 * N, (unsigned long long)hi);
    atomicAdd(acc + 2 * N, (unsigned long long)msr);
    atomicAdd(acc + 3 * N, (unsigned long long)(int64_t)(int32_t)ch);
    atomicAdd(acc + 4 * N, (unsigned long long)(int64_t)(int32_t)mdec);
    atomicAdd(acc + 5 * N, (unsigned long long)(int64_t)(int32_t)mint);
    atomicAdd(acc + 6 * N, qmin);
    atomicAdd(acc + 7 * N, qmax);
    atomicAdd(acc + 8 * N, qbase);
    atomicAdd(acc + 9 * N, dig);
  }
  __threadfence();
  consumer_sync();
  if (tid == 0) sh_last = (atomicAdd(wk.arrive + (int64_t)c * ngroups + g, 1u) == (uint32_t)(nseg - 1));
  consumer_sync();
  if (sh_last) {  // all segments of (config c, group g) are in: finalise the 128 traces
    __threadfence();
    unsigned long long tv[kTotAcc];
#pragma unroll
    for (int k = 0; k < kTotAcc; ++k) tv[k] = 0;
    if (valid) {
      unsigned long long* acc = wk.acc + (int64_t)c * kAccFields * N + n;
      unsigned long long a[kAccFields];
#pragma unroll
      for (int k = 0; k < kAccFields; ++k) {
        a[k] = __ldcg(acc + k * N);
        acc[k * N] = 0ULL;  // self-cleaning for the next replay
      }
      magus_summary sm_out;
      finalize_summary(plat, T, (int64_t)a[0], (int64_t)a[1], (int64_t)a[2], (int64_t)a[3],
                       (int64_t)a[4], (int64_t)a[5], a[6], a[7], a[8], a[9], &sm_out,
                       (wk.base && c == 0) ? wk.base + n : nullptr);
      if (wk.summary) wk.summary[(int64_t)c * N + n] = sm_out;
      tv[0] = (unsigned long long)sm_out.viol;
#pragma unroll
      for (int k = 0; k < 6; ++k) tv[1 + k] = a[k];
      tv[7] = a[6] & 0xFFFFFFFFULL; tv[8] = a[6] >> 32;
      tv[9] = a[7] & 0xFFFFFFFFULL; tv[10] = a[7] >> 32;
      tv[11] = a[8] & 0xFFFFFFFFULL; tv[12] = a[8] >> 32;
    }
    if (wk.totals) {  // per-config fleet totals (exact integer sums)
#pragma unroll
      for (int k = 0; k < kTotAcc; ++k) {
        unsigned long long v = tv[k];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xFFFFFFFFu, v, o);
        if (lane == 0) sh_red[warp][k] = v;
      }
      consumer_sync();
      if (tid < kTotAcc) {
        unsigned long long v = 0;
        for (int q = 0; q < kConsumerWarps; ++q) v += sh_red[q][tid];
        atomicAdd(wk.tacc + (int64_t)c * kTotAcc + tid, v);
      }
      __threadfence();
      consumer_sync();
      if (tid == 0) sh_last2 = (atomicAdd(wk.tarrive + c, 1u) == (uint32_t)(ngroups - 1));
      consumer_sync();
      if (sh_last2) {
        __threadfence();
        uint64_t* out = wk.totals + (int64_t)c * MAGUS_TOT_WORDS;
        if (tid < kTotAcc) {
          out[1 + tid] = __ldcg(wk.tacc + (int64_t)c * kTotAcc + tid);
          wk.tacc[(int64_t)c * kTotAcc + tid] = 0ULL;
        }
        if (tid == 0) {
          out[MAGUS_TOT_N_TRACES] = (uint64_t)N;
          out[MAGUS_TOT_N_STEPS] = (uint64_t)N * (uint64_t)T;
          out[MAGUS_TOT_RESERVED] = 0;
          wk.tarrive[c] = 0;
        }
      }
    }
    if (tid == 0) wk.arrive[(int64_t)c * ngroups + g] = 0;
  }
  if (tid == 0) {  // the last CTA of the launch re-arms the ticket counter
    __threadfence();
    if (atomicAdd(wk.done, 1u) == gridDim.x - 1) {
      *wk.ticket = 0;
      *wk.done = 0;
    }
  }
}

typedef void (*stream_fn)(CUtensorMap, int64_t, int64_t, const DevPolicy*, const int32_t*,
                          DevPlatform, int64_t, int64_t, int32_t, int32_t, StreamWork);

struct Pick {
  stream_fn f;
  int smem;
};

Pick pick(int32_t W, int32_t H) {
  if (H == 10) {
    switch (W) {
      case 4: return {stream_kernel<4, 10>, Stages<4>::smem};
      case 6: return {stream_kernel<6, 10>, Stages<6>::smem};
      case 10: return {stream_kernel<10, 10>, Stages<10>::smem};
      case 16: return {stream_kernel<16, 10>, Stages<16>::smem};
      default: break;
    }
    if (W >= 2 && W <= 33) return {stream_kernel<0, 10>, Stages<0>::smem};
  }
  if (W >= 2 && W <= 33 && H >= 1 && H <= 32) return {stream_kernel<0, 0>, Stages<0>::smem};
  return {nullptr, 0};
}

}  // namespace

bool stream_supported(int32_t W, int32_t H) { return pick(W, H).f != nullptr; }

int stream_ctas_per_sm(int32_t W, int32_t H) {
  Pick p = pick(W, H);
  if (!p.f) return 0;
  cudaFuncSetAttribute((const void*)p.f, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem);
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, (const void*)p.f, kThreads, p.smem) !=
      cudaSuccess)
    return 0;
  return nb;
}

int launch_stream(cudaStream_t st, const void* tmap, int64_t N, int64_t T,
                  const DevPolicy* pol_dev, const int32_t* cidx_dev, int32_t nc, int32_t W,
                  int32_t H, const DevPlatform& plat, int64_t nseg, int64_t seg_len,
                  const StreamWork& wk, int* grid_out) {
  Pick p = pick(W, H);
  if (!p.f) return -1;
  cudaFuncSetAttribute((const void*)p.f, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem);
  const int32_t ngroups = (int32_t)((N + kTraces - 1) / kTraces);
  const int64_t grid = (int64_t)ngroups * nseg * nc;
  if (grid_out) *grid_out = (int)grid;
  const CUtensorMap* m = reinterpret_cast<const CUtensorMap*>(tmap);
  p.f<<<(unsigned)grid, kThreads, p.smem, st>>>(*m, N, T, pol_dev, cidx_dev, plat, nseg, seg_len,
                                                ngroups, nc, wk);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
