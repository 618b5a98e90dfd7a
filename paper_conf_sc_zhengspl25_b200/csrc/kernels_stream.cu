// kernels_stream.cu -- the B200 hot path: TMA-staged, bit-parallel,
// time-segmented replay of Alg. 1-3 + model M, in ONE launch per (W, H).
//
// Layout and mapping:
//   * traces are time-major fp32 x[t][ld]; one CTA owns TR consecutive traces
//     (512 for one config per thread -- one CTA per SM, 16 consumer warps on
//     one ring; 128 for the config bundles of the sweeps, 3 CTAs per SM) x one
//     time segment [t0, t1) x one bundle of configs; one consumer thread owns
//     one trace and scans it sequentially.
//   * a producer warp streams [32 steps x 128 traces] TMA boxes (16 KB each,
//     TR / 128 per stage) into a shared-memory ring with
//     cp.async.bulk.tensor completing on mbarriers.  For a compile-time W the
//     Alg. 1 lag x[t-W+1] is kept in registers (each sample is widened to
//     fp64 once), so a stage is released as soon as its word is done
//     (3 stages).
//   * each consumer handles 32 steps at a time ("a word"): per sample it only
//     computes the Alg. 1 predicates (delta vs. host-inverted thresholds,
//     precompute.cpp) and the stretch flag, packed into 32-bit masks.  Alg. 2
//     (count of the H previous events >= k) is a bit-sliced carry-save
//     counter over 32 positions at once; Alg. 3's sample-and-hold of the
//     frequency is one carry-chain add (forward_fill); every counter is a
//     popc.
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

#include "bitops.cuh"
#include "device_common.cuh"
#include "ptx.cuh"

#ifndef MAGUS_BUNDLE_OCC
#define MAGUS_BUNDLE_OCC 4  // CTAs per SM of the compile-time-W config-bundle kernels (NB > 1): with
                            // 2 stages of 16 KB and <= 102 registers, 4 fit (config 3: 25.3 -> 24.0 ms
                            // against 3 CTAs x 3 stages; 4 CTAs x 3 stages do not fit the shared memory)
#endif

namespace magus {
namespace {

constexpr int kBox = 128;   // traces per TMA box ([32 steps x 128 traces], 16 KB)
constexpr int kRows = 32;
// A CTA owns TR traces (TR / 128 boxes per stage; the stage is laid out
// box-major, [box][32 steps][128 traces]).  TR = 512 for one config per
// thread (one CTA per SM: its 16 consumer warps share one ring, so they
// cannot drift apart the way 4 independent CTAs on an SM did), 128 else.
template <int TR>
struct Cta {
  static constexpr int traces = TR;
  static constexpr int boxes = TR / kBox;
  static constexpr int stage_floats = TR * kRows;            // 16 / 64 KB
  static constexpr uint32_t stage_bytes = stage_floats * 4;
  static constexpr int consumer_warps = TR / 32;
  static constexpr int threads = TR + 32;                    // + producer warp
};
constexpr int kTotAcc = kTotAccWords;

template <int TR>
__device__ __forceinline__ void consumer_sync() {  // the TR consumer threads only
  asm volatile("bar.sync 1, %0;" ::"n"(TR) : "memory");
}

template <int W_T, int TR>
struct Stages {
  // register lag (compile-time W): a stage is free once its word is read;
  // runtime W reads the lag from the previous stage, held one word longer.
  static constexpr int n = W_T > 0 ? (TR == 128 && MAGUS_BUNDLE_OCC > 3 ? 2 : 3) : 4;
  static constexpr int smem = n * Cta<TR>::stage_floats * 4;
};
// CTAs per SM the launch bounds aim for: NB configs per thread cost registers
template <int W_T, int NB, int TR>
struct Occ {
  static constexpr int v = TR > 128 ? 1 : (NB == 1 ? (W_T > 0 ? 4 : 3) : (W_T > 0 ? MAGUS_BUNDLE_OCC : 3));
};

// Per-config state of a bundle (NB configs that share W, H, L, tau_inc and
// tau_dec and differ only in t_hi, i.e. in k).  Hot state lives in registers
// (arrays indexed by compile-time constants only); state touched once per
// segment or only on rare paths lives in shared memory, [k][thread].
// For NB > 1 the per-segment counters are packed in 16-bit pairs (the host
// keeps segments <= 65,504 steps), which keeps NB = 4 at 3 CTAs/SM.
template <int NB>
struct BundleRegs {
  uint32_t cnt_a[NB];  // NB == 1: hi;   NB > 1: hi | msr << 16
  uint32_t cnt_b[NB];  // NB == 1: msr;  NB > 1: mdec | mint << 16
  uint32_t cnt_c[NB];  // NB == 1: mdec; NB > 1: ch
  uint32_t cnt_d[NB];  // NB == 1: mint, ch packed separately below
  uint32_t cnt_e[NB];
  uint32_t cnt_f[NB];  // bursts kept under MAGUS (NB > 1: | prefix bursts << 16)
  uint32_t cnt_g[NB];  // NB == 1: bursts in the carry-dependent prefix
  unsigned long long qmin[NB], dig[NB], pqmin[NB];
  uint32_t carry, seen, va;  // bit k per config
};
struct BundleSmem {  // rarely touched, per (config slot, thread)
  unsigned long long qmax, pqmax, pdig;
  int32_t apos, wa;
  uint32_t dwa, pre_dec_a;
};

template <int W_T, int H_T, int NB, bool BURST, int TR>
__global__ void __launch_bounds__(Cta<TR>::threads, Occ<W_T, NB, TR>::v)
stream_kernel(const __grid_constant__ CUtensorMap tmap, const __grid_constant__ CUtensorMap tmul,
              int64_t N, int64_t T,
              const DevPolicy* __restrict__ pol, const int32_t* __restrict__ bundles, DevPlatform plat,
              int64_t nseg, int64_t seg_len, int32_t ngroups, int32_t nbund, StreamWork wk) {
  constexpr int kStages = Stages<W_T, TR>::n;
  constexpr bool kPack = NB > 1;
  constexpr int kTraces = TR;
  constexpr int kStageFloats = Cta<TR>::stage_floats;
  constexpr uint32_t kStageBytes = Cta<TR>::stage_bytes;
  constexpr int kConsumerWarps = Cta<TR>::consumer_warps;
  constexpr int kThreads = Cta<TR>::threads;
  extern __shared__ __align__(1024) float sm[];
  __shared__ __align__(8) uint64_t full_bar[kStages];
  __shared__ __align__(8) uint64_t empty_bar[kStages];
  __shared__ uint32_t sh_last;
  __shared__ int32_t sh_work[4];  // segment, bundle, group of this CTA; its ticket
  __shared__ unsigned long long sh_red[kConsumerWarps][kTotAcc];
  // digest multiplier of each staged word, delivered by a 16-B bulk copy from
  // the context's table on the stage's own full barrier (async proxy, like
  // the samples; generic-proxy stores here would race the consumers' reads)
  // (tensor-copy destinations are 128-B aligned: one 128-B slot per stage)
  __shared__ __align__(128) unsigned long long st_mul[kStages][16];
  __shared__ BundleSmem bs[NB][kTraces];
  __shared__ __align__(16) uint32_t s_km[NB][8];

  if (threadIdx.x == 0) {
    // launch-order work ticket -> (segment, bundle, group), segment-major so
    // that the predecessor segment of the same (bundle, group) always holds a
    // smaller ticket; bundles of one (segment, group) take consecutive
    // tickets, so they start together and stream the same trace tiles while
    // those are still in L2
    const uint32_t ticket = atomicAdd(wk.ticket, 1u);
    sh_work[3] = (int32_t)ticket;
    const uint32_t per_seg = (uint32_t)ngroups * (uint32_t)nbund;
    const uint32_t sg = ticket / per_seg, rem = ticket - sg * per_seg;
    sh_work[0] = (int32_t)sg;
    sh_work[1] = (int32_t)(rem % (uint32_t)nbund);
    sh_work[2] = (int32_t)(rem / (uint32_t)nbund);
    for (int i = 0; i < kStages; ++i) {
      mbar_init(&full_bar[i], 1);
      mbar_init(&empty_bar[i], kConsumerWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if constexpr (W_T == 0) {  // the runtime-W path's first word reads a "previous" stage
    for (int i = threadIdx.x; i < kStages * kStageFloats; i += kThreads) sm[i] = 0.0f;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  if (sh_work[3] == 0 && wk.totals) {
    // The first CTA of the launch initialises the totals rows of the launch's
    // configs (the finalisers add into them, so no per-group hand-off through
    // a second arrival counter is needed) and raises the launch's flag.
    const int32_t rows = nbund * NB;
    for (int i = threadIdx.x; i < rows * MAGUS_TOT_WORDS; i += blockDim.x) {
      const int32_t c = bundles[i / MAGUS_TOT_WORDS];
      const int w = i % MAGUS_TOT_WORDS;
      if (c >= 0)
        wk.totals[(int64_t)c * MAGUS_TOT_WORDS + w] =
            w == MAGUS_TOT_N_TRACES ? (uint64_t)N : (w == MAGUS_TOT_N_STEPS ? (uint64_t)N * (uint64_t)T : 0ull);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      st_release(wk.ticket + kTotalsFlagWord, 1u);
    }
  }

  const int32_t s = sh_work[0];
  const int32_t bidx = sh_work[1];
  const int32_t g = sh_work[2];
  if (threadIdx.x == 0) {  // MAGUS_OPT_TRACE: per-CTA timeline
    if (unsigned long long* tr = trace_buf(wk)) {
      uint32_t smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      trace_put(tr, 0, gtimer());
      trace_put(tr, 4, smid);
      trace_put(tr, 5, (unsigned long long)s);
      trace_put(tr, 6, (unsigned long long)g);
    }
  }
  int32_t cfg[NB];
#pragma unroll
  for (int k = 0; k < NB; ++k) cfg[k] = bundles[bidx * NB + k];  // global config, -1 = pad
  const int32_t c0 = cfg[0];
  // global intervals (T = end of this call, buffer row r = interval wk.tb + r);
  // T <= 2^24: time fits in 32 bits
  const int32_t t0 = wk.ts + (int32_t)(s * seg_len);
  const int32_t t1 = (int32_t)((t0 + seg_len < T) ? t0 + seg_len : T);
  const DevPolicy P = pol[c0];
  const int W = W_T > 0 ? W_T : P.W;
  const int H = H_T > 0 ? H_T : P.H;
  const int32_t wt0 = t0 >> 5;
  const int32_t wend = (t1 + 31) >> 5;
  const int32_t ws = wk.ts >> 5;  // first output word
  int32_t nhalo = (W + H - 1 + 31) / 32;  // rows t0-W-H+1 .. t0-1 fix p and the history
  if (nhalo > wt0 - (wk.tb >> 5)) nhalo = wt0 - (wk.tb >> 5);  // (none before the buffer)
  const int32_t w_first = wt0 - nhalo;
  const int32_t nwords = wend - w_first;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == kConsumerWarps) {  // ---------------- producer warp ----------------
    if (lane == 0) {
      int st = 0;
      uint32_t ph = 0;
      for (int32_t j = 0; j < nwords; ++j) {
        if (j >= kStages) mbar_wait(&empty_bar[st], ph ^ 1u);
        mbar_expect_tx(&full_bar[st], kStageBytes + 16u);
        tma_load_1d(st_mul[st], &tmul, &full_bar[st], 2 * (w_first + j));
#pragma unroll
        for (int b = 0; b < Cta<TR>::boxes; ++b)
          tma_load_2d(sm + st * kStageFloats + b * (kBox * kRows), &tmap, &full_bar[st], g * kTraces + b * kBox,
                      (int32_t)((w_first + j) * kRows - wk.tb));
        if (++st == kStages) { st = 0; ph ^= 1u; }
      }
    }
    return;
  }

  // ---------------- consumer: one trace x NB configs per thread ----------------
  const int tid = threadIdx.x;
  const int64_t n = (int64_t)g * kTraces + tid;
  const bool valid = n < N;
  const double d_inc = P.d_inc, d_dec = P.d_dec;  // shared by the bundle
  int32_t kk[NB];
#pragma unroll
  for (int k = 0; k < NB; ++k) kk[k] = cfg[k] >= 0 ? pol[cfg[k]].k : 0x3F;
  const float xthr_min = plat.xthr_min, xthr_max = plat.xthr_max;
  const double invB24_min = plat.invB24_min, invB24_max = plat.invB24_max;
  // carry hypothesis, bit k per config: later segments assume min; segment 0
  // starts from the true dec[t_start-1] (max at t = 0, else the resume state)
  // (re-read in the epilogue rather than kept live across the scan)
  uint32_t hypm = (s > 0) ? (1u << NB) - 1u : 0u;
  if (s == 0 && wk.carry && valid) {
#pragma unroll
    for (int k = 0; k < NB; ++k)
      if (cfg[k] >= 0) hypm |= (__ldg(wk.carry + (int64_t)cfg[k] * N + n) & 1u) << k;
  }
  BundleRegs<NB> B;
#pragma unroll
  for (int k = 0; k < NB; ++k) {
    B.cnt_a[k] = 0; B.cnt_b[k] = 0; B.cnt_c[k] = 0; B.cnt_d[k] = 0; B.cnt_e[k] = 0;
    B.cnt_f[k] = 0; B.cnt_g[k] = 0;
    B.qmin[k] = 0; B.dig[k] = 0; B.pqmin[k] = 0;
    bs[k][tid].qmax = 0; bs[k][tid].pqmax = 0; bs[k][tid].pdig = 0;
    bs[k][tid].apos = -1; bs[k][tid].wa = -1; bs[k][tid].dwa = 0; bs[k][tid].pre_dec_a = 0;
  }
  B.carry = hypm;
  B.seen = 0; B.va = 0;
  uint32_t Eprev = 0, ev = 0, bbase = 0;
  unsigned long long qbase = 0;
  constexpr bool bursts = BURST;                    // Sec. 6.3 Jaccard counters (f1)
  const bool bkeep = plat.burst_min_keeps != 0;     // B_min > theta: no burst is hidden
  const float xburst = plat.xburst;
  const bool want_dec = wk.dec != nullptr && valid;
  // decision words of config cfg[0] (other bundle slots: + (cfg[k] - cfg[0]) * cstride)
  // (an integer address, advanced every word whether or not it is used)
  uint64_t dec_row = want_dec ? reinterpret_cast<uint64_t>(wk.dec + (int64_t)c0 * wk.dec_cstride +
                                                           (int64_t)(wt0 - ws) * N + n)
                              : 0;
  const uint64_t dec_step = 4ull * (uint64_t)N;
  double pd[W_T > 1 ? W_T - 1 : 1];  // previous word's last W-1 samples, widened
#pragma unroll
  for (int k = 0; k < (W_T > 1 ? W_T - 1 : 1); ++k) pd[k] = 0.0;

  // Alg. 2 threshold masks of each bundle slot (km[j] = all-ones iff bit j of
  // k is set), read back with one 16-B shared load per word and slot
  constexpr int kNBits = Window<H_T>::NBITS;
  static_assert(kNBits <= 8, "km table");
  if (tid < NB * kNBits) {
    const int kslot = tid / kNBits, j = tid % kNBits;
    int32_t kv = 0x3F;
#pragma unroll
    for (int k = 0; k < NB; ++k)
      if (k == kslot) kv = kk[k];
    s_km[kslot][j] = ((kv >> j) & 1) ? ~0u : 0u;
  }
  consumer_sync<TR>();
  const uint32_t km_s = smem_u32(&s_km[0][0]);
  const uint32_t full_s = smem_u32(&full_bar[0]), empty_s = smem_u32(&empty_bar[0]);
  // this thread's column: box tid / 128, lane-in-box tid % 128, row stride 128
  const int col = TR == kBox ? tid : (tid / kBox) * (kBox * kRows) + (tid % kBox);
  const uint32_t sm_s = smem_u32(sm) + 4u * (uint32_t)col;
  const uint32_t mul_s = smem_u32(&st_mul[0][0]);
  // words of the trace's last (partial) word and of the warm-up
  const int32_t Ti = (int32_t)T;
  const int32_t w_tail = (Ti - 1) >> 5;
  const uint32_t tail_m = (Ti & 31) ? ((1u << (Ti & 31)) - 1u) : ~0u;

  // one 32-step word of the scan; st / pst = stage of this / the previous word
  auto word = [&](const int st, const int pst, const uint32_t ph, const int32_t j)
                  __attribute__((always_inline)) {
    mbar_wait_full(full_s + 8u * (uint32_t)st, ph);
    const float* cur = sm + st * kStageFloats + col;
    const uint32_t cur_s = sm_s + (uint32_t)(st * kStageFloats * 4);
    const int32_t w = w_first + j;
    const int32_t p0 = w * 32;

    // ---- per sample: Alg. 1 predicates + stretch flag, packed ----
    uint32_t incw = 0, decw = 0, smin = 0;
    float wmax = 0.0f;
    if constexpr (W_T > 0) {
      double xd[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const float xi = cur[i * kBox];
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
      const float* prv = sm + pst * kStageFloats + col;
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const float xi = cur[i * kBox];
        const float* b = (i >= W - 1) ? cur : prv + 32 * kBox;
        const float xl = b[(i - (W - 1)) * kBox];
        const double D = (double)xi - (double)xl;
        if (D > d_inc) incw |= 1u << i;
        if (D < d_dec) decw |= 1u << i;
        if (xi > xthr_min) smin |= 1u << i;
        wmax = fmaxf(wmax, xi);
      }
    }
    // warm-up rounds t < W (Alg. 3 runs from t = W): words 0 and (W = 33) 1 only
    uint32_t warm;
    if constexpr (W_T > 0) {
      constexpr uint32_t kWarm0 = W_T >= 32 ? ~0u : ((1u << W_T) - 1u);
      constexpr uint32_t kWarm1 = W_T > 32 ? ((1u << (W_T - 32)) - 1u) : 0u;
      warm = (p0 == 0) ? kWarm0 : ((W_T > 32 && p0 == 32) ? kWarm1 : 0u);
    } else {
      warm = (p0 >= W) ? 0u : ((W - p0) >= 32 ? ~0u : ((1u << (W - p0)) - 1u));
    }
    const uint32_t incv = incw & ~warm;          // p = +1
    const uint32_t decv = decw & ~warm & ~incv;  // p = -1 (line 4 before line 6)
    const uint32_t E = incv | decv;              // uncore_tune_ls.push_back(1)

    if (w >= wt0) {
      const uint32_t outm = (w == w_tail) ? tail_m : ~0u;
      const uint64_t M = lds_u64(mul_s + 128u * (uint32_t)st);  // digest multiplier mix64(w) | 1
      ev += __popc(E & outm);
      uint32_t bb = 0;  // bursts at max uncore: delivered x > theta
      if constexpr (bursts) {
#pragma unroll
        for (int i = 0; i < 32; ++i) or_if_gt(bb, cur[i * kBox], xburst, 1u << i);
        bb &= outm;
        bbase += __popc(bb);
      }
      // Alg. 2 (l.9): the count of the H previous events, shared by the bundle
      uint32_t cnt[kNBits];
      Window<H_T>::count(E, Eprev, H, cnt);
      uint32_t Lv[NB], pre_int[NB];
      uint32_t need_q = 0, pre_any = 0;
#pragma unroll
      for (int k = 0; k < NB; ++k) {
        const uint32_t ck = (B.carry >> k) & 1u;
        uint32_t km[kNBits];
        {
          const uint4 a = lds_v4(km_s + 32u * k);
          km[0] = a.x; km[1] = a.y; km[2] = a.z; km[3] = a.w;
          if constexpr (kNBits > 4) {
            const uint4 b2 = lds_v4(km_s + 32u * k + 16u);
            km[4] = b2.x; km[5] = b2.y;
          }
        }
        const uint32_t HI = ge_k<kNBits>(cnt, km) & ~warm;
        const uint32_t act = HI | E;                 // tune_uncore_freq calls (l.11/19/25)
        const uint32_t A = act | warm;               // positions that set the frequency
        const uint32_t V = decv & ~HI;               // ... to min (l.25)
        const uint32_t D = forward_fill(A, V, ck);
        Lv[k] = (D << 1) | ck;                       // interval level = dec[t-1]
        // (t = 0: D_0 = 0 (warm-up) and the carry is max, so bit 0 is clear)
        const uint32_t chm = (D ^ Lv[k]) & outm;
        const uint32_t Dout = D & outm;
        if constexpr (kPack) {
          B.cnt_a[k] += (uint32_t)__popc(HI & outm) | ((uint32_t)__popc(act & outm) << 16);
          B.cnt_b[k] += (uint32_t)__popc(Dout) | ((uint32_t)__popc(Lv[k] & outm) << 16);
          B.cnt_c[k] += (uint32_t)__popc(chm);
        } else {
          B.cnt_a[k] += __popc(HI & outm);
          B.cnt_b[k] += __popc(act & outm);
          B.cnt_c[k] += __popc(Dout);
          B.cnt_d[k] += __popc(Lv[k] & outm);
          B.cnt_e[k] += __popc(chm);
        }
        B.dig[k] += (unsigned long long)Dout * M;
        pre_int[k] = 0;
        if (!((B.seen >> k) & 1u)) {  // prefix: depends on the carry -> resolved later
          const uint32_t Am = A & outm;
          uint32_t pre_dec;
          if (Am) {
            const int i = __ffs(Am) - 1;
            B.seen |= 1u << k;
            B.va |= ((V >> i) & 1u) << k;
            pre_int[k] = (i == 31) ? ~0u : ((2u << i) - 1u);
            pre_dec = (1u << i) - 1u;
            bs[k][tid].apos = (int32_t)(p0 + i - t0);
            bs[k][tid].wa = (int32_t)(w - wt0);
            bs[k][tid].dwa = Dout;
            bs[k][tid].pre_dec_a = pre_dec;
          } else {
            pre_int[k] = outm;
            pre_dec = outm;
          }
          bs[k][tid].pdig += (unsigned long long)pre_dec * M;
        } else if (want_dec && cfg[k] >= 0) {
          reinterpret_cast<uint32_t*>(dec_row)[(int64_t)(cfg[k] - c0) * wk.dec_cstride] = Dout;
        }
        if constexpr (bursts) {  // kept unless the interval ran at a level whose capacity hides it
          const uint32_t kept = bkeep ? bb : (bb & ~Lv[k]);
          const uint32_t pb = bkeep ? 0u : (bb & pre_int[k]);
          if constexpr (kPack) B.cnt_f[k] += (uint32_t)__popc(kept) | ((uint32_t)__popc(pb) << 16);
          else { B.cnt_f[k] += __popc(kept); B.cnt_g[k] += __popc(pb); }
        }
        need_q |= Lv[k];
        pre_any |= pre_int[k];
        B.carry = (B.carry & ~(1u << k)) | ((D >> 31) << k);
      }
      dec_row += dec_step;
      // model M stretch at min: once per sample, shared by the bundle
      if (wmax <= xthr_max && pre_any == 0) {
        // common case: no sample above the capacity at max (so s24 < 127 * 2^24
        // needs no cap: ratio_max <= 127), no carry-dependent prefix
        uint32_t mq = smin & need_q & outm;
        while (mq) {  // order-free integer sums; two independent chains per trip
          const int i1 = 31 - __clz(mq);
          mq ^= 1u << i1;
          const int i2 = mq ? 31 - __clz(mq) : i1;
          const uint32_t m2 = mq ? 1u << i2 : 0u;
          mq ^= m2;
          const unsigned long long q1 = q_scaled_nocap(lds_f32(cur_s + 512u * i1), invB24_min);
          const unsigned long long q2 = q_scaled_nocap(lds_f32(cur_s + 512u * i2), invB24_min);
          if constexpr (NB == 1) {
            B.qmin[0] += q1 + (m2 ? q2 : 0ULL);
          } else {
#pragma unroll
            for (int k = 0; k < NB; ++k) {
              if ((Lv[k] >> i1) & 1u) B.qmin[k] += q1;
              if (Lv[k] & m2) B.qmin[k] += q2;
            }
          }
        }
      } else {
        uint32_t mq = smin & (need_q | pre_any) & outm;
        while (mq) {
          const int i1 = 31 - __clz(mq);
          const uint32_t m1 = 1u << i1;
          mq ^= m1;
          const unsigned long long q1 = q_scaled(lds_f32(cur_s + 512u * i1), invB24_min);
#pragma unroll
          for (int k = 0; k < NB; ++k) {
            if (Lv[k] & m1) B.qmin[k] += q1;
            if (pre_int[k] & m1) B.pqmin[k] += q1;
          }
        }
        if (wmax > xthr_max) {  // some sample exceeds even the capacity at max (rare)
          uint32_t mx = smin & outm;  // x > xthr_max implies x > xthr_min
          while (mx) {
            const int i = 31 - __clz(mx);
            const uint32_t m1 = 1u << i;
            mx ^= m1;
            const float xi = lds_f32(cur_s + 512u * i);
            if (xi > xthr_max) {
              const unsigned long long q = q_scaled(xi, invB24_max);
              qbase += q;
#pragma unroll
              for (int k = 0; k < NB; ++k) {
                if (!(Lv[k] & m1)) bs[k][tid].qmax += q;
                if (pre_int[k] & m1) bs[k][tid].pqmax += q;
              }
            }
          }
        }
      }
    }
    Eprev = E;
    __syncwarp();
    if constexpr (W_T > 0) {
      if (lane == 0) mbar_arrive_s(empty_s + 8u * (uint32_t)st);          // word read: free
    } else {
      if (j >= 1 && lane == 0) mbar_arrive_s(empty_s + 8u * (uint32_t)pst);  // lag read: free
    }
  };
  if constexpr (NB == 1) {
    // one config per thread: the ring is unrolled by its depth, so the stage
    // (and with it every shared address of the word) is a compile-time
    // constant (the 4-config body is too large to triple: I-cache)
    uint32_t ph = 0;
    for (int32_t j0 = 0; j0 < nwords; j0 += kStages, ph ^= 1u) {
#pragma unroll
      for (int st = 0; st < kStages; ++st) {
        if (j0 + st >= nwords) break;
        word(st, st == 0 ? kStages - 1 : st - 1, ph, j0 + st);
      }
    }
  } else {
    int st = 0, pst = kStages - 1;
    uint32_t ph = 0;
    for (int32_t j = 0; j < nwords; ++j) {
      word(st, pst, ph, j);
      pst = st;
      if (++st == kStages) { st = 0; ph ^= 1u; }
    }
  }

  // ---------------- epilogue: publish, look back, correct ----------------
  if (tid == 0)
    if (unsigned long long* tr = trace_buf(wk)) trace_put(tr, 1, gtimer());
  {
  // the work coordinates, re-derived from the ticket rather than kept live
  // across the scan (shadowing the names above)
  const int32_t s = *(volatile int32_t*)&sh_work[0];
  const int32_t bidx = *(volatile int32_t*)&sh_work[1];
  const int32_t g = *(volatile int32_t*)&sh_work[2];
  int32_t cfg[NB];
#pragma unroll
  for (int k = 0; k < NB; ++k) cfg[k] = __ldg(bundles + bidx * NB + k);
  const int32_t c0 = cfg[0];
  const int32_t t0 = wk.ts + (int32_t)(s * seg_len);
  const int32_t t1 = (int32_t)((t0 + seg_len < T) ? t0 + seg_len : T);
  const int32_t wt0 = t0 >> 5;
  const int32_t wend = (t1 + 31) >> 5;
  const int32_t ws = wk.ts >> 5;
  const int64_t n = (int64_t)g * kTraces + tid;
  const bool valid = n < N;
#pragma unroll
  for (int k = 0; k < NB; ++k) {
    const int32_t c = cfg[k];
    if (!valid || c < 0) continue;
    // dec[t1-1] = bit 31 of the last word's fill when t1 % 32 == 0, i.e. for
    // every segment but a trace's final one, whose status nobody reads (a
    // resumed chunk boundary is a multiple of 32 by contract)
    const uint32_t seen = (B.seen >> k) & 1u, last_min = (B.carry >> k) & 1u;
    uint32_t* status = wk.status + ((int64_t)c * nseg) * N + n;
    st_release(status + s * N, (wk.epoch << 3) | 1u | (seen << 1) | (last_min << 2));
  }
#pragma unroll
  for (int k = 0; k < NB; ++k) {
    const int32_t c = cfg[k];
    if (!valid || c < 0) continue;
    const bool seen = (B.seen >> k) & 1u;
    const BundleSmem& S = bs[k][tid];
    uint32_t* status = wk.status + ((int64_t)c * nseg) * N + n;
    const uint32_t hyp =
        (s > 0) ? 1u : (wk.carry ? (__ldg(wk.carry + (int64_t)c * N + n) & 1u) : 0u);
    uint32_t cin = hyp;  // true dec[t0-1] (segment 0: known)
    if (s > 0) {
      // no action since the chunk start: the resume carry (read before this
      // launch's finaliser may rewrite it: that waits for every segment)
      cin = wk.carry ? (wk.carry[(int64_t)c * N + n] & 1u) : 0u;
      for (int64_t jj = s - 1; jj >= 0; --jj) {
        uint32_t v;
        while (((v = ld_acquire(status + jj * N)) >> 3) != wk.epoch) __nanosleep(MAGUS_LOOKBACK_SLEEP);
        if (v & 2u) { cin = (v >> 2) & 1u; break; }
      }
    }
    if (tid == 0 && k == 0)
      if (unsigned long long* tr = trace_buf(wk)) trace_put(tr, 2, gtimer());
    if (wk.carry && s == nseg - 1)  // no successor reads it: republish as the chunk's final dec
      st_release(status + s * N, (wk.epoch << 3) | 3u | ((seen ? (B.carry >> k) & 1u : cin) << 2));
    uint32_t hi, msr, mdec, mint, ch, bm, pb;
    if constexpr (kPack) {
      hi = B.cnt_a[k] & 0xFFFFu; msr = B.cnt_a[k] >> 16;
      mdec = B.cnt_b[k] & 0xFFFFu; mint = B.cnt_b[k] >> 16;
      ch = B.cnt_c[k];
      bm = B.cnt_f[k] & 0xFFFFu; pb = B.cnt_f[k] >> 16;
    } else {
      hi = B.cnt_a[k]; msr = B.cnt_b[k]; mdec = B.cnt_c[k]; mint = B.cnt_d[k]; ch = B.cnt_e[k];
      bm = B.cnt_f[k]; pb = B.cnt_g[k];
    }
    unsigned long long qmin = B.qmin[k], qmax = S.qmax, dig = B.dig[k];
    if (cin != hyp) {
      const uint32_t n_int = seen ? (uint32_t)S.apos + 1u : (uint32_t)(t1 - t0);
      const uint32_t n_dec = seen ? (uint32_t)S.apos : (uint32_t)(t1 - t0);
      if (hyp) {  // assumed min, truly max
        mint -= n_int; mdec -= n_dec;
        qmin -= B.pqmin[k]; qmax += S.pqmax; dig -= S.pdig;
        bm += pb;
      } else {    // assumed max, truly min
        mint += n_int; mdec += n_dec;
        qmin += B.pqmin[k]; qmax -= S.pqmax; dig += S.pdig;
        bm -= pb;
      }
      const uint32_t va = (B.va >> k) & 1u;
      if (seen) ch += (uint32_t)((int)(va != cin) - (int)(va != hyp));
    }
    if (want_dec) {  // deferred prefix decision words
      uint32_t* dec_out = wk.dec + (int64_t)c * wk.dec_cstride + n;
      const uint32_t fill = cin ? ~0u : 0u;
      const int32_t wlast = seen ? wt0 + S.wa : wend;
      for (int32_t w = wt0; w < wlast; ++w) dec_out[(w - ws) * N] = fill & tail_mask(w * 32, T);
      if (seen) dec_out[(wt0 + S.wa - ws) * N] = (S.dwa & ~S.pre_dec_a) | (fill & S.pre_dec_a);
    }
    // segment sums -> per-(config, trace) accumulators (exact integer atomics)
    unsigned long long* acc = wk.acc + (int64_t)c * kAccFields * N + n;
    atomicAdd(acc + 0 * N, (unsigned long long)ev);
    atomicAdd(acc + 1 * N, (unsigned long long)hi);
    atomicAdd(acc + 2 * N, (unsigned long long)msr);
    atomicAdd(acc + 3 * N, (unsigned long long)ch);
    atomicAdd(acc + 4 * N, (unsigned long long)mdec);
    atomicAdd(acc + 5 * N, (unsigned long long)mint);
    atomicAdd(acc + 6 * N, qmin);
    atomicAdd(acc + 7 * N, qmax);
    atomicAdd(acc + 8 * N, qbase);
    atomicAdd(acc + 9 * N, dig);
    if constexpr (BURST) {  // (the burst accumulators stay zero otherwise)
      atomicAdd(acc + 10 * N, (unsigned long long)bbase);
      atomicAdd(acc + 11 * N, (unsigned long long)bm);
    }
  }
  __threadfence();
  consumer_sync<TR>();
  if (tid == 0) sh_last = (atomicAdd(wk.arrive + (int64_t)c0 * ngroups + g, 1u) == (uint32_t)(nseg - 1));
  consumer_sync<TR>();
  if (sh_last) {  // all segments of (bundle, group g) are in: finalise the 128 traces
    __threadfence();
#pragma unroll 1
    for (int k = 0; k < NB; ++k) {
      const int32_t c = cfg[k];
      if (c < 0) continue;  // uniform across the CTA
      unsigned long long tv[kTotAcc];
#pragma unroll
      for (int q = 0; q < kTotAcc; ++q) tv[q] = 0;
      if (valid) {
        unsigned long long* acc = wk.acc + (int64_t)c * kAccFields * N + n;
        unsigned long long a[kAccFields];
#pragma unroll
        for (int q = 0; q < kAccFields; ++q) {
          a[q] = __ldcg(acc + q * N);
          if (!wk.carry) acc[q * N] = 0ULL;  // self-cleaning for the next replay
        }
        if (wk.carry)  // resume state: dec at the chunk's last interval (see above)
          wk.carry[(int64_t)c * N + n] = (__ldcg(wk.status + ((int64_t)c * nseg + nseg - 1) * N + n) >> 2) & 1u;
        magus_summary sm_out;
        finalize_summary(plat, T, (int64_t)a[0], (int64_t)a[1], (int64_t)a[2], (int64_t)a[3],
                         (int64_t)a[4], (int64_t)a[5], a[6], a[7], a[8], a[9], (int64_t)a[10],
                         (int64_t)a[11], &sm_out,
                         (wk.base && c == 0) ? wk.base + n : nullptr);
        if (wk.summary) wk.summary[(int64_t)c * N + n] = sm_out;
        tv[0] = (unsigned long long)sm_out.viol;
#pragma unroll
        for (int q = 0; q < 6; ++q) tv[1 + q] = a[q];
        tv[7] = a[6] & 0xFFFFFFFFULL; tv[8] = a[6] >> 32;
        tv[9] = a[7] & 0xFFFFFFFFULL; tv[10] = a[7] >> 32;
        tv[11] = a[8] & 0xFFFFFFFFULL; tv[12] = a[8] >> 32;
        tv[13] = a[10]; tv[14] = a[11];
      }
      if (wk.totals) {  // per-config fleet totals (exact integer sums)
#pragma unroll
        for (int q = 0; q < kTotAcc; ++q) {
          const unsigned long long v = warp_sum_tot(tv[q], q);
          if (lane == 0) sh_red[warp][q] = v;
        }
        consumer_sync<TR>();
        if (tid < kTotAcc) {  // accumulators 0..12 -> words 1..13; 13, 14 -> bursts (exact integer adds)
          unsigned long long v = 0;
          for (int q = 0; q < kConsumerWarps; ++q) v += sh_red[q][tid];
          // the launch's first CTA initialised the rows (its flag, normally
          // raised long before any group is complete)
          while (ld_acquire(wk.ticket + kTotalsFlagWord) == 0u) __nanosleep(MAGUS_LOOKBACK_SLEEP);
          const int word = tid < 13 ? 1 + tid : MAGUS_TOT_BURST_BASE + (tid - 13);
          atomicAdd(reinterpret_cast<unsigned long long*>(wk.totals + (int64_t)c * MAGUS_TOT_WORDS + word), v);
        }
        consumer_sync<TR>();  // sh_red is reused by the next config
      }
    }
    if (tid == 0) wk.arrive[(int64_t)c0 * ngroups + g] = 0;
  }
  }
  if (tid == 0) {
    if (unsigned long long* tr = trace_buf(wk)) {
      trace_put(tr, 3, gtimer());
      trace_put(tr, 7, sh_last);
    }
  }
  if (tid == 0) {  // the last CTA of the launch re-arms the ticket counter
    __threadfence();
    if (atomicAdd(wk.done, 1u) == gridDim.x - 1) {
      *wk.ticket = 0;
      *wk.done = 0;
      wk.ticket[kTotalsFlagWord] = 0;
    }
  }
}

typedef void (*stream_fn)(CUtensorMap, CUtensorMap, int64_t, int64_t, const DevPolicy*, const int32_t*,
                          DevPlatform, int64_t, int64_t, int32_t, int32_t, StreamWork);

struct Pick {
  stream_fn f;
  int smem;
  int threads;
  int traces;  // per CTA
};

template <int W_T, int H_T, int NB, bool BURST, int TR>
Pick mk() {
  return {stream_kernel<W_T, H_T, NB, BURST, TR>, Stages<W_T, TR>::smem, Cta<TR>::threads, TR};
}

// one config per thread with a compile-time W (the paper's H = 10): 512
// traces per CTA unless `narrow`; everything else 128
template <int NB, bool BURST>
Pick pick_nb(int32_t W, int32_t H, bool narrow) {
  if (H == 10) {
    if constexpr (NB == 1) {
      if (!narrow) {
        switch (W) {
          case 4: return mk<4, 10, NB, BURST, 512>();
          case 6: return mk<6, 10, NB, BURST, 512>();
          case 10: return mk<10, 10, NB, BURST, 512>();
          case 16: return mk<16, 10, NB, BURST, 512>();
          default: break;
        }
      }
    }
    switch (W) {
      case 4: return mk<4, 10, NB, BURST, 128>();
      case 6: return mk<6, 10, NB, BURST, 128>();
      case 10: return mk<10, 10, NB, BURST, 128>();
      case 16: return mk<16, 10, NB, BURST, 128>();
      default: break;
    }
    if (W >= 2 && W <= 33) return mk<0, 10, NB, BURST, 128>();
  }
  if (W >= 2 && W <= 33 && H >= 1 && H <= 32) return mk<0, 0, NB, BURST, 128>();
  return {nullptr, 0, 0, 0};
}

// The Sec. 6.3 burst counters are a compile-time flag so that the default
// path carries none of their registers.
Pick pick(int32_t W, int32_t H, int32_t NB, bool burst, bool narrow) {
  switch (NB * 2 + (burst ? 1 : 0)) {
    case 2: return pick_nb<1, false>(W, H, narrow);
    case 3: return pick_nb<1, true>(W, H, narrow);
    case 4: return pick_nb<2, false>(W, H, narrow);
    case 5: return pick_nb<2, true>(W, H, narrow);
    case 8: return pick_nb<4, false>(W, H, narrow);
    case 9: return pick_nb<4, true>(W, H, narrow);
    default: return {nullptr, 0, 0, 0};
  }
}

}  // namespace

bool stream_supported(int32_t W, int32_t H) { return pick(W, H, 1, false, false).f != nullptr; }

int stream_cta_traces(int32_t W, int32_t H, int32_t NB, bool burst, bool narrow) {
  return pick(W, H, NB, burst, narrow).traces;
}

int stream_ctas_per_sm(int32_t W, int32_t H, int32_t NB, bool burst, bool narrow) {
  Pick p = pick(W, H, NB, burst, narrow);
  if (!p.f) return 0;
  cudaFuncSetAttribute((const void*)p.f, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem);
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, (const void*)p.f, p.threads, p.smem) != cudaSuccess)
    return 0;
  return nb;
}

int launch_stream(cudaStream_t st, const void* tmap, const void* tmap_mul, int64_t N, int64_t T,
                  const DevPolicy* pol_dev, const int32_t* bundles_dev, int32_t nbund, int32_t NB,
                  int32_t W, int32_t H, const DevPlatform& plat, int64_t nseg, int64_t seg_len,
                  const StreamWork& wk, bool narrow, int* grid_out) {
  Pick p = pick(W, H, NB, plat.burst_on != 0, narrow);
  if (!p.f) return -1;
  cudaFuncSetAttribute((const void*)p.f, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem);
  const int32_t ngroups = (int32_t)((N + p.traces - 1) / p.traces);
  const int64_t grid = (int64_t)ngroups * nseg * nbund;
  if (grid_out) *grid_out = (int)grid;
  const CUtensorMap* m = reinterpret_cast<const CUtensorMap*>(tmap);
  const CUtensorMap* mm = reinterpret_cast<const CUtensorMap*>(tmap_mul);
  p.f<<<(unsigned)grid, p.threads, p.smem, st>>>(*m, *mm, N, T, pol_dev, bundles_dev, plat, nseg, seg_len,
                                                 ngroups, nbund, wk);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
