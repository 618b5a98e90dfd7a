// kernels_seq.cu -- the sequential-variant replay kernel (NEXT f3 / f4 and
// every per-interval level output).
//
// f3 (closed loop) makes Alg. 1 observe the delivered
// throughput min(x_t, B(l_t)), which depends on the decision that governed
// interval t, so the scan of one (trace, config) is a true recurrence; f4
// (gradual step) keeps p_t / hi_t pure but walks +-step ratios.  Both run
// here as one lane per (trace, config), sequential over T, in the paper's
// per-round order (Alg. 2 on the H previous events, the override of Alg. 3
// l.9-15, Alg. 1 on the window ends, event logging l.17/22/28/31, the step
// rule l.18-25) -- the same recurrence as ref_kernel.
//
// With ~4k recurrences on 148 SMs the time is the latency of ONE chain per
// step, so the kernel takes everything that does not depend on the
// decisions off that chain (warp specialisation, one CTA per 32 traces):
//   * 9 producer warps, round-robin over 32-step words: the samples x[t] and
//     the Alg. 1 lags x[t-W+1] of the word (64 independent loads per lane),
//     then the decision-independent predicates: the Alg. 1 outcomes as masks
//     -- for the binary closed loop all four outcomes (interval t at r_min /
//     r_max x lag interval at r_min / r_max), 8 bits per step -- and the
//     stretch / burst masks; the samples go to the slot for the accountant;
//   * 1 consumer warp, alone on its SMSP, runs only the recurrence,
//     integer-only and branch-free over a word: pick the outcome, the Alg. 2
//     count (incremental, vs the host-inverted k), the step rule, the event
//     history; it publishes the word's decision masks (or ratios);
//   * 1 accountant warp, alone on its SMSP too, turns them into model M (q only for the sparse
//     samples above the capacity at r_min), the counters (popc), the
//     decision words / ratios in HBM and the digest, and finalises.
// Slots move full -> done -> empty on mbarriers (16-slot ring); the three
// accountants release slots in word order (a token mbarrier each), so no
// parity wait can alias two phases.  The closed
// loop's record of which ratio governed interval t-W+1 is a 32/64-bit shift
// register (binary jumps) or a shared-memory byte ring (gradual); per-level
// model-M interval counts are run-length accumulated.  No local memory.
// Alg. 1 / Alg. 2 use the host-inverted thresholds of precompute.cpp
// (delta > d_inc <=> RN(delta / L) > tau_inc, s >= k <=> RN(s / H) >= t_hi),
// exact for every double; model M uses the literal quantiser q_literal of
// device_common.cuh.  ref_kernel (kernels_ref.cu) keeps the printed
// divisions and is the parity baseline this kernel is tested against.
#include "bitops.cuh"
#include "device_common.cuh"

#ifndef SEQ_ABLATE
#define SEQ_ABLATE 0  // developer timing experiments, a bit mask: 1 no accounting, 2 no producer math,
                      // 4 no chain, 8 no producer loads (constant samples)
#endif

namespace magus {
namespace {

constexpr int kLanes = 32;         // traces per CTA (one lane each)
constexpr int kWord = 32;          // steps per slot (= one decision word)
constexpr int kProducers = 9;
constexpr int kAccountants = 3;
// 16 warps, by SMSP (warp % 4): SMSP 0 = the consumer (warp 0) alone (4, 8,
// 12 idle); SMSP 1 = accountants 1, 5, 9 + producer 13; SMSPs 2 and 3 =
// producers 2, 3, 6, 7, 10, 11, 14, 15
constexpr int kThreads = 32 * 16;
constexpr int kAccFieldsSeq = 12;  // partial sums combined at the end (see the accountant)
constexpr int kRingL = 128;        // CLOSED && MULTI: ratios of the last 128 intervals
constexpr int kMaxLv = 128;

// slot layout (bytes)
constexpr int kOffX = 0;                              // float [32 steps][32 lanes] samples
constexpr int kOffCode = kOffX + 4 * kWord * kLanes;  // u32 [16][32] closed-binary transition codes (2 steps per word)
constexpr int kOffPM = kOffCode + 4 * 16 * kLanes;    // u32 [5][32] big, burst, inc, dec, big-at-max
constexpr int kOffCM = kOffPM + 4 * 5 * kLanes;       // u32 [5][32] dec, leff|change, event, hi masks, dec[t0-1]
constexpr int kOffLv = kOffCM + 4 * 5 * kLanes;       // u8 [32][32] MULTI ratios dec[t0+i]
constexpr int kOffL = kOffLv + kWord * kLanes;        // float [32][32] Alg. 1 lags (CLOSED && MULTI)
template <bool CLOSED, bool MULTI>
__host__ __device__ constexpr int slot_bytes() { return MULTI ? (CLOSED ? kOffL + 4 * kWord * kLanes : kOffL) : kOffLv; }
template <bool CLOSED, bool MULTI>
__host__ __device__ constexpr int n_slots() { return CLOSED && MULTI ? 12 : 16; }

__device__ __forceinline__ uint32_t sm_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mb_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mb_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mb_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
// every lane arrives (the slot barriers count 32 arrivals): each lane's own
// release orders its shared-memory writes of the word before the waiter's
// acquire (also what compute-sanitizer's racecheck can follow)
__device__ __forceinline__ void warp_arrive(uint32_t bar) {
  __syncwarp();
  mb_arrive(bar);
}

// The closed binary loop's transition code of one round (16 bits), from the
// four Alg. 1 differences d[a*2+b] (a = interval t at r_min, b = the lag
// interval t-W+1 at r_min).  Byte b (the lag's level) holds, for the level
// lm of interval t (= dec[t-1]): bit 4*lm = the next decision is min (lm = 0:
// -1 and not +1, Alg. 3 l.25; lm = 1: not +1, l.18 -- both unless hi, l.10),
// bit 4*lm + 1 = an event (+1 or -1 logged, l.17/22).  The consumer picks
// the byte by the lag's level and the nibble by lm with one LOP3.
__device__ __forceinline__ void code_bits(uint32_t& c, double d, double d_inc, double d_dec, uint32_t dnb,
                                          uint32_t ev, uint32_t stay) {
  // -1 (d < d_dec): set dnb (stay | ev for lm = 0, ev for lm = 1, whose stay
  // bit is preset); then +1 (d > d_inc): set ev, clear stay.  NaN: neither.
  asm("{\n.reg .pred p, q;\nsetp.lt.f64 p, %1, %2;\nsetp.gt.f64 q, %1, %3;\n@p or.b32 %0, %0, %4;\n"
      "@q lop3.b32 %0, %0, %5, %6, 0x54;\n}"
      : "+r"(c) : "d"(d), "d"(d_dec), "d"(d_inc), "r"(dnb), "r"(ev), "r"(stay));
}
// the 16-bit code of one round from the samples of intervals t and t-W+1
// (delivered = min(x, capacity) at each of the two levels, model M)
__device__ __forceinline__ uint32_t closed_code(float xt, float xl, double Bmin, double Bmax, bool capfree,
                                                double d_inc, double d_dec) {
  const double vt = (double)xt, vl = (double)xl;
  const double ytm = vt > Bmin ? Bmin : vt, ylm = vl > Bmin ? Bmin : vl;
  const double ytM = capfree ? vt : (vt > Bmax ? Bmax : vt), ylM = capfree ? vl : (vl > Bmax ? Bmax : vl);
  uint32_t c = 0x1010u;                                    // lm = 1: stays min unless +1
  code_bits(c, ytM - ylM, d_inc, d_dec, 0x0003u, 0x0002u, 0x0001u);   // a = 0, b = 0
  code_bits(c, ytM - ylm, d_inc, d_dec, 0x0300u, 0x0200u, 0x0100u);   // a = 0, b = 1
  code_bits(c, ytm - ylM, d_inc, d_dec, 0x0020u, 0x0020u, 0x0010u);   // a = 1, b = 0
  code_bits(c, ytm - ylm, d_inc, d_dec, 0x2000u, 0x2000u, 0x1000u);   // a = 1, b = 1
  return c;
}

template <uint32_t LUT>
__device__ __forceinline__ uint32_t lop3(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(d) : "r"(a), "r"(b), "r"(c), "n"(LUT));
  return d;
}

// delivered throughput of model M at capacity B (oracle `observed`)
__device__ __forceinline__ double delivered(float x, double B) {
  const double v = (double)x;
  return v > B ? B : v;
}

struct SeqArgs {
  const float* x;
  int64_t N, T, ld;
  const DevPolicy* pol;
  int32_t C;
  double bw_max, p_lo, p_span;
  magus_summary* summary;
  magus_base* base;
  uint32_t* dec;
  uint8_t* levels;
};

// CLOSED: f3 observation; MULTI: gradual walk with per-level accounting
// (variants 2, 3; the jump rule is the walk with step = r_max - r_min);
// otherwise the binary jump rule of the paper.
template <bool CLOSED, bool MULTI>
__global__ void __launch_bounds__(kThreads) seq_kernel(SeqArgs a, DevPlatform plat) {
  constexpr int kSlots = n_slots<CLOSED, MULTI>();
  constexpr int kSlotBytes = slot_bytes<CLOSED, MULTI>();
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ double s_B[kMaxLv], s_invB[kMaxLv];
  __shared__ __align__(8) uint64_t s_bar[3 * 16 + 4];    // full, done, empty, release tokens
  const int nlev = plat.r_max - plat.r_min + 1;
  for (int i = threadIdx.x; i < nlev; i += blockDim.x) {
    const int l = plat.r_min + i;
    const double B = (a.bw_max * (double)l) / (double)plat.r_max;  // capacity(), kernels_ref.cu
    s_B[i] = B;
    s_invB[i] = 1.0 / B;
  }
  const uint32_t bar0 = sm_addr(s_bar);
  if (threadIdx.x == 0)
    for (int i = 0; i < 3 * kSlots + kAccountants; ++i) mb_init(bar0 + 8u * i, i < 3 * kSlots ? 32u : 1u);
  __syncthreads();
  // mbarrier addresses (plain arithmetic: no closures on the wait paths)
#define full(s) (bar0 + 8u * (uint32_t)(s))
#define done(s) (bar0 + 8u * (uint32_t)(kSlots + (s)))
#define empty(s) (bar0 + 8u * (uint32_t)(2 * kSlots + (s)))
  // Release tokens: the accountant of word j releases its slot only after
  // word j - 1 was released (token tok[j % 3], armed by that release), so
  // slots return in word order.  A producer at word j has seen the release
  // of word j - 6 - 16 and hence of every earlier word: its parity wait on
  // empty(j % 16) is for the next phase, never two behind.
  // producer of word j >= 16: word j - 16 released (the accountants release
  // in word order, so this is the next phase of empty(j % 16))
  auto reclaim = [&](int64_t j) {
    mb_wait(empty((int)(j % kSlots)), (uint32_t)(((j / kSlots) + 1) & 1));
  };
#define tok(r) (bar0 + 8u * (uint32_t)(3 * kSlots + (int)((r) % kAccountants)))
  auto release = [&](int64_t j) {
    if (j > 0) {
      const int64_t ph = j / kAccountants - ((j % kAccountants) == 0 ? 1 : 0);  // arrivals from words j' = j - 1 (mod 3)
      mb_wait(tok(j), (uint32_t)(ph & 1));
    }
    warp_arrive(empty((int)(j % kSlots)));
    if ((threadIdx.x & 31) == 0) mb_arrive(tok(j + 1));
  };
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t gid = (int64_t)blockIdx.x * kLanes + lane;
  const bool active = gid < a.N * a.C;
  const int32_t c = active ? (int32_t)(gid / a.N) : 0;
  const int64_t n = active ? gid - (int64_t)c * a.N : 0;
  const DevPolicy P = a.pol[c];
  const int64_t T = a.T, W = P.W;
  const int64_t nwords = (T + kWord - 1) / kWord;
  const int lmin = plat.r_min, lmax = plat.r_max;
  const bool closed = CLOSED && (P.variant & MAGUS_VARIANT_CLOSED_LOOP) != 0;
  unsigned char* slots = smem;
  const uint32_t slots_a = sm_addr(smem);
  // per-lane word geometry
  auto word_cnt = [&](int64_t j) -> int {
    if (!active) return 0;
    const int64_t r = T - j * kWord;
    return r < kWord ? (int)r : kWord;
  };
  auto word_mdfs = [&](int64_t j, uint32_t live) -> uint32_t {  // MDFS rounds t >= W (reading R5)
    const int64_t t0 = j * kWord;
    const int r0 = W <= t0 ? 0 : (W - t0 >= kWord ? kWord : (int)(W - t0));
    return live & (r0 >= 32 ? 0u : (0xFFFFFFFFu << r0));
  };

  if (warp >= 4 && (warp & 3) == 0) return;   // keeps SMSP 0 for the consumer
  if ((warp & 3) >= 2 || warp == 13) {
    // =========================== producers ===============================
    const int p = warp == 13 ? 8 : (warp >> 2) * 2 + (warp & 1);   // warps 2,3,6,7,10,11,14,15,13 -> 0..8
    const float* xcol = a.x + n;
    // the closed loop is per config; an open-loop config observes through an
    // infinite capacity (delivered(x, inf) = x, NaN included)
    const double obs_min = closed ? plat.Bmin : (double)INFINITY;
    const double obs_max = closed ? plat.Bmax : (double)INFINITY;
    const bool bursts = plat.burst_mbs > 0.0;
    const float xthr = plat.xthr_min;  // x <= xthr: no stretch at any ratio (B_l >= B_min)
    // Each producer owns every 9th word.  Waiting on empty(j) needs word
    // j - kSlots < j to be accounted, which by induction on the word index
    // never waits on an unpublished word.
    const double d_inc = P.d_inc, d_dec = P.d_dec;
    const float xburst = bursts ? plat.xburst : INFINITY;   // x > xburst <=> (double)x > theta
    const int ld32 = (int)a.ld;                              // ld < 2^31 / 32 (checked on the host)
    // Alg. 1 outcome bits of one step: 8-bit closed-loop code or inc/dec
    auto eval = [&](float xt, float xl, uint32_t& cd, uint32_t& up, uint32_t& dn) {
      if constexpr (CLOSED) {
        // index a*2+b: a = interval t at r_min, b = lag interval at r_min;
        // bits 0-3 increase, bits 4-7 decrease
        const double ytm = delivered(xt, obs_min), ytM = delivered(xt, obs_max);
        const double ylm = delivered(xl, obs_min), ylM = delivered(xl, obs_max);
        const double d0 = ytM - ylM, d1 = ytM - ylm, d2 = ytm - ylM, d3 = ytm - ylm;
        cd = (uint32_t)(d0 > d_inc) | ((uint32_t)(d1 > d_inc) << 1) | ((uint32_t)(d2 > d_inc) << 2) |
             ((uint32_t)(d3 > d_inc) << 3) | ((uint32_t)(d0 < d_dec) << 4) | ((uint32_t)(d1 < d_dec) << 5) |
             ((uint32_t)(d2 < d_dec) << 6) | ((uint32_t)(d3 < d_dec) << 7);
      } else {
        const double D = (double)xt - (double)xl;
        up = D > d_inc;
        dn = D < d_dec;
      }
    };
    const float xthrM = plat.xthr_max;  // x <= xthrM: no stretch at r_max
    const float xobsM = closed ? plat.xobs_max : INFINITY;   // x > xobsM <=> (double)x > B_max
    // Half-word pipeline: the 32 loads of the next half (this word's second
    // half, or the first half of this producer's next word) are in flight
    // while the current half is evaluated.
    auto load_half = [&](int64_t jj, int h, float (&xv)[16], float (&lg)[16]) {
      if (jj >= nwords) return;
      const int64_t t0 = jj * kWord + 16 * h;
      const int cnt = word_cnt(jj);
      const uint32_t live = cnt == 32 ? 0xFFFFFFFFu : ((1u << cnt) - 1u);
      const uint32_t mdfs = word_mdfs(jj, live) >> (16 * h), lv = live >> (16 * h);
      const float* src = xcol + t0 * a.ld;
      const float* lsrc = xcol + (t0 - W + 1) * a.ld;
      if (SEQ_ABLATE & 8) {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
          xv[u] = (float)(lane + u);
          lg[u] = (float)(lane + 2 * u);
        }
        return;
      }
      if (__all_sync(0xFFFFFFFFu, (mdfs & 0xFFFFu) == 0xFFFFu)) {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
          xv[u] = __ldg(src + u * ld32);
          lg[u] = __ldg(lsrc + u * ld32);
        }
      } else {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
          xv[u] = ((lv >> u) & 1) ? __ldg(src + u * ld32) : 0.0f;
          lg[u] = ((mdfs >> u) & 1) ? __ldg(lsrc + u * ld32) : 0.0f;
        }
      }
    };
    float cx[16], cl[16];
    load_half(p, 0, cx, cl);
    for (int64_t j = p; j < nwords; j += kProducers) {
      const int s = (int)(j % kSlots);
      unsigned char* sl = slots + s * kSlotBytes;
      const int cnt = word_cnt(j);
      const uint32_t live = cnt == 32 ? 0xFFFFFFFFu : ((1u << cnt) - 1u);
      const uint32_t mdfs = word_mdfs(j, live);
      uint32_t big = 0, bigM = 0, brst = 0, inc = 0, dcr = 0;
      float* xs = reinterpret_cast<float*>(sl + kOffX) + lane;
      uint32_t* cwp = reinterpret_cast<uint32_t*>(sl + kOffCode) + lane;
#pragma unroll 1
      for (int h = 0; h < 2; ++h) {
        float nx[16], nl[16];
        if (h == 0) load_half(j, 1, nx, nl);
        else load_half(j + kProducers, 0, nx, nl);
        if (h == 0 && j >= kSlots) reclaim(j);
#pragma unroll
        for (int u = 0; u < 16; ++u) xs[(16 * h + u) * kLanes] = cx[u];
        if constexpr (CLOSED && MULTI) {
          float* ls = reinterpret_cast<float*>(sl + kOffL) + lane;
#pragma unroll
          for (int u = 0; u < 16; ++u) ls[(16 * h + u) * kLanes] = cl[u];
        }
        const uint32_t rd16 = (mdfs >> (16 * h)) & 0xFFFFu;
        uint32_t b16 = 0, bm16 = 0, r16 = 0, i16 = 0, d16 = 0, cw = 0;
        // no sample of the half above the capacity at r_max (the common case):
        // delivered = x there, two fewer selects per sample
        bool capfree = false;
        if constexpr (CLOSED && !MULTI) {
          float mx = cx[0];
#pragma unroll
          for (int u = 0; u < 16; ++u) mx = fmaxf(mx, fmaxf(cx[u], cl[u]));
          capfree = __all_sync(0xFFFFFFFFu, !(mx > xobsM));   // NaN: delivered = NaN either way
        }
#pragma unroll
        for (int u = 0; u < ((SEQ_ABLATE & 2) ? 0 : 16); ++u) {
          const float xt = cx[u];
          or_if_gt(b16, xt, xthr, 1u << u);
          or_if_gt(bm16, xt, xthrM, 1u << u);
          or_if_gt(r16, xt, xburst, 1u << u);
          if constexpr (CLOSED && !MULTI) {
            // every round (the consumer reads the codes of MDFS rounds only)
            cw |= closed_code(xt, cl[u], obs_min, obs_max, capfree, d_inc, d_dec) << (16 * (u & 1));
            if (u & 1) {
              cwp[(8 * h + (u >> 1)) * kLanes] = cw;
              cw = 0;
            }
          } else if (!(CLOSED && MULTI) && ((rd16 >> u) & 1)) {
            uint32_t cd = 0, up = 0, dn = 0;
            eval(xt, cl[u], cd, up, dn);
            i16 |= up << u;
            d16 |= dn << u;
          }
        }
        big |= b16 << (16 * h);
        bigM |= bm16 << (16 * h);
        brst |= r16 << (16 * h);
        inc |= i16 << (16 * h);
        dcr |= d16 << (16 * h);
#pragma unroll
        for (int u = 0; u < 16; ++u) {
          cx[u] = nx[u];
          cl[u] = nl[u];
        }
      }
      big &= live;
      bigM &= live;
      brst &= live;
      uint32_t* pm = reinterpret_cast<uint32_t*>(sl + kOffPM) + lane;
      pm[0] = big;
      pm[kLanes] = brst;
      pm[2 * kLanes] = inc;
      pm[3 * kLanes] = dcr;
      pm[4 * kLanes] = bigM;
      warp_arrive(full(s));
    }
    return;
  }

  if (warp == 0) {
    // ============================ consumer ===============================
    const uint64_t hmask = P.H >= 64 ? ~0ULL : ((1ULL << P.H) - 1ULL);
    const int hsh = P.H - 1;
    const int k = P.k;
    const int step = (P.variant & MAGUS_VARIANT_GRADUAL) ? P.step : (lmax - lmin);
    const int wsh = (int)(W - 1) & 63;
    // branch-free 32-bit words when every lane has W, H <= 32 and the word is
    // all MDFS rounds (everything but a trace's first and last word)
    const bool narrow = __all_sync(0xFFFFFFFFu, !active || (W <= 32 && P.H <= 32 && (!CLOSED || (W >= 3 && P.H >= 2))));
    const uint32_t hmask32 = (uint32_t)hmask;
    uint64_t hist = 0;               // uncore_tune_ls: H zeros (P@24182); bit j = round t-1-j
    int s_cnt = 0;                   // popc(hist)
    int lvl = lmax;                  // uncore_freq starts at max (P@23755)
    uint32_t lm = 0;                 // binary form: 1 = at r_min
    uint64_t lvb = 0;                // CLOSED binary: bit j = [interval t-j ran at r_min]
    uint8_t* lvr = slots + kSlots * kSlotBytes;   // CLOSED && MULTI ratio ring [kRingL][32]
    for (int64_t j = 0; j < nwords; ++j) {
      const int s = (int)(j % kSlots);
      mb_wait(full(s), (uint32_t)((j / kSlots) & 1));
      unsigned char* sl = slots + s * kSlotBytes;
      const int cnt = word_cnt(j);
      const uint32_t live = cnt == 32 ? 0xFFFFFFFFu : ((1u << cnt) - 1u);
      const uint32_t mdfs = word_mdfs(j, live);
      const bool fast = narrow && __all_sync(0xFFFFFFFFu, mdfs == 0xFFFFFFFFu);
      if (SEQ_ABLATE & 4) { warp_arrive(done(s)); continue; }
      const uint32_t* pm = reinterpret_cast<const uint32_t*>(sl + kOffPM) + lane;
      const uint32_t inc = pm[2 * kLanes], dcr = pm[3 * kLanes];
      uint32_t decm = 0, m1 = 0, evm = 0, him = 0;   // m1: binary leff mask / MULTI change mask
      const int lvl_in = lvl;                         // dec[t0-1] (MULTI)
      if constexpr (!MULTI) {
        if (fast) {
          // 8 groups of 4 steps (a small loop body stays in the instruction
          // cache); masks fill from the top by funnel shifts, so after the 32
          // steps bit i is step i
          const uint32_t* cwp = reinterpret_cast<const uint32_t*>(sl + kOffCode) + lane;
          uint32_t h = (uint32_t)hist, lb = (uint32_t)lvb, iv = inc, dv = dcr;
          if constexpr (CLOSED) {
            // The chain of a round is two LOP3: the code nibble picked by the
            // level of interval t (LM, all ones at r_min) and the override
            // (lt = !hi, Alg. 2 as the sign of D = s - k).  Everything else
            // accumulates by multiply-adds (the FMA pipe, next to the ALU
            // pipe's LOP3 / shifts), in reversed bit order (bit 31 = round 0).
            // lag interval of the NEXT round = bit W-3 of lb before this
            // round's push (W >= 3), the outgoing event of the next round =
            // bit H-2 of h before the push (H >= 2): both read from registers
            // this round's decision does not write (off the chain)
            const uint32_t wsh2 = (uint32_t)(W - 3), hsh2 = (uint32_t)(hsh - 1);
            uint32_t lag = (lb >> (wsh2 + 1)) & 1u, out = (h >> hsh) & 1u;
            uint32_t LM = 0u - lm;
            int D = s_cnt - k;                          // hi <=> s >= k <=> D >= 0
            uint32_t lt = (uint32_t)D >> 31;
            uint32_t dacc = 0, eacc = 0, lacc = 0;
            const uint32_t lm0 = lm;
            uint32_t wa = cwp[0], wb = cwp[kLanes];
#pragma unroll 1
            for (int g = 0; g < kWord / 4; ++g) {
              const uint32_t w0 = wa, w1 = wb;
              if (g < kWord / 4 - 1) {
                wa = cwp[(2 * g + 2) * kLanes];
                wb = cwp[(2 * g + 3) * kLanes];
              }
#pragma unroll
              for (int u = 0; u < 4; ++u) {
                const uint32_t w = u < 2 ? w0 : w1;
                const uint32_t P = w >> (16 * (u & 1) + 8 * lag);     // byte of the lag's level
                const uint32_t V = lop3<0xD8>(P, P >> 4, LM);           // nibble of interval t's level
                const uint32_t nlm = lop3<0x80>(V, lt, 1u);             // l.10 override, else l.18 / l.25 / hold
                const uint32_t e = (V >> 1) & 1u;                       // l.17 / l.22 event
                D += (int)e - (int)out;
                lag = (lb >> wsh2) & 1u;
                out = (h >> hsh2) & 1u;
                lacc = lacc * 2u + lt;
                lt = (uint32_t)D >> 31;
                lb = lb * 2u + (LM & 1u);
                h = h * 2u + e;
                eacc = eacc * 2u + e;
                LM = 0u - nlm;
                dacc = dacc * 2u + nlm;
              }
            }
            decm = __brev(dacc);
            evm = __brev(eacc);
            him = ~__brev(lacc);
            m1 = (decm << 1) | lm0;                     // interval t runs at dec[t-1] (reading R6)
            lm = LM & 1u;
            s_cnt = D + k;
            hist = h & hmask32;
            lvb = lb;
          } else {
#pragma unroll 1
          for (int g = 0; g < kWord / 4; ++g) {
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              m1 = __funnelshift_r(m1, lm, 1);      // interval t runs at dec[t-1] (reading R6)
              uint32_t up, dn, e;
              {
                up = iv & 1u;
                dn = dv & 1u;
                iv >>= 1;
                dv >>= 1;
                e = up | dn;
              }
              const uint32_t hi = s_cnt >= k;                   // Alg. 2
              // l.9-15 override, else l.18 (+1 -> max) / l.25 (-1 -> min) / hold
              lm = (hi | up) ? 0u : (dn | lm);
              him = __funnelshift_r(him, hi, 1);
              evm = __funnelshift_r(evm, e, 1);
              const uint32_t out = (h >> hsh) & 1u;
              h = ((h << 1) | e) & hmask32;
              s_cnt += (int)e - (int)out;
              decm = __funnelshift_r(decm, lm, 1);
            }
          }
          hist = h;
          }
        } else {
#pragma unroll 1
          for (int i = 0; i < kWord; ++i) {
            if ((live >> i) & 1) {
              m1 |= lm << i;
              if constexpr (CLOSED) lvb = (lvb << 1) | lm;
              if ((mdfs >> i) & 1) {
                uint32_t e, up, dn;
                const uint32_t hi = s_cnt >= k;
                if constexpr (CLOSED) {   // closed_code: byte by the lag's level, nibble by lm
                  const uint32_t lag = (uint32_t)((lvb >> wsh) & 1ULL);
                  const uint32_t cw = reinterpret_cast<const uint32_t*>(sl + kOffCode)[(i >> 1) * kLanes + lane];
                  const uint32_t V = (cw >> (16 * (i & 1) + 8 * lag)) >> (4 * lm);
                  e = (V >> 1) & 1u;
                  lm = hi ? 0u : (V & 1u);
                } else {
                  up = (inc >> i) & 1u;
                  dn = (dcr >> i) & 1u;
                  e = up | dn;
                  lm = (hi | up) ? 0u : (dn | lm);
                }
                him |= hi << i;
                const int out = (int)((hist >> hsh) & 1ULL);
                hist = ((hist << 1) | e) & hmask;
                s_cnt += (int)e - out;
                evm |= e << i;
              }
              decm |= lm << i;
            }
          }
        }
      } else {
        uint8_t* lvw = sl + kOffLv + lane;
        if (!CLOSED && fast) {
          uint32_t h = (uint32_t)hist, iv = inc, dv = dcr;
#pragma unroll 1
          for (int g = 0; g < kWord / 4; ++g) {
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              const uint32_t up = iv & 1u, dn = dv & 1u, e = up | dn;
              iv >>= 1;
              dv >>= 1;
              const uint32_t hi = s_cnt >= k;                   // Alg. 2
              const int upl = min(lvl + step, lmax), dnl = max(lvl - step, lmin);
              const int nl = hi ? lmax : (up ? upl : (dn ? dnl : lvl));   // f4: +-step, hi -> max
              him = __funnelshift_r(him, hi, 1);
              evm = __funnelshift_r(evm, e, 1);
              m1 = __funnelshift_r(m1, (uint32_t)(nl != lvl), 1);
              lvl = nl;
              const uint32_t out = (h >> hsh) & 1u;
              h = ((h << 1) | e) & hmask32;
              s_cnt += (int)e - (int)out;
              lvw[(4 * g + u) * kLanes] = (uint8_t)lvl;
              decm = __funnelshift_r(decm, (uint32_t)(lvl == lmin), 1);
            }
          }
          hist = h;
        } else {
          const float* xs = reinterpret_cast<const float*>(sl + kOffX) + lane;
          const float* ls = reinterpret_cast<const float*>(sl + kOffL) + lane;
#pragma unroll 1
          for (int i = 0; i < kWord; ++i) {
            if ((live >> i) & 1) {
              const int64_t t = j * kWord + i;
              const int prev = lvl;
              if constexpr (CLOSED) lvr[(int)(t & (kRingL - 1)) * kLanes + lane] = (uint8_t)lvl;
              if ((mdfs >> i) & 1) {
                uint32_t up, dn;
                if constexpr (CLOSED) {  // f3 + f4: capacities of 15+ ratios, read on the chain
                  double yt = (double)xs[i * kLanes], yl = (double)ls[i * kLanes];
                  if (closed) {
                    yt = delivered(xs[i * kLanes], s_B[lvl - lmin]);
                    yl = delivered(ls[i * kLanes],
                                   s_B[lvr[(int)((t - W + 1) & (kRingL - 1)) * kLanes + lane] - lmin]);
                  }
                  const double D = yt - yl;
                  up = D > P.d_inc;
                  dn = D < P.d_dec;
                } else {
                  up = (inc >> i) & 1u;
                  dn = (dcr >> i) & 1u;
                }
                const uint32_t e = up | dn;
                const uint32_t hi = s_cnt >= k;                 // Alg. 2
                if (hi) lvl = lmax;
                else if (up) lvl = min(lvl + step, lmax);       // f4 (+step), l.18 for the jump
                else if (dn) lvl = max(lvl - step, lmin);       // f4 (-step), l.25 for the jump
                him |= hi << i;
                evm |= e << i;
                const int out = (int)((hist >> hsh) & 1ULL);
                hist = ((hist << 1) | e) & hmask;
                s_cnt += (int)e - out;
              }
              m1 |= (uint32_t)(lvl != prev) << i;
              lvw[i * kLanes] = (uint8_t)lvl;
              decm |= (uint32_t)(lvl == lmin) << i;
            }
          }
        }
      }
      uint32_t* cm = reinterpret_cast<uint32_t*>(sl + kOffCM) + lane;
      cm[4 * kLanes] = (uint32_t)lvl_in;
      cm[0] = decm;
      cm[kLanes] = m1;
      cm[2 * kLanes] = evm;
      cm[3 * kLanes] = him;
      warp_arrive(done(s));
    }
    return;
  }

  // ============================= accountants ============================
  // kAccountants warps take the words round-robin; every quantity is an
  // integer sum over words (per-level model-M rows private to each
  // accountant), combined by accountant 0 at the end.
  const int acc_id = warp >> 2;      // warps 1, 5, 9 -> 0, 1, 2
  const bool bursts = plat.burst_mbs > 0.0;
  const int burst_at_max = plat.Bmax > plat.burst_mbs, burst_at_min = plat.Bmin > plat.burst_mbs;
  const double invB_min = plat.invB_min, invB_max = plat.invB_max;
  unsigned char* tail = slots + kSlots * kSlotBytes + (CLOSED && MULTI ? kRingL * kLanes : 0);
  // MULTI: qacc [kAccountants][nlev][32] u64, nacc [kAccountants][nlev][32] u32
  unsigned long long* qacc0 = reinterpret_cast<unsigned long long*>(tail);
  uint32_t* nacc0 = reinterpret_cast<uint32_t*>(qacc0 + (MULTI ? kAccountants * nlev * kLanes : 0));
  unsigned long long* part = reinterpret_cast<unsigned long long*>(nacc0 + (MULTI ? kAccountants * nlev * kLanes : 0));
  // part: [kAccountants - 1][kAccFieldsSeq][32] partial sums of accountants 1..
  unsigned long long* qacc = qacc0 + (size_t)acc_id * nlev * kLanes;
  uint32_t* nacc = nacc0 + (size_t)acc_id * nlev * kLanes;
  if constexpr (MULTI) {
    for (int i = 0; i < nlev; ++i) {
      qacc[i * kLanes + lane] = 0;
      nacc[i * kLanes + lane] = 0;
    }
  }
  asm volatile("bar.sync 1, %0;" ::"n"(32 * kAccountants) : "memory");
  // q of model M without the F2I: RN(x / B) > 1 first, then
  // the exact power-of-two-scaled form of device_common.cuh
  auto q_at = [](float x, double invB) -> uint64_t {
    return ((double)x * invB > 1.0) ? q_scaled(x, invB * kQScale) : 0ull;
  };
  int32_t events = 0, hi_rounds = 0, msr = 0, changes = 0, n_min_dec = 0, n_min_int = 0;
  uint64_t q_min = 0, q_max = 0, q_base = 0, digest = 0;
  int32_t b_base = 0, b_magus = 0;
  for (int64_t j = acc_id; j < nwords; j += kAccountants) {
    const int s = (int)(j % kSlots);
    mb_wait(done(s), (uint32_t)((j / kSlots) & 1));
    if (SEQ_ABLATE & 1) { release(j); continue; }
    const unsigned char* sl = slots + s * kSlotBytes;
    const int64_t t0 = j * kWord;
    const int cnt = word_cnt(j);
    const uint32_t live = cnt == 32 ? 0xFFFFFFFFu : ((1u << cnt) - 1u);
    const uint32_t* pm = reinterpret_cast<const uint32_t*>(sl + kOffPM) + lane;
    const uint32_t* cm = reinterpret_cast<const uint32_t*>(sl + kOffCM) + lane;
    const float* xs = reinterpret_cast<const float*>(sl + kOffX) + lane;
    const uint32_t big = pm[0] & live, brst = pm[kLanes] & live, bigM = pm[4 * kLanes] & live;
    const uint32_t decm = cm[0] & live, m1 = cm[kLanes] & live, evm = cm[2 * kLanes], him = cm[3 * kLanes];
    events += __popc(evm);
    hi_rounds += __popc(him);
    msr += __popc(evm | him);        // tune calls: every hi round + every non-hi event
    n_min_dec += __popc(decm);
    if (active) {
      if (a.dec) a.dec[((int64_t)c * nwords + j) * a.N + n] = decm;
      digest += (uint64_t)decm * digest_mul(j);
    }
    if constexpr (MULTI) {
      // g_i, the ratio governing interval t0+i, is dec[t0+i-1]: the word's
      // incoming ratio for i = 0, then the consumer's ratios; it changes
      // after step i iff bit i of the change mask m1 is set
      const uint8_t* lvw = sl + kOffLv + lane;
      const int lin = (int)cm[4 * kLanes];
      changes += __popc(t0 == 0 ? (m1 & ~1u) : m1);     // t >= 1 only
      if (active) {
        uint32_t cb = m1;
        int pos = 0, g = lin;
        while (cb) {                   // runs of g (one per ratio change)
          const int i = __ffs(cb) - 1;
          cb &= cb - 1;
          nacc[(g - lmin) * kLanes + lane] += (uint32_t)(i + 1 - pos);
          g = lvw[i * kLanes];
          pos = i + 1;
        }
        if (cnt > pos) nacc[(g - lmin) * kLanes + lane] += (uint32_t)(cnt - pos);
        uint32_t bm = big | brst;
        while (bm) {                   // samples above the capacity at r_min / bursts (sparse)
          const int i = __ffs(bm) - 1;
          bm &= bm - 1;
          const int gi = i == 0 ? lin : (int)lvw[(i - 1) * kLanes];
          const float xt = xs[i * kLanes];
          if ((big >> i) & 1) {
            const uint64_t qb = ((bigM >> i) & 1) ? q_scaled(xt, invB_max * kQScale) : 0ull;
            q_base += qb;
            const uint64_t q = gi == lmax ? qb : q_at(xt, s_invB[gi - lmin]);
            qacc[(gi - lmin) * kLanes + lane] += q;
          }
          if ((brst >> i) & 1) {       // delivered min(x, B_l) > theta
            b_base += burst_at_max;
            b_magus += s_B[gi - lmin] > plat.burst_mbs;
          }
        }
        if (a.levels) {
          uint8_t* lo = a.levels + ((int64_t)c * T + t0) * a.N + n;
          for (int i = 0; i < cnt; ++i) lo[(int64_t)i * a.N] = lvw[i * kLanes];
        }
      }
    } else {
      uint32_t ch = decm ^ m1;       // changes at t >= 1: dec[t] != dec[t-1] (m1 = leff mask)
      if (t0 == 0) ch &= ~1u;
      changes += __popc(ch);
      if (a.levels && active) {
        uint8_t* lo = a.levels + ((int64_t)c * T + t0) * a.N + n;
        for (int i = 0; i < cnt; ++i) lo[(int64_t)i * a.N] = (uint8_t)(((decm >> i) & 1) ? lmin : lmax);
      }
      n_min_int += __popc(m1);
      uint32_t bm = big;
      while (bm) {                   // samples above the capacity at r_min (sparse)
        const int i = __ffs(bm) - 1;
        bm &= bm - 1;
        const float xt = xs[i * kLanes];
        const uint64_t qb = ((bigM >> i) & 1) ? q_scaled(xt, invB_max * kQScale) : 0ull;
        q_base += qb;
        if ((m1 >> i) & 1) q_min += q_scaled(xt, invB_min * kQScale);   // big: x > xthr_min
        else q_max += qb;
      }
      if (bursts) {
        b_base += burst_at_max * __popc(brst);
        b_magus += burst_at_min * __popc(brst & m1) + burst_at_max * __popc(brst & ~m1);
      }
    }
    release(j);
  }
  // combine the partial sums (integer, order-free) in accountant 0
  if (acc_id > 0) {
    unsigned long long* pp = part + (size_t)(acc_id - 1) * kAccFieldsSeq * kLanes + lane;
    const unsigned long long v[kAccFieldsSeq] = {
        (unsigned long long)events, (unsigned long long)hi_rounds, (unsigned long long)msr,
        (unsigned long long)changes, (unsigned long long)n_min_dec, (unsigned long long)n_min_int,
        q_min, q_max, q_base, digest, (unsigned long long)b_base, (unsigned long long)b_magus};
#pragma unroll
    for (int f = 0; f < kAccFieldsSeq; ++f) pp[f * kLanes] = v[f];
  }
  asm volatile("bar.sync 1, %0;" ::"n"(32 * kAccountants) : "memory");
  if (acc_id > 0 || !active) return;
  for (int w = 0; w < kAccountants - 1; ++w) {
    const unsigned long long* pp = part + (size_t)w * kAccFieldsSeq * kLanes + lane;
    events += (int32_t)pp[0];
    hi_rounds += (int32_t)pp[kLanes];
    msr += (int32_t)pp[2 * kLanes];
    changes += (int32_t)pp[3 * kLanes];
    n_min_dec += (int32_t)pp[4 * kLanes];
    n_min_int += (int32_t)pp[5 * kLanes];
    q_min += pp[6 * kLanes];
    q_max += pp[7 * kLanes];
    q_base += pp[8 * kLanes];
    digest += pp[9 * kLanes];
    b_base += (int32_t)pp[10 * kLanes];
    b_magus += (int32_t)pp[11 * kLanes];
  }
  magus_summary* so = a.summary ? a.summary + (int64_t)c * a.N + n : nullptr;
  magus_base* bo = (a.base && c == 0) ? a.base + n : nullptr;
  if constexpr (MULTI) {   // per-level rows: sum over the accountants (integers)
    for (int w = 1; w < kAccountants; ++w)
      for (int i = 0; i < nlev; ++i) {
        qacc0[i * kLanes + lane] += qacc0[((size_t)w * nlev + i) * kLanes + lane];
        nacc0[i * kLanes + lane] += nacc0[((size_t)w * nlev + i) * kLanes + lane];
      }
    n_min_int = (int32_t)nacc0[lane];
    q_min = qacc0[lane];
    for (int i = 1; i < nlev; ++i) q_max += qacc0[i * kLanes + lane];
  }
  finalize_summary(plat, T, events, hi_rounds, msr, changes, n_min_dec, n_min_int, q_min, q_max, q_base,
                   digest, b_base, b_magus, so, bo);
  if constexpr (MULTI) {
    if (so) {  // general model M: energy = sum over the ratios, ascending
      double energy = 0.0;
      for (int i = 0; i < nlev; ++i) {
        const int l = lmin + i;
        const double Pl = a.p_lo + (a.p_span * (double)(l - lmin)) / (double)(lmax - lmin);
        energy = energy + Pl * (plat.dt * (double)nacc0[i * kLanes + lane] +
                                plat.cQ * (double)qacc0[i * kLanes + lane]);
      }
      so->energy_j = energy + plat.e_sw * (double)changes;
    }
  }
}

#undef full
#undef done
#undef empty
#undef tok

template <bool CLOSED, bool MULTI>
size_t smem_bytes(const DevPlatform& plat) {
  const int nlev = plat.r_max - plat.r_min + 1;
  size_t smem = (size_t)n_slots<CLOSED, MULTI>() * slot_bytes<CLOSED, MULTI>();
  if (CLOSED && MULTI) smem += (size_t)kRingL * kLanes;
  if (MULTI) smem += (size_t)kAccountants * nlev * kLanes * (sizeof(uint64_t) + sizeof(uint32_t));
  smem += (size_t)(kAccountants - 1) * kAccFieldsSeq * kLanes * sizeof(uint64_t);
  return smem;
}
constexpr size_t kSmemLimit = 227 * 1024;

template <bool CLOSED, bool MULTI>
int launch_one(cudaStream_t s, const SeqArgs& a, const DevPlatform& plat) {
  const size_t smem = smem_bytes<CLOSED, MULTI>(plat);
  auto k = seq_kernel<CLOSED, MULTI>;
  if (smem > 48 * 1024 &&
      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return -1;
  const int64_t total = a.N * a.C;
  const unsigned blocks = (unsigned)((total + kLanes - 1) / kLanes);
  k<<<blocks, kThreads, smem, s>>>(a, plat);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace

bool seq_fits(const DevPlatform& plat, bool closed, bool multi) {
  const size_t b = closed ? (multi ? smem_bytes<true, true>(plat) : smem_bytes<true, false>(plat))
                          : (multi ? smem_bytes<false, true>(plat) : smem_bytes<false, false>(plat));
  return b <= kSmemLimit;
}

bool seq_supported(const magus_policy& p) {
  if (!(p.variant & MAGUS_VARIANT_CLOSED_LOOP)) return true;
  // the closed loop reads the ratio that governed interval t-W+1 from a
  // 64-bit shift register (binary) or a 128-step ring (gradual)
  return (p.variant & MAGUS_VARIANT_GRADUAL) ? p.window <= kRingL : p.window <= 64;
}

int launch_seq(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
               const DevPolicy* pol_dev, int32_t C, const DevPlatform& plat, double bw_max,
               double p_lo, double p_span, bool closed, bool multi, magus_summary* out_summary,
               magus_base* out_base, uint32_t* out_dec, uint8_t* out_levels) {
  SeqArgs a{x, N, T, ld, pol_dev, C, bw_max, p_lo, p_span, out_summary, out_base, out_dec, out_levels};
  if (closed) return multi ? launch_one<true, true>(s, a, plat) : launch_one<true, false>(s, a, plat);
  return multi ? launch_one<false, true>(s, a, plat) : launch_one<false, false>(s, a, plat);
}

}  // namespace magus
