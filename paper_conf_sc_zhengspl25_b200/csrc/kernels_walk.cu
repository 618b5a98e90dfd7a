// kernels_walk.cu -- the time-segmented replay of the open-loop variants:
// NEXT f4 (gradual +-step rule, P@35554) and the paper's jump rule whenever
// per-interval levels are requested.
//
// Why it segments exactly.  In the open loop, Alg. 1's outcome p_t and
// Alg. 2's hi_t are pure functions of the trace (closed form);
// only the level walk is sequential, and every round applies to the level
// one map of the form
//     l -> min(max(l + d, a), b)          (r_min <= a <= b <= r_max)
// -- hold (d = 0, a = r_min, b = r_max), step up (Alg. 3 l.18 with the f4
// step: min(l + s, r_max)), step down (l.23-25: max(l - s, r_min)), the
// override to max (l.10: a = b = r_max).  These clamp-shift maps are closed
// under composition: applying up-step s to (d, a, b) gives
// (d + s, min(a + s, r_max), min(b + s, r_max)), down-step symmetrically,
// and on the domain [r_min, r_max] every d beyond +-(r_max - r_min) acts like
// the bound, so d saturates there.  A segment's whole effect on the carry is
// therefore one packed 32-bit map.
//
// Three launches (plus the totals kernel of kernels_post.cu):
//   walk_map_kernel     one thread per (trace, segment, config): rebuild the
//                       event history of the H rounds before the segment
//                       (the halo), compose the segment's map; segment-0
//                       threads also zero the (config, trace) accumulators;
//   walk_replay_kernel  same threads: carry-in = the composition of the maps
//                       of all earlier segments applied to r_max (interval 0
//                       runs at max, P@23755), then the rounds of the
//                       segment in the paper's order with model-M accounting
//                       at the level that governs each interval (dec[t-1],
//                       reading R6); integer segment sums go into the
//                       accumulators with 64-bit atomics (exact, any order);
//                       per-level (intervals, stretch) pairs are
//                       run-length accumulated and flushed on level changes;
//   walk_final_kernel   one thread per (trace, config): model M (the general
//                       per-level form of DESIGN.md 4.3, the fp64 order of
//                       kernels_ref.cu) into the summaries.
// Compared with the latency-optimised seq_kernel (one chain per trace), the
// segments give ~10^5 independent chains, so the walk is throughput-bound;
// the price is reading the traces twice.
#include <algorithm>

#include "bitops.cuh"
#include "device_common.cuh"

namespace magus {
namespace {

constexpr int kWalkThreads = 128;
constexpr int kWalkChunk = 16;   // samples (and lags) loaded ahead of the chain
constexpr int kWalkMaxLv = 128;  // ratios 1..127

enum { WF_EV, WF_HI, WF_MSR, WF_CH, WF_MDEC, WF_QBASE, WF_DIG, WF_BB, WF_BM, kWalkFields };

struct WalkArgs {
  const float* x;
  int64_t N, ld;
  int32_t T, nw;                 // intervals (<= 2^24), 32-step words
  const DevPolicy* pol;
  int32_t C, c0;                 // all configs; first config of this launch (grid z = batch)
  int32_t nseg, seg_len;         // seg_len % 32 == 0
  uint32_t* map;                 // [batch][nseg][N] packed segment maps
  uint32_t* mask;                // [batch][3][nw][N] Alg. 1 +1 / -1 and Alg. 2 hi bits per round
  unsigned long long* acc;       // [C][kWalkFields][N]
  unsigned int* lvn;             // [C][nlev][N] intervals per level
  unsigned long long* lvq;       // [C][nlev][N] stretch q per level
  magus_summary* summary;        // [C][N] (required)
  magus_base* base;              // [N] or NULL
  uint32_t* dec;                 // [C][nw][N] or NULL
  uint8_t* levels;               // [C][T][N] or NULL
  double p_lo, p_span;
};

// per-level constants, host-computed (the same formulas as kernels_ref.cu);
// passed by value (1.7 KB of kernel parameters)
struct WalkLevels {
  double invB[kWalkMaxLv];       // 1 / B_l
  float xthr[kWalkMaxLv];        // x > xthr[l] <=> RN(x * invB[l]) > 1
  uint8_t bkeep[kWalkMaxLv];     // B_l > theta (a burst stays a burst at l)
};

__device__ __forceinline__ uint32_t map_pack(int d, int a, int b) {
  return (uint32_t)(uint8_t)(int8_t)d | ((uint32_t)a << 8) | ((uint32_t)b << 16);
}
__device__ __forceinline__ int map_apply(uint32_t m, int l) {
  const int d = (int)(int8_t)(m & 0xFFu), a = (int)((m >> 8) & 0xFFu), b = (int)((m >> 16) & 0xFFu);
  return min(max(l + d, a), b);
}

// uncore_tune_ls at the start of round t0: the events of rounds
// max(W, t0 - H) .. t0 - 1 (bit j = round t0 - 1 - j); Alg. 1 with the
// host-inverted thresholds (delta > d_inc <=> RN(delta / L) > tau_inc; NaN:
// neither, reading R9)
__device__ __forceinline__ uint64_t history_at(const WalkArgs& a, const DevPolicy& P, int64_t n, int32_t t0) {
  uint64_t hist = 0;
  for (int32_t t = max(P.W, t0 - P.H); t < t0; ++t) {
    const double D = (double)a.x[(int64_t)t * a.ld + n] - (double)a.x[(int64_t)(t - P.W + 1) * a.ld + n];
    hist = (hist << 1) | (uint64_t)(D > P.d_inc || D < P.d_dec);
  }
  return hist;
}

// K samples x[t0 + i rows] (32-bit row offsets: ld < 2^26, checked
// by the dispatcher, keeps every address one IMAD from the base)
template <int K>
__device__ __forceinline__ void load_rows(const float* __restrict__ p, int ld32, float (&v)[K]) {
#pragma unroll
  for (int i = 0; i < K; ++i) v[i] = __ldg(p + i * ld32);
}

// Pass 1: per (trace, segment, config) thread, the rounds of the segment in
// the paper's order -- Alg. 2 on the H previous events (s >= k <=> RN(s/H)
// >= t_hi), Alg. 1 (host-inverted thresholds), event logging -- recorded as
// three bit masks per 32-step word, and composed into the segment's map.
// WT > 0: every config of the launch has W = WT; a full word loads its 32
// samples once and takes the Alg. 1 lags x[t-W+1] from a register window
// (the word's own samples and the previous word's last W-1, each widened to
// fp64 once), instead of a second row load and conversion per sample.
template <typename HT, int WT>
__global__ void __launch_bounds__(kWalkThreads, 5) walk_map_kernel(WalkArgs a, int32_t lmin, int32_t lmax, int32_t nlev) {
  const int64_t n = (int64_t)blockIdx.x * kWalkThreads + threadIdx.x;
  const int32_t s = blockIdx.y, cl = blockIdx.z, c = a.c0 + cl;
  if (n >= a.N) return;
  if (s == 0) {  // fresh accumulators for this replay
    for (int f = 0; f < kWalkFields; ++f) a.acc[((int64_t)c * kWalkFields + f) * a.N + n] = 0ull;
    for (int i = 0; i < nlev; ++i) {
      a.lvn[((int64_t)c * nlev + i) * a.N + n] = 0u;
      a.lvq[((int64_t)c * nlev + i) * a.N + n] = 0ull;
    }
  }
  const DevPolicy P = a.pol[c];
  const HT hmask = P.H >= (int)(8 * sizeof(HT)) ? (HT)~(HT)0 : (HT)(((HT)1 << P.H) - 1);
  const int32_t t0 = s * a.seg_len, t1 = min(a.T, t0 + a.seg_len);
  const int K = lmax - lmin;
  const int step = (P.variant & MAGUS_VARIANT_GRADUAL) ? P.step : K;
  HT hist = (HT)history_at(a, P, n, max(t0, P.W)) & hmask;
  // H <= 32: Alg. 2 bit-parallel per 32-round word (the events of the H
  // rounds before each position, counted by a carry-save tree / ripple
  // counter and compared with k), instead of a popcount per round
  constexpr bool kBits = sizeof(HT) == 4;
  uint32_t Eprev = kBits ? __brev((uint32_t)hist) : 0u;  // bit i = round t0 - 32 + i
  uint32_t km[6];
#pragma unroll
  for (int j = 0; j < 6; ++j) km[j] = ((P.k >> j) & 1) ? ~0u : 0u;
  int d = 0, lo = lmin, hi = lmax;  // identity (the clamp-shift map l -> min(max(l + d, lo), hi))
  uint32_t* mk = a.mask + (int64_t)cl * 3 * a.nw * a.N + n;
  const int ld32 = (int)a.ld;
  uint32_t inc = 0, dcr = 0, hw = 0;
  // one round: Alg. 2, Alg. 1, the event log, and the composition with this
  // round's map: hold, +-step (l.18 / l.23-25), or the override to max (l.10)
  // one round: Alg. 2 on the H previous events, Alg. 1, the event log
  auto round_d = [&](int i, double D) {
    const bool pi = D > P.d_inc, pd = !pi && D < P.d_dec;
    inc |= (uint32_t)pi << i;
    dcr |= (uint32_t)pd << i;
    if constexpr (!kBits) {
      const bool hf = __popc((uint32_t)(hist & hmask)) + __popc((uint32_t)((uint64_t)hist >> 32)) >= P.k;
      hw |= (uint32_t)hf << i;
      hist = ((hist << 1) | (HT)(pi || pd)) & hmask;
    }
  };
  double pdw[WT > 1 ? WT - 1 : 1];   // WT: x[tw-W+1 .. tw-1], widened (valid when have_pd)
  bool have_pd = false;
  auto round = [&](int i, float xt, float xl) {
    const double D = (double)xt - (double)xl;
    const bool pi = D > P.d_inc, pd = !pi && D < P.d_dec;
    inc |= (uint32_t)pi << i;
    dcr |= (uint32_t)pd << i;
    if constexpr (!kBits) {
      const bool hf = __popc((uint32_t)(hist & hmask)) + __popc((uint32_t)((uint64_t)hist >> 32)) >= P.k;
      hw |= (uint32_t)hf << i;
      hist = ((hist << 1) | (HT)(pi || pd)) & hmask;
    }
  };
  for (int32_t tw = t0; tw < t1; tw += 32) {
    inc = dcr = hw = 0;
    if (WT > 0 && tw >= P.W && tw + 32 <= t1) {   // a full word, lags from registers
      const float* px = a.x + (int64_t)tw * a.ld + n;
      if (!have_pd) {
#pragma unroll
        for (int k = 0; k < (WT > 1 ? WT - 1 : 0); ++k) pdw[k] = (double)__ldg(px + (k - (WT - 1)) * ld32);
        have_pd = true;
      }
      float xs[32];
      load_rows<32>(px, ld32, xs);
      double xd[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        xd[i] = (double)xs[i];                                   // exact widening, once
        const double xl = (i >= WT - 1) ? xd[i - (WT > 1 ? WT - 1 : 0)] : pdw[i < WT - 1 ? i : 0];
        round_d(i, xd[i] - xl);                                 // Alg. 1 l.3 numerator (RN)
      }
#pragma unroll
      for (int k = 0; k < (WT > 1 ? WT - 1 : 0); ++k) pdw[k] = xd[32 - (WT - 1) + k];
    } else if (tw >= P.W && tw + 32 <= t1) {   // a full word of MDFS rounds
      const float* px = a.x + (int64_t)tw * a.ld + n;
      const float* pl = px - (int64_t)(P.W - 1) * a.ld;
      constexpr int kq = kWalkChunk / 2;  // samples + lags: 16 loads ahead
#pragma unroll
      for (int h = 0; h < 32 / kq; ++h) {
        float xs[kq], xl[kq];
        load_rows<kq>(px + h * kq * ld32, ld32, xs);
        load_rows<kq>(pl + h * kq * ld32, ld32, xl);
#pragma unroll
        for (int i = 0; i < kq; ++i) round(h * kq + i, xs[i], xl[i]);
      }
    } else {                            // warm-up rounds (t < W) / the ragged tail
      for (int32_t t = max(tw, P.W); t < min(tw + 32, t1); ++t)
        round(t - tw, a.x[(int64_t)t * a.ld + n], a.x[(int64_t)(t - P.W + 1) * a.ld + n]);
      have_pd = false;
    }
    if constexpr (kBits) {
      // rounds of this word that ran Alg. 2: t >= W and t < t1 (inc / dcr
      // are zero elsewhere, so E = inc | dcr is the event log of the word)
      const uint32_t E = inc | dcr;
      uint32_t valid = ~0u;
      if (tw < P.W) valid = (P.W - tw >= 32) ? 0u : (~0u << (P.W - tw));
      if (tw + 32 > t1) valid &= (1u << (t1 - tw)) - 1u;
      if (P.H == 10) {
        uint32_t cnt[4];
        Window<10>::count(E, Eprev, 10, cnt);
        hw = ge_k<4>(cnt, km) & valid;
      } else {
        uint32_t cnt[6];
        Window<0>::count(E, Eprev, P.H, cnt);
        hw = ge_k<6>(cnt, km) & valid;
      }
      Eprev = E;
    }
    const int64_t w = tw >> 5;
    mk[w * a.N] = inc;
    mk[(a.nw + w) * a.N] = dcr;
    mk[(2 * (int64_t)a.nw + w) * a.N] = hw;
    // compose the word's rounds into the map: everything up to the last
    // override (l.10) collapses to the constant r_max; after it only the
    // +-step actions (l.18 / l.23-25) remain, visited sparsely
    uint32_t acts = inc | dcr;
    if (hw) {
      const int j = 31 - __clz(hw);
      d = 0;
      lo = hi = lmax;
      acts = j == 31 ? 0u : acts & (0xFFFFFFFEu << j);
    }
    while (acts) {
      const int i = __ffs(acts) - 1;
      acts &= acts - 1;
      const int sd = ((inc >> i) & 1u) ? step : -step;
      d = min(max(d + sd, -K), K);
      lo = min(max(lo + sd, lmin), lmax);
      hi = min(max(hi + sd, lmin), lmax);
    }
  }
  if (s < a.nseg - 1) a.map[((int64_t)cl * a.nseg + s) * a.N + n] = map_pack(d, lo, hi);
}

// Pass 2: the same threads replay the step rule from the true carry-in and
// meter model M at the level that governs each interval.  Per round only
// the level walk and three bit masks (decision at r_min, level change,
// sample above the capacity at r_min -- a superset of every level's stretch
// since B_l grows with l -- and bursts) are on the per-sample path; the
// word's levels go to shared memory, and the sparse work (stretch q at the
// level of each flagged interval, per-level run lengths at each change,
// burst counts) runs once per word over the set bits.
template <bool BURST>
__global__ void __launch_bounds__(kWalkThreads, 6) walk_replay_kernel(WalkArgs a, DevPlatform plat,
                                                                   const __grid_constant__ WalkLevels lv) {
  __shared__ double s_invB[kWalkMaxLv];
  __shared__ float s_xthr[kWalkMaxLv];
  __shared__ uint8_t s_bkeep[kWalkMaxLv];
  __shared__ uint8_t s_lv[32][kWalkThreads];  // dec[32w + i] of the current word
  // level offsets of 4 rounds as signed bytes (byte j: +step up, -step down,
  // +K the override -- min(l + K, r_max) = r_max --, 0 hold), indexed by the
  // rounds' (up | override) nibble and, above it, their (down | override) nibble
  __shared__ uint32_t s_off[256];
  extern __shared__ unsigned int s_cnt[];     // [nlev][kWalkThreads] intervals per level
  const int lmin = plat.r_min, lmax = plat.r_max, nlev = lmax - lmin + 1;
  const int32_t s = blockIdx.y, cl = blockIdx.z, c = a.c0 + cl;
  const DevPolicy P = a.pol[c];
  const int step = (P.variant & MAGUS_VARIANT_GRADUAL) ? P.step : (lmax - lmin);
  const int K = lmax - lmin;
  for (int i = 0; i < nlev; ++i) s_cnt[i * kWalkThreads + threadIdx.x] = 0u;
  for (int i = threadIdx.x; i < nlev; i += kWalkThreads) {
    s_invB[i] = lv.invB[i];
    s_xthr[i] = lv.xthr[i];
    s_bkeep[i] = lv.bkeep[i];
  }
  for (int idx = threadIdx.x; idx < 256; idx += kWalkThreads) {
    uint32_t F = 0;
    for (int j = 0; j < 4; ++j) {
      const int code = ((idx >> j) & 1) | (((idx >> (4 + j)) & 1) << 1);
      const uint32_t b = code == 1 ? (uint32_t)step : (code == 2 ? (uint32_t)(256 - step) : (code == 3 ? (uint32_t)K : 0u));
      F |= b << (8 * j);
    }
    s_off[idx] = F;
  }
  __syncthreads();
  const int tid = threadIdx.x;
  const int64_t n = (int64_t)blockIdx.x * kWalkThreads + tid;
  if (n >= a.N) return;
  const int32_t t0 = s * a.seg_len, t1 = min(a.T, t0 + a.seg_len);

  // carry-in dec[t0 - 1]: dec[-1] := r_max (P@23755), then every earlier
  // segment's map
  int lvl = lmax;
  for (int32_t j = 0; j < s; ++j) lvl = map_apply(a.map[((int64_t)cl * a.nseg + j) * a.N + n], lvl);

  int cur = lvl;                       // level of the current run of intervals
  int32_t run_start = t0;
  float xthr_cur = s_xthr[lvl - lmin];  // x > xthr_cur <=> interval t stretches at dec[t-1]
  int qlev = lvl;                      // stretch q of level qlev not yet flushed
  unsigned long long qacc = 0;
  int32_t events = 0, hi_rounds = 0, msr = 0, changes = 0, n_min_dec = 0, b_base = 0, b_magus = 0;
  unsigned long long q_base = 0, digest = 0;
  const double invB_max = plat.invB_max;
  const float xthr_max = plat.xthr_max, xburst = plat.xburst;
  unsigned int* lvn = a.lvn + (int64_t)c * nlev * a.N + n;
  unsigned long long* lvq = a.lvq + (int64_t)c * nlev * a.N + n;
  const uint32_t* mk = a.mask + (int64_t)cl * 3 * a.nw * a.N + n;
  const int ld32 = (int)a.ld;
  uint32_t inc = 0, dcr = 0, hw = 0, word = 0, chg = 0, big = 0, bmx = 0, bst = 0;

  // round i of the word: the step rule from the pass-1 masks (all zero in
  // the warm-up, t < W), and the per-sample flags of interval 32w + i
  // full words: round i's level offset as a signed byte (+K on the override --
  // min(l + K, r_max) = r_max -- +-step, 0), byte i % 4 of F[i / 4]; one
  // sign-extending byte permute per round instead of three bit tests and
  // selects
  auto round_f = [&](int i, float xt, uint32_t F) {
    or_if_gt(big, xt, xthr_cur, 1u << i);     // stretched at its level (sparse)
    or_if_gt(bmx, xt, xthr_max, 1u << i);     // ... and at r_max (q_base; rarer still)
    if (BURST) or_if_gt(bst, xt, xburst, 1u << i);
    int dl;
    asm("prmt.b32 %0, %1, 0, %2;" : "=r"(dl) : "r"(F), "r"((uint32_t)((i & 3) | ((8 | (i & 3)) * 0x1110))));
    const int prev = lvl;
    lvl = min(max(lvl + dl, lmin), lmax);                      // l.10 / l.18-19 / l.23-25
    s_lv[i][tid] = (uint8_t)lvl;
    xthr_cur = s_xthr[lvl - lmin];
    or_if_eq(word, lvl, lmin, 1u << i);
    or_if_ne(chg, lvl, prev, 1u << i);
  };
  auto round = [&](int i, float xt) {
    big |= (uint32_t)(xt > xthr_cur) << i;    // stretched at its level (sparse)
    bmx |= (uint32_t)(xt > xthr_max) << i;    // ... and at r_max (q_base; rarer still)
    if (BURST) bst |= (uint32_t)(xt > xburst) << i;
    const bool hf = (hw >> i) & 1u, pi = (inc >> i) & 1u, pd = (dcr >> i) & 1u;
    const int sd = pi ? step : (pd ? -step : 0);
    const int nl = min(max(lvl + sd, lmin), lmax);
    const int prev = lvl;
    lvl = hf ? lmax : nl;                                      // l.10 / l.18-19 / l.23-25
    s_lv[i][tid] = (uint8_t)lvl;
    xthr_cur = s_xthr[lvl - lmin];
    word |= (uint32_t)(lvl == lmin) << i;
    chg |= (uint32_t)(lvl != prev) << i;
  };
  for (int32_t tw = t0; tw < t1; tw += 32) {
    const int64_t w = tw >> 5;
    inc = mk[w * a.N];
    dcr = mk[(a.nw + w) * a.N];
    hw = mk[(2 * (int64_t)a.nw + w) * a.N];
    events += __popc(inc | dcr);                               // l.17 / l.22
    hi_rounds += __popc(hw);
    msr += __popc(inc | dcr | hw);                             // tune_uncore_freq calls
    const int before = lvl;                                    // dec[32w - 1]
    word = chg = big = bmx = bst = 0;
    const int rem = min(32, t1 - tw);
    const float* px = a.x + (int64_t)tw * a.ld + n;
    if (rem == 32) {
      // the offset bytes of each 4 rounds from the shared table (inc, dcr
      // exclusive; the override sets both nibbles)
      const uint32_t clo = inc | hw, chi = dcr | hw;
      const uint32_t off_s = (uint32_t)__cvta_generic_to_shared(s_off);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        float xs[kWalkChunk];
        load_rows<kWalkChunk>(px + h * kWalkChunk * ld32, ld32, xs);
#pragma unroll
        for (int q = 0; q < kWalkChunk / 4; ++q) {
          const int sh = 4 * (h * (kWalkChunk / 4) + q);
          const uint32_t idx = ((clo >> sh) & 15u) | (((chi >> sh) & 15u) << 4);
          uint32_t F;
          asm("ld.shared.u32 %0, [%1];" : "=r"(F) : "r"(off_s + 4u * idx));
#pragma unroll
          for (int i = 0; i < 4; ++i) round_f(h * kWalkChunk + 4 * q + i, xs[4 * q + i], F);
        }
      }
    } else {
      for (int i = 0; i < rem; ++i) round(i, __ldg(px + i * ld32));
    }
    n_min_dec += __popc(word);
    changes += __popc(chg);                                    // never at t = 0 (dec[-1] := max)
    if (a.dec) a.dec[((int64_t)c * a.nw + w) * a.N + n] = word;
    digest += (unsigned long long)word * digest_mul(w);
    if (a.levels)
      for (int i = 0; i < rem; ++i) a.levels[((int64_t)c * a.T + tw + i) * a.N + n] = s_lv[i][tid];
    // model M at dec[t-1]: stretch of the flagged intervals, bursts
    uint32_t m = big | bmx | bst;
    while (m) {
      const int i = __ffs(m) - 1;
      m &= m - 1;
      const int L = i ? (int)s_lv[i - 1][tid] : before;
      const float xt = __ldg(px + i * ld32);
      if ((big >> i) & 1u) {
        if (L != qlev) {
          if (qacc) atomicAdd(lvq + (int64_t)(qlev - lmin) * a.N, qacc);
          qacc = 0;
          qlev = L;
        }
        qacc += q_literal(xt, s_invB[L - lmin]);
      }
      if ((bmx >> i) & 1u) q_base += q_literal(xt, invB_max);
      if (BURST && ((bst >> i) & 1u)) {                        // Sec. 6.3 bursts
        ++b_base;
        b_magus += s_bkeep[L - lmin];
      }
    }
    // per-level interval counts: a change in round 32w + i ends the run of
    // intervals that ran at cur
    m = chg;
    while (m) {
      const int i = __ffs(m) - 1;
      m &= m - 1;
      s_cnt[(cur - lmin) * kWalkThreads + tid] += (unsigned int)(tw + i + 1 - run_start);
      run_start = tw + i + 1;
      cur = s_lv[i][tid];
    }
  }
  s_cnt[(cur - lmin) * kWalkThreads + tid] += (unsigned int)(t1 - run_start);
  for (int l = 0; l < nlev; ++l) {
    const unsigned int v = s_cnt[l * kWalkThreads + tid];
    if (v) atomicAdd(lvn + (int64_t)l * a.N, v);
  }
  if (qacc) atomicAdd(lvq + (int64_t)(qlev - lmin) * a.N, qacc);
  unsigned long long* acc = a.acc + (int64_t)c * kWalkFields * a.N + n;
  const unsigned long long vals[kWalkFields] = {
      (unsigned long long)events, (unsigned long long)hi_rounds, (unsigned long long)msr,
      (unsigned long long)changes, (unsigned long long)n_min_dec, q_base, digest,
      (unsigned long long)b_base, (unsigned long long)b_magus};
#pragma unroll
  for (int f = 0; f < kWalkFields; ++f)
    if (vals[f]) atomicAdd(acc + (int64_t)f * a.N, vals[f]);
}

__global__ void __launch_bounds__(kWalkThreads) walk_final_kernel(WalkArgs a, DevPlatform plat) {
  const int64_t gid = (int64_t)blockIdx.x * kWalkThreads + threadIdx.x;
  if (gid >= a.N * a.C) return;
  const int32_t c = (int32_t)(gid / a.N);
  const int64_t n = gid - (int64_t)c * a.N;
  const int lmin = plat.r_min, lmax = plat.r_max, nlev = lmax - lmin + 1;
  const unsigned long long* acc = a.acc + (int64_t)c * kWalkFields * a.N + n;
  const unsigned int* lvn = a.lvn + (int64_t)c * nlev * a.N + n;
  const unsigned long long* lvq = a.lvq + (int64_t)c * nlev * a.N + n;
  const int64_t n_min_int = lvn[0];
  const uint64_t q_min = lvq[0];
  uint64_t q_max = 0;
  for (int i = 1; i < nlev; ++i) q_max += lvq[(int64_t)i * a.N];
  magus_summary* so = a.summary + gid;
  magus_base* bo = (a.base && c == 0) ? a.base + n : nullptr;
  const int64_t changes = (int64_t)acc[WF_CH * a.N];
  finalize_summary(plat, a.T, (int64_t)acc[WF_EV * a.N], (int64_t)acc[WF_HI * a.N], (int64_t)acc[WF_MSR * a.N],
                   changes, (int64_t)acc[WF_MDEC * a.N], n_min_int, q_min, q_max, acc[WF_QBASE * a.N],
                   acc[WF_DIG * a.N], (int64_t)acc[WF_BB * a.N], (int64_t)acc[WF_BM * a.N], so, bo);
  // general model M: energy = sum over the ratios, ascending
  double energy = 0.0;
  for (int i = 0; i < nlev; ++i) {
    const int l = lmin + i;
    const double Pl = a.p_lo + (a.p_span * (double)(l - lmin)) / (double)(lmax - lmin);
    energy = energy + Pl * (plat.dt * (double)lvn[(int64_t)i * a.N] + plat.cQ * (double)lvq[(int64_t)i * a.N]);
  }
  so->energy_j = energy + plat.e_sw * (double)changes;
}


// ---------------------------------------------------------------------------
// One pass (walk_fused_kernel): the map and the replay of a segment in the
// same scan, carry by decoupled look-back.
//
// Every round applies a clamp-shift map with the offset dl in {+K (the
// override, l.10: min(l + K, r_max) = r_max), +step, -step, 0}, so one
// thread walks three values per round: the level reached from r_max (hi),
// from r_min (lo) and the saturated offset d.  The clamp-shift maps are
// monotone, so every carry-in gives a level between lo and hi: once lo == hi
// (after an override, or after the steps saturate at a bound) the level is
// the same for every carry-in and equals hi.  From the word after that point
// on, the thread meters model M on the fly; the words before it (the
// carry-dependent prefix, usually short) keep their Alg. 1 / Alg. 2 masks in
// scratch and are replayed from the true carry once the look-back has it.
// The segment's status is its map (lo == hi: the end level itself).
// Work tickets are taken in (config, segment, trace group) order, so every
// predecessor segment holds a CTA already: the look-back never waits on a
// CTA that is not running.
// ---------------------------------------------------------------------------
constexpr uint32_t kWalkPub = 1u << 24;  // status published (map in bits 0..23)

struct FusedArgs {
  uint32_t* status;   // [C][nseg][N] (zero at launch)
  uint32_t* ticket;   // [batches] (zero at launch)
  int32_t ngroups;    // trace groups of kWalkThreads
};

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <typename HT, bool BURST>
__global__ void __launch_bounds__(kWalkThreads, 4) walk_fused_kernel(WalkArgs a, DevPlatform plat,
                                                                  const __grid_constant__ WalkLevels lv,
                                                                  FusedArgs f, int32_t batch) {
  __shared__ double s_invB[kWalkMaxLv];
  __shared__ float s_xthr[kWalkMaxLv];
  __shared__ uint8_t s_bkeep[kWalkMaxLv];
  __shared__ uint8_t s_lv[32][kWalkThreads];  // dec[32w + i] of the current word
  __shared__ uint32_t s_ticket;
  extern __shared__ unsigned int s_cnt[];     // [nlev][kWalkThreads] intervals per level
  const int lmin = plat.r_min, lmax = plat.r_max, nlev = lmax - lmin + 1;
  const int tid = threadIdx.x;
  for (int i = 0; i < nlev; ++i) s_cnt[i * kWalkThreads + tid] = 0u;
  for (int i = tid; i < nlev; i += kWalkThreads) {
    s_invB[i] = lv.invB[i];
    s_xthr[i] = lv.xthr[i];
    s_bkeep[i] = lv.bkeep[i];
  }
  if (tid == 0) s_ticket = atomicAdd(f.ticket + batch, 1u);
  __syncthreads();
  const uint32_t per_cfg = (uint32_t)a.nseg * (uint32_t)f.ngroups;
  const int32_t cl = (int32_t)(s_ticket / per_cfg);
  const int32_t s = (int32_t)((s_ticket % per_cfg) / (uint32_t)f.ngroups);
  const int32_t g = (int32_t)(s_ticket % (uint32_t)f.ngroups);
  const int32_t c = a.c0 + cl;
  const int64_t n = (int64_t)g * kWalkThreads + tid;
  if (n >= a.N) return;
  const DevPolicy P = a.pol[c];
  const int32_t t0 = s * a.seg_len, t1 = min(a.T, t0 + a.seg_len);
  const int K = lmax - lmin;
  const int step = (P.variant & MAGUS_VARIANT_GRADUAL) ? P.step : K;
  const HT hmask = P.H >= (int)(8 * sizeof(HT)) ? (HT)~(HT)0 : (HT)(((HT)1 << P.H) - 1);
  HT hist = (HT)history_at(a, P, n, max(t0, P.W)) & hmask;
  constexpr bool kBits = sizeof(HT) == 4;
  uint32_t Eprev = kBits ? __brev((uint32_t)hist) : 0u;  // bit i = round t0 - 32 + i
  uint32_t km[6];
#pragma unroll
  for (int j = 0; j < 6; ++j) km[j] = ((P.k >> j) & 1) ? ~0u : 0u;
  const int ld32 = (int)a.ld;
  const float xthr_max = plat.xthr_max, xburst = plat.xburst;
  const double invB_max = plat.invB_max;
  unsigned int* lvn = a.lvn + (int64_t)c * nlev * a.N + n;
  unsigned long long* lvq = a.lvq + (int64_t)c * nlev * a.N + n;
  uint32_t* mk = a.mask + (int64_t)cl * 3 * a.nw * a.N + n;

  // the three walks (segment 0 starts from the known dec[-1] = r_max)
  int lh = lmax, ll = s == 0 ? lmax : lmin, dd = 0;
  int32_t t_live = s == 0 ? t0 : -1;   // first interval metered in the scan (-1: none yet)
  // model-M state of the metered intervals
  int cur = lmax;                      // level of the current run of intervals
  int32_t run_start = t0;
  int qlev = lmax;                     // stretch q of level qlev not yet flushed
  unsigned long long qacc = 0, q_base = 0, digest = 0;
  int32_t events = 0, hi_rounds = 0, msr = 0, changes = 0, n_min_dec = 0, b_base = 0, b_magus = 0;

  // The replay of one word at the level `lvl` (dec[32w - 1]) with model M:
  // the step rule from the masks, the per-interval flags, and the sparse
  // stretch / run-length / burst work over the word's set bits.
  auto meter_word = [&](int32_t tw, uint32_t inc, uint32_t dcr, uint32_t hw, const float (&xs)[32], int& lvl) {
    const int64_t w = tw >> 5;
    const int rem = min(32, t1 - tw);
    const uint32_t live = rem == 32 ? ~0u : ((1u << rem) - 1u);
    const int before = lvl;
    uint32_t word = 0, chg = 0, big = 0, bmx = 0, bst = 0;
    float xthr_cur = s_xthr[lvl - lmin];
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      big |= (uint32_t)(xs[i] > xthr_cur) << i;   // stretched at its level dec[t-1]
      bmx |= (uint32_t)(xs[i] > xthr_max) << i;
      if (BURST) bst |= (uint32_t)(xs[i] > xburst) << i;
      const int dl = ((hw >> i) & 1u) ? K : (((inc >> i) & 1u) ? step : (((dcr >> i) & 1u) ? -step : 0));
      const int prev = lvl;
      lvl = min(max(lvl + dl, lmin), lmax);        // l.10 / l.18-19 / l.23-25
      s_lv[i][tid] = (uint8_t)lvl;
      xthr_cur = s_xthr[lvl - lmin];
      word |= (uint32_t)(lvl == lmin) << i;
      chg |= (uint32_t)(lvl != prev) << i;
    }
    word &= live;
    big &= live;
    bmx &= live;
    bst &= live;
    n_min_dec += __popc(word);
    changes += __popc(chg);                       // rounds past T hold: no change
    if (a.dec) a.dec[((int64_t)c * a.nw + w) * a.N + n] = word;
    digest += (unsigned long long)word * digest_mul(w);
    if (a.levels)
      for (int i = 0; i < rem; ++i) a.levels[((int64_t)c * a.T + tw + i) * a.N + n] = s_lv[i][tid];
    uint32_t m = big | bmx | bst;
    while (m) {
      const int i = __ffs(m) - 1;
      m &= m - 1;
      const int L = i ? (int)s_lv[i - 1][tid] : before;
      const float xt = __ldg(a.x + (int64_t)(tw + i) * a.ld + n);
      if ((big >> i) & 1u) {
        if (L != qlev) {
          if (qacc) atomicAdd(lvq + (int64_t)(qlev - lmin) * a.N, qacc);
          qacc = 0;
          qlev = L;
        }
        qacc += q_literal(xt, s_invB[L - lmin]);
      }
      if ((bmx >> i) & 1u) q_base += q_literal(xt, invB_max);
      if (BURST && ((bst >> i) & 1u)) {
        ++b_base;
        b_magus += s_bkeep[L - lmin];
      }
    }
    m = chg;
    while (m) {
      const int i = __ffs(m) - 1;
      m &= m - 1;
      s_cnt[(cur - lmin) * kWalkThreads + tid] += (unsigned int)(tw + i + 1 - run_start);
      run_start = tw + i + 1;
      cur = s_lv[i][tid];
    }
  };

  for (int32_t tw = t0; tw < t1; tw += 32) {
    // ---- Alg. 1 (and Alg. 2 for H > 32) over the word ----
    float xs[32];
    uint32_t inc = 0, dcr = 0, hw = 0;
    const float* px = a.x + (int64_t)tw * a.ld + n;
    auto round = [&](int i, float xt, float xl) {
      const double D = (double)xt - (double)xl;
      const bool pi = D > P.d_inc, pd = !pi && D < P.d_dec;
      inc |= (uint32_t)pi << i;
      dcr |= (uint32_t)pd << i;
      if constexpr (!kBits) {
        const bool hf = __popc((uint32_t)(hist & hmask)) + __popc((uint32_t)((uint64_t)hist >> 32)) >= P.k;
        hw |= (uint32_t)hf << i;
        hist = ((hist << 1) | (HT)(pi || pd)) & hmask;
      }
    };
    if (tw >= P.W && tw + 32 <= t1) {   // a full word of MDFS rounds
      const float* pl = px - (int64_t)(P.W - 1) * a.ld;
#pragma unroll
      for (int h = 0; h < 4; ++h) {
        float xl[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) xs[h * 8 + i] = __ldg(px + (h * 8 + i) * ld32);
        load_rows<8>(pl + h * 8 * ld32, ld32, xl);
#pragma unroll
        for (int i = 0; i < 8; ++i) round(h * 8 + i, xs[h * 8 + i], xl[i]);
      }
    } else {                            // warm-up rounds (t < W) / the ragged tail
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const int32_t t = tw + i;
        xs[i] = t < t1 ? __ldg(px + i * ld32) : 0.0f;
        if (t >= P.W && t < t1) round(i, xs[i], __ldg(a.x + (int64_t)(t - P.W + 1) * a.ld + n));
      }
    }
    if constexpr (kBits) {   // Alg. 2 bit-parallel (E = the word's event log)
      const uint32_t E = inc | dcr;
      uint32_t valid = ~0u;
      if (tw < P.W) valid = (P.W - tw >= 32) ? 0u : (~0u << (P.W - tw));
      if (tw + 32 > t1) valid &= (1u << (t1 - tw)) - 1u;
      if (P.H == 10) {
        uint32_t cnt[4];
        Window<10>::count(E, Eprev, 10, cnt);
        hw = ge_k<4>(cnt, km) & valid;
      } else {
        uint32_t cnt[6];
        Window<0>::count(E, Eprev, P.H, cnt);
        hw = ge_k<6>(cnt, km) & valid;
      }
      Eprev = E;
    }
    events += __popc(inc | dcr);                   // l.17 / l.22
    hi_rounds += __popc(hw);
    msr += __popc(inc | dcr | hw);                 // tune_uncore_freq calls
    // ---- the step rule ----
    if (t_live >= 0) {
      meter_word(tw, inc, dcr, hw, xs, lh);        // levels known: replay and meter
    } else {
      // carry-dependent: walk the three values, keep the masks for the replay
      const int64_t w = tw >> 5;
      mk[w * a.N] = inc;
      mk[(a.nw + w) * a.N] = dcr;
      mk[(2 * (int64_t)a.nw + w) * a.N] = hw;
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const int dl = ((hw >> i) & 1u) ? K : (((inc >> i) & 1u) ? step : (((dcr >> i) & 1u) ? -step : 0));
        lh = min(max(lh + dl, lmin), lmax);
        ll = min(max(ll + dl, lmin), lmax);
        dd = min(max(dd + dl, -K), K);
      }
      if (ll == lh && tw + 32 < t1) {              // collapsed: meter from the next word on
        t_live = tw + 32;
        cur = qlev = lh;
        run_start = t_live;
      }
    }
  }
  // ---- publish the segment's map, look back for the carry ----
  uint32_t* st = f.status + ((int64_t)cl * a.nseg) * a.N + n;
  const bool known = t_live >= 0 || ll == lh;
  st_release_u32(st + (int64_t)s * a.N, kWalkPub | (known ? map_pack(0, lh, lh) : map_pack(dd, ll, lh)));
  if (t_live >= 0) s_cnt[(cur - lmin) * kWalkThreads + tid] += (unsigned int)(t1 - run_start);
  const int32_t t_def = t_live >= 0 ? t_live : t1;   // intervals [t0, t_def) replayed from the carry
  if (s > 0 && t_def > t0) {
    int32_t j = s - 1;
    uint32_t v;
    for (;; --j) {   // the nearest predecessor whose end level is known (segment 0's always is)
      while (((v = ld_acquire_u32(st + (int64_t)j * a.N)) & kWalkPub) == 0u) __nanosleep(64);
      if (((v >> 8) & 0xFFu) == ((v >> 16) & 0xFFu)) break;
    }
    int lvl = (int)((v >> 16) & 0xFFu);
    for (++j; j < s; ++j) lvl = map_apply(ld_acquire_u32(st + (int64_t)j * a.N), lvl);
    if (!known)   // the true end level, for the segments after this one
      st_release_u32(st + (int64_t)s * a.N, kWalkPub | map_pack(0, map_apply(map_pack(dd, ll, lh), lvl),
                                                                  map_apply(map_pack(dd, ll, lh), lvl)));
    // replay the carry-dependent words from the true carry
    if (qacc) atomicAdd(lvq + (int64_t)(qlev - lmin) * a.N, qacc);
    qacc = 0;
    cur = qlev = lvl;
    run_start = t0;
    for (int32_t tw = t0; tw < t_def; tw += 32) {
      const int64_t w = tw >> 5;
      const uint32_t inc = mk[w * a.N], dcr = mk[(a.nw + w) * a.N], hw = mk[(2 * (int64_t)a.nw + w) * a.N];
      const float* px = a.x + (int64_t)tw * a.ld + n;
      float xs[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) xs[i] = tw + i < t1 ? __ldg(px + i * ld32) : 0.0f;
      meter_word(tw, inc, dcr, hw, xs, lvl);
    }
    s_cnt[(cur - lmin) * kWalkThreads + tid] += (unsigned int)(t_def - run_start);
  }
  for (int l = 0; l < nlev; ++l) {
    const unsigned int v = s_cnt[l * kWalkThreads + tid];
    if (v) atomicAdd(lvn + (int64_t)l * a.N, v);
  }
  if (qacc) atomicAdd(lvq + (int64_t)(qlev - lmin) * a.N, qacc);
  unsigned long long* acc = a.acc + (int64_t)c * kWalkFields * a.N + n;
#ifdef WALK_STATS  // developer statistics in the burst fields: deferred words, look-back steps
  b_base = (t_def - t0 + 31) / 32;
  b_magus = s > 0 && t_def > t0 ? 1 : 0;
#endif
  const unsigned long long vals[kWalkFields] = {
      (unsigned long long)events, (unsigned long long)hi_rounds, (unsigned long long)msr,
      (unsigned long long)changes, (unsigned long long)n_min_dec, q_base, digest,
      (unsigned long long)b_base, (unsigned long long)b_magus};
#pragma unroll
  for (int fi = 0; fi < kWalkFields; ++fi)
    if (vals[fi]) atomicAdd(acc + (int64_t)fi * a.N, vals[fi]);
}

}  // namespace

// configs per launch: the pass-1 masks of a batch stay below this
constexpr size_t kWalkMaskBudget = size_t(1) << 30;

static int64_t walk_batch(int64_t N, int32_t C, int64_t T) {
  const size_t per = 3 * 4 * (size_t)((T + 31) / 32) * (size_t)N;
  return std::max<int64_t>(1, std::min<int64_t>(C, (int64_t)(kWalkMaskBudget / std::max<size_t>(per, 1))));
}

size_t walk_scratch_bytes(int64_t N, int32_t C, int64_t T, int64_t nseg, const DevPlatform& plat) {
  const int nlev = plat.r_max - plat.r_min + 1;
  const int64_t B = walk_batch(N, C, T), nw = (T + 31) / 32;
  auto al = [](size_t b) { return (b + 255) / 256 * 256; };
  return al(4 * (size_t)B * nseg * N) + al(12 * (size_t)B * nw * N) + al(8 * (size_t)C * kWalkFields * N) +
         al(4 * (size_t)C * nlev * N) + al(8 * (size_t)C * nlev * N) + al(4 * (size_t)((C + B - 1) / B));
}

int launch_walk(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld, const DevPolicy* pol_dev,
                int32_t C, int32_t max_H, const DevPlatform& plat, double bw_max, double p_lo, double p_span,
                int64_t nseg, int64_t seg_len, void* scratch, magus_summary* out_summary, magus_base* out_base,
                uint32_t* out_dec, uint8_t* out_levels, bool fused, int32_t same_W) {
  const int nlev = plat.r_max - plat.r_min + 1;
  const int64_t B = walk_batch(N, C, T), nw = (T + 31) / 32;
  auto al = [](size_t b) { return (b + 255) / 256 * 256; };
  char* sp = (char*)scratch;
  WalkArgs a;
  a.x = x;
  a.N = N;
  a.ld = ld;
  a.T = (int32_t)T;
  a.nw = (int32_t)nw;
  a.pol = pol_dev;
  a.C = C;
  a.c0 = 0;
  a.nseg = (int32_t)nseg;
  a.seg_len = (int32_t)seg_len;
  a.map = (uint32_t*)sp;
  sp += al(4 * (size_t)B * nseg * N);
  a.mask = (uint32_t*)sp;
  sp += al(12 * (size_t)B * nw * N);
  a.acc = (unsigned long long*)sp;
  sp += al(8 * (size_t)C * kWalkFields * N);
  a.lvn = (unsigned int*)sp;
  sp += al(4 * (size_t)C * nlev * N);
  a.lvq = (unsigned long long*)sp;
  sp += al(8 * (size_t)C * nlev * N);
  uint32_t* tickets = (uint32_t*)sp;
  a.summary = out_summary;
  a.base = out_base;
  a.dec = out_dec;
  a.levels = out_levels;
  a.p_lo = p_lo;
  a.p_span = p_span;
  // per-level constants: B_l = (bw_max * l) / r_max, 1 / B_l (kernels_ref.cu capacity())
  WalkLevels lv{};
  for (int i = 0; i < nlev; ++i) {
    const int l = plat.r_min + i;
    const double Bl = (bw_max * (double)l) / (double)plat.r_max;
    lv.invB[i] = 1.0 / Bl;
    lv.xthr[i] = stretch_threshold(lv.invB[i]);
    lv.bkeep[i] = (plat.burst_on && Bl > plat.burst_mbs) ? 1 : 0;
  }
  int launched = 0;
  // one compile-time W for the whole launch when every config shares it
  auto mk = max_H > 32 ? walk_map_kernel<uint64_t, 0> : walk_map_kernel<uint32_t, 0>;
  if (max_H <= 32) {
    switch (same_W) {
      case 4: mk = walk_map_kernel<uint32_t, 4>; break;
      case 6: mk = walk_map_kernel<uint32_t, 6>; break;
      case 10: mk = walk_map_kernel<uint32_t, 10>; break;
      case 16: mk = walk_map_kernel<uint32_t, 16>; break;
      default: break;
    }
  }
  const size_t cnt_smem = (size_t)nlev * kWalkThreads * sizeof(unsigned int);  // <= 65 KB (127 ratios)
  if (cnt_smem > 48 * 1024) {
    if (cudaFuncSetAttribute(walk_replay_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)cnt_smem) !=
            cudaSuccess ||
        cudaFuncSetAttribute(walk_replay_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)cnt_smem) !=
            cudaSuccess)
      return -1;
  }
  if (fused) {
    // one pass: the accumulators and the batch tickets start at zero, the
    // status words of every batch too (cleared before each batch)
    const int64_t nb = (C + B - 1) / B;
    if (cudaMemsetAsync(a.acc, 0, (size_t)((char*)tickets - (char*)a.acc) + 4 * (size_t)nb, s) != cudaSuccess) return -1;
    auto fk = max_H > 32 ? (plat.burst_on ? walk_fused_kernel<uint64_t, true> : walk_fused_kernel<uint64_t, false>)
                         : (plat.burst_on ? walk_fused_kernel<uint32_t, true> : walk_fused_kernel<uint32_t, false>);
    if (cnt_smem > 48 * 1024 &&
        cudaFuncSetAttribute(fk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)cnt_smem) != cudaSuccess)
      return -1;
    FusedArgs fa;
    fa.status = a.map;
    fa.ticket = tickets;
    fa.ngroups = (int32_t)((N + kWalkThreads - 1) / kWalkThreads);
    for (int64_t c0 = 0, bi = 0; c0 < C; c0 += B, ++bi) {
      a.c0 = (int32_t)c0;
      const int64_t nc = std::min<int64_t>(B, C - c0);
      if (cudaMemsetAsync(a.map, 0, 4 * (size_t)nc * nseg * N, s) != cudaSuccess) return -1;
      const unsigned grid = (unsigned)(fa.ngroups * nseg * nc);
      fk<<<grid, kWalkThreads, cnt_smem, s>>>(a, plat, lv, fa, (int32_t)bi);
      launched += 1;
    }
  }
  for (int64_t c0 = 0; c0 < C && !fused; c0 += B) {
    a.c0 = (int32_t)c0;
    const dim3 grid((unsigned)((N + kWalkThreads - 1) / kWalkThreads), (unsigned)nseg,
                    (unsigned)std::min<int64_t>(B, C - c0));
    mk<<<grid, kWalkThreads, 0, s>>>(a, plat.r_min, plat.r_max, nlev);
    if (plat.burst_on) walk_replay_kernel<true><<<grid, kWalkThreads, cnt_smem, s>>>(a, plat, lv);
    else walk_replay_kernel<false><<<grid, kWalkThreads, cnt_smem, s>>>(a, plat, lv);
    launched += 2;
  }
  const unsigned fb = (unsigned)((N * C + kWalkThreads - 1) / kWalkThreads);
  walk_final_kernel<<<fb, kWalkThreads, 0, s>>>(a, plat);
  return cudaGetLastError() == cudaSuccess ? launched + 1 : -1;
}

}  // namespace magus
