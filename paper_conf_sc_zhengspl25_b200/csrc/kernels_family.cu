// kernels_family.cu -- the sweeps' kernel (configs 3 and 4): one CTA replays
// a whole configuration FAMILY -- up to 16 bundles x 4 t_hi of one (W, H) --
// for 32 traces x one time segment, so the per-sample work is done once per
// trace instead of once per bundle.
//
// In a sweep grid (SWEEP256: 4 tau_inc x 4 tau_dec x 4 t_hi per W) every
// config of a W shares the Alg. 1 numerator Delta_t = x_t - x_{t-W+1}; the
// configs differ only in which inverted threshold Delta is compared with
// (d_inc, d_dec: 4 + 4 distinct values) and in k (t_hi).  The stream kernel's
// bundles share Delta only inside a bundle (4 configs), so each of the 16
// bundles re-reads and re-compares every sample.  Here:
//   * [32 steps x 32 traces] TMA boxes (4 KB) stream into a 6-stage ring (a
//     stage is held one word longer: it is the next word's lag), issued by
//     the first mask warp once all four have passed the word's barrier (no
//     producer warp: 20 warps leave 96 registers per thread);
//   * 4 MASK warps (lane = trace, warp m = steps 8m .. 8m+7 of the word)
//     compute Delta once per sample, compare it with every distinct threshold
//     of the family and write the 32-bit masks (one byte per warp), the
//     stretch masks (x > capacity at min / at max) and the word's inclusive
//     prefix sums P of the metered stretch q (model M) into a mask buffer;
//   * 16 BUNDLE warps (warp b = bundle b, lane = trace) read their bundle's
//     two masks and run the bit-parallel Alg. 2 / Alg. 3 of kernels_stream.cu
//     for the 4 configs.  The stretch sums over "interval at min" need no
//     per-sample loop: sum over the runs of the level mask of P[end] -
//     P[start - 1] (P is flat where no sample exceeds the capacity), one
//     shared load per level change;
//   * segments, carry look-back, integer accumulators, finalisation and the
//     totals rows are the stream kernel's, per config.
// Bit-identical to the stream kernel and the oracle for any family split,
// segmentation or time chunking.
#include <cuda.h>

#include <cstddef>

#include "bitops.cuh"
#include "device_common.cuh"
#include "ptx.cuh"

namespace magus {
namespace {

constexpr int kFT = 32;            // traces per CTA (= lanes of a bundle warp)
constexpr int kFStages = 6;        // TMA ring depth ([32 steps x 32 traces] = 4 KB each)
constexpr uint32_t kFStageBytes = 32u * kFT * 4u;
constexpr int kMaskWarps = 4;      // steps 8m .. 8m+7 of every word
constexpr int kMB = 3;             // mask buffers in flight between mask and bundle warps
constexpr int kFNB = 4;            // configs per bundle (t_hi variants)
constexpr int kFMaxWarps = kFamMaxBund + kMaskWarps;
constexpr int kTotAcc = kTotAccWords;

struct MaskBuf {  // one 32-step word of the CTA's 32 traces, [field][trace]
  uint32_t inc[kFamMaxThr][kFT];          // Delta > d_inc[i]
  uint32_t dec[kFamMaxThr][kFT];          // Delta < d_dec[i]
  uint32_t smin[kFT];                     // x > capacity at r_min
  uint32_t xmx[kFT];                      // x > capacity at r_max
  unsigned long long tot[kMaskWarps][kFT];   // per-byte sums of q_min (phase 1)
  unsigned long long totx[kMaskWarps][kFT];  // per-byte sums of q_max
  unsigned long long P[32][kFT];          // inclusive prefix of q_min over the word (smin != 0)
  unsigned long long Px[32][kFT];         // inclusive prefix of q_max (xmx != 0)
  unsigned long long M;                   // digest multiplier of the word
  unsigned long long pad_[15];
};
struct FamSmem {  // rarely touched per-(config slot, bundle thread) state
  unsigned long long qmax, pqmax, pdig;
  int32_t apos, wa;
  uint32_t dwa, pre_dec_a;
};

__device__ __forceinline__ void bar_named(int id, int count) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
__device__ __forceinline__ void sts_u8(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts_u64(uint32_t a, unsigned long long v) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long lds_u64v(uint32_t a) {
  unsigned long long v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}

// sum of q over the positions of `lv` (any mask), from the word's inclusive
// prefix P (column `col`, row stride 256 B): sum_t lv_t (P_t - P_t-1) = sum
// over run ends P_end - sum over the positions just before a run start.
// q is zero where the sample does not stretch (P flat there), so only lv's
// bits at the stretched positions matter: the callers pass lv held forward
// from one stretched position to the next (the carry-chain sample-and-hold of
// bitops.cuh), whose runs change only where lv changes between consecutive
// stretched samples -- never more runs than lv, one run (one load) for a
// word whose stretched samples are all in lv; the loop's trip count is the
// maximum over the warp's lanes.
__device__ __forceinline__ unsigned long long run_sum(uint32_t lv, uint32_t col) {
  const uint32_t nx = lv >> 1;
  uint32_t plus = lv & ~nx, minus = ~lv & nx;
  unsigned long long s = 0;
  // one trip per run: its end and (unless the run starts at 0) the position
  // before its start -- every minus bit belongs to a run, so popc(minus) <=
  // popc(plus) and one loop over the runs covers both (half the trips and
  // loop control of two loops)
  while (plus) {
    const int t = 31 - __clz(plus);
    plus ^= 1u << t;
    const int tm = 31 - __clz(minus | 1u);               // 0 when no minus bit is left
    const unsigned long long pm = lds_u64v(col + 256u * (uint32_t)tm);
    s += lds_u64v(col + 256u * (uint32_t)t);
    if (minus) s -= pm;
    minus &= ~(1u << tm);
  }
  return s;
}

template <int H_T, bool DEC, int NT>
__global__ void __launch_bounds__(32 * kFMaxWarps, 1)
family_kernel(const __grid_constant__ CUtensorMap tmap, const __grid_constant__ CUtensorMap tmul, int64_t N,
              int64_t T, const DevPolicy* __restrict__ pol, const int32_t* __restrict__ bundles,
              DevPlatform plat, int64_t nseg, int64_t seg_len, int32_t ngroups, int32_t nbund,
              const __grid_constant__ FamilyDev fam, StreamWork wk) {
  constexpr int kNBits = Window<H_T>::NBITS;
  extern __shared__ __align__(1024) unsigned char fsm[];
  __shared__ __align__(8) uint64_t full_bar[kFStages];
  __shared__ __align__(8) uint64_t mfull[kMB];
  __shared__ __align__(8) uint64_t mempty[kMB];
  __shared__ __align__(128) unsigned long long st_mul[kFStages][16];
  __shared__ uint32_t sh_last;
  __shared__ int32_t sh_work[4];
  __shared__ __align__(16) uint32_t s_km[kFamMaxBund][kFNB][8];

  float* stage = reinterpret_cast<float*>(fsm);
  MaskBuf* mbuf = reinterpret_cast<MaskBuf*>(fsm + kFStages * kFStageBytes);
  FamSmem* fs = reinterpret_cast<FamSmem*>(fsm + kFStages * kFStageBytes + kMB * sizeof(MaskBuf));
  const int nbt = nbund * 32;  // bundle threads
  auto FS = [&](int k, int t) -> FamSmem& { return fs[k * nbt + t]; };

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    // launch-order ticket -> (segment, trace group), segment-major: the
    // predecessor segment of a group always holds a smaller ticket
    const uint32_t ticket = atomicAdd(wk.ticket, 1u);
    sh_work[3] = (int32_t)ticket;
    sh_work[0] = (int32_t)(ticket / (uint32_t)ngroups);
    sh_work[2] = (int32_t)(ticket % (uint32_t)ngroups);
    for (int i = 0; i < kFStages; ++i) mbar_init(&full_bar[i], 1);
    for (int i = 0; i < kMB; ++i) {
      mbar_init(&mfull[i], 32 * kMaskWarps);
      mbar_init(&mempty[i], (uint32_t)nbt);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  // the first word's lag rows come from a "previous" stage never loaded:
  // zeros (those positions lie before the halo's needed history / in warm-up)
  for (int i = threadIdx.x; i < kFStages * 32 * kFT; i += blockDim.x) stage[i] = 0.0f;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (threadIdx.x < nbund * kFNB * 8) {  // Alg. 2 threshold masks of every (bundle, slot)
    const int b = threadIdx.x / (kFNB * 8), k = (threadIdx.x / 8) % kFNB, jb = threadIdx.x % 8;
    const int32_t c = bundles[b * kFNB + k];
    const int32_t kv = c >= 0 ? pol[c].k : 0x3F;
    s_km[b][k][jb] = ((kv >> jb) & 1) ? ~0u : 0u;
  }
  __syncthreads();
  if (sh_work[3] == 0 && wk.totals) {  // the launch's first CTA initialises the totals rows
    const int32_t rows = nbund * kFNB;
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
  const int32_t g = sh_work[2];
  if (threadIdx.x == 0) {
    if (unsigned long long* tr = trace_buf(wk)) {
      uint32_t smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      trace_put(tr, 0, gtimer());
      trace_put(tr, 4, smid);
      trace_put(tr, 5, (unsigned long long)s);
      trace_put(tr, 6, (unsigned long long)g);
    }
  }
  const int32_t cfirst = bundles[0];
  const DevPolicy P0 = pol[cfirst];
  const int W = P0.W;
  const int H = H_T > 0 ? H_T : P0.H;
  const int32_t t0 = wk.ts + (int32_t)(s * seg_len);
  const int32_t t1 = (int32_t)((t0 + seg_len < T) ? t0 + seg_len : T);
  const int32_t wt0 = t0 >> 5;
  const int32_t wend = (t1 + 31) >> 5;
  const int32_t ws = wk.ts >> 5;
  int32_t nhalo = (W + H - 1 + 31) / 32;
  if (nhalo > wt0 - (wk.tb >> 5)) nhalo = wt0 - (wk.tb >> 5);
  const int32_t w_first = wt0 - nhalo;
  const int32_t nwords = wend - w_first;
  const uint32_t stage_s = smem_u32(stage);
  const uint32_t mbuf_s = smem_u32(mbuf);

  // word j -> stage j % kFStages (issued by the first mask warp's lane 0)
  auto load_word = [&](int32_t j) {
    const int st = j % kFStages;
    mbar_expect_tx(&full_bar[st], kFStageBytes + 16u);
    tma_load_1d(st_mul[st], &tmul, &full_bar[st], 2 * (w_first + j));
    tma_load_2d(stage + st * 32 * kFT, &tmap, &full_bar[st], g * kFT, (int32_t)((w_first + j) * 32 - wk.tb));
  };

  if (warp >= nbund) {  // ---------------- mask warps ----------------
    const int m = warp - nbund;
    const float xthr_min = plat.xthr_min, xthr_max = plat.xthr_max;
    const double invB24_min = plat.invB24_min, invB24_max = plat.invB24_max;
    const int ni = NT > 0 ? NT : fam.ni, nd = NT > 0 ? NT : fam.nd;  // NT: compile-time threshold counts
    const bool issuer = m == 0 && lane == 0;
    if (issuer)
      for (int32_t j = 0; j < kFStages - 1 && j < nwords; ++j) load_word(j);
    int st = 0;
    uint32_t ph = 0;
    for (int32_t j = 0; j < nwords; ++j) {
      const int b = j % kMB;
      const uint32_t mb_s = mbuf_s + (uint32_t)(b * sizeof(MaskBuf));
      mbar_wait(&full_bar[st], ph);
      if (j >= kMB) mbar_wait(&mempty[b], ((uint32_t)(j / kMB) & 1u) ^ 1u);
      const int pst = st == 0 ? kFStages - 1 : st - 1;
      const uint32_t cur = stage_s + (uint32_t)(st * 32 * kFT * 4) + 4u * lane;
      const uint32_t prv = stage_s + (uint32_t)(pst * 32 * kFT * 4) + 4u * lane;
      float xv[8];
      double D[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int t = 8 * m + i;
        xv[i] = lds_f32(cur + 128u * (uint32_t)t);
        const int tl = t - (W - 1);  // Alg. 1 lag row (W <= 33: the previous word at most)
        const float xl = lds_f32(tl >= 0 ? cur + 128u * (uint32_t)tl : prv + 128u * (uint32_t)(tl + 32));
        D[i] = (double)xv[i] - (double)xl;  // Alg. 1 l.3 numerator (exact widening, RN difference)
      }
      const uint32_t byte_off = (uint32_t)m;
#pragma unroll(NT > 0 ? NT : 1)
      for (int ii = 0; ii < ni; ++ii) {
        const double d = fam.d_inc[ii];
        uint32_t by = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) or_if_gt(by, D[i], d, 1u << i);   // <=> RN(D / L) > tau_inc
        sts_u8(mb_s + (uint32_t)offsetof(MaskBuf, inc) + 128u * ii + 4u * lane + byte_off, by);
      }
#pragma unroll(NT > 0 ? NT : 1)
      for (int ii = 0; ii < nd; ++ii) {
        const double d = fam.d_dec[ii];
        uint32_t by = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) or_if_lt(by, D[i], d, 1u << i);   // <=> RN(D / L) < tau_dec
        sts_u8(mb_s + (uint32_t)offsetof(MaskBuf, dec) + 128u * ii + 4u * lane + byte_off, by);
      }
      uint32_t bmin = 0, bmax = 0;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        or_if_gt(bmin, xv[i], xthr_min, 1u << i);  // <=> RN(x / B_min) > 1
        or_if_gt(bmax, xv[i], xthr_max, 1u << i);  // <=> RN(x / B_max) > 1
      }
      sts_u8(mb_s + (uint32_t)offsetof(MaskBuf, smin) + 4u * lane + byte_off, bmin);
      sts_u8(mb_s + (uint32_t)offsetof(MaskBuf, xmx) + 4u * lane + byte_off, bmax);
      unsigned long long pl[8], plx[8];
      unsigned long long run = 0, runx = 0;
      if (bmax == 0) {  // no sample above the capacity at max: s24 < 127 * 2^24, no cap (branch-free)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const unsigned long long q = q_scaled_nocap(xv[i], invB24_min);
          run += ((bmin >> i) & 1u) ? q : 0ull;
          pl[i] = run;
        }
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          if ((bmin >> i) & 1u) run += q_scaled(xv[i], invB24_min);
          pl[i] = run;
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          if ((bmax >> i) & 1u) runx += q_scaled(xv[i], invB24_max);
          plx[i] = runx;
        }
      }
      sts_u64(mb_s + (uint32_t)offsetof(MaskBuf, tot) + 256u * m + 8u * lane, run);
      sts_u64(mb_s + (uint32_t)offsetof(MaskBuf, totx) + 256u * m + 8u * lane, runx);
      if (m == 0 && lane == 0) sts_u64(mb_s + (uint32_t)offsetof(MaskBuf, M), lds_u64(smem_u32(&st_mul[st][0])));
      bar_named(2, 32 * kMaskWarps);
      // every mask warp is past this word's samples and the previous word's
      // (its lag): the previous word's stage takes word j + kFStages - 1
      if (issuer && j + kFStages - 1 < nwords) load_word(j + kFStages - 1);
      // phase 2: the word's prefix sums, offset by the earlier bytes' totals
      const uint32_t sw = lds_u32(mb_s + (uint32_t)offsetof(MaskBuf, smin) + 4u * lane);
      if (sw) {
        unsigned long long off = 0;
        for (int q = 0; q < m; ++q) off += lds_u64v(mb_s + (uint32_t)offsetof(MaskBuf, tot) + 256u * q + 8u * lane);
#pragma unroll
        for (int i = 0; i < 8; ++i)
          sts_u64(mb_s + (uint32_t)offsetof(MaskBuf, P) + 256u * (8 * m + i) + 8u * lane, pl[i] + off);
      }
      const uint32_t xw = lds_u32(mb_s + (uint32_t)offsetof(MaskBuf, xmx) + 4u * lane);
      if (xw) {
        unsigned long long off = 0;
        for (int q = 0; q < m; ++q) off += lds_u64v(mb_s + (uint32_t)offsetof(MaskBuf, totx) + 256u * q + 8u * lane);
#pragma unroll
        for (int i = 0; i < 8; ++i)
          sts_u64(mb_s + (uint32_t)offsetof(MaskBuf, Px) + 256u * (8 * m + i) + 8u * lane,
                  (bmax ? plx[i] : 0ull) + off);
      }
      mbar_arrive(&mfull[b]);
      if (++st == kFStages) { st = 0; ph ^= 1u; }
    }
    return;
  }

  // ---------------- bundle warps: one trace x 4 configs per thread ----------------
  const int bw = warp;                 // bundle index in the family
  const int tidb = threadIdx.x;        // bundle-thread index (warps 0 .. nbund-1)
  const int64_t n = (int64_t)g * kFT + lane;
  const bool valid = n < N;
  int32_t cfg[kFNB];
#pragma unroll
  for (int k = 0; k < kFNB; ++k) cfg[k] = bundles[bw * kFNB + k];
  const int32_t c0 = cfg[0];
  const uint32_t inc_off = (uint32_t)offsetof(MaskBuf, inc) + 128u * fam.bi[bw] + 4u * lane;
  const uint32_t dec_off = (uint32_t)offsetof(MaskBuf, dec) + 128u * fam.bd[bw] + 4u * lane;
  uint32_t hypm = (s > 0) ? (1u << kFNB) - 1u : 0u;
  if (s == 0 && wk.carry && valid) {
#pragma unroll
    for (int k = 0; k < kFNB; ++k)
      if (cfg[k] >= 0) hypm |= (__ldg(wk.carry + (int64_t)cfg[k] * N + n) & 1u) << k;
  }
  // per-config hot state (16-bit packed counters: segments <= 65,504 steps)
  uint32_t cnt_a[kFNB], cnt_b[kFNB], cnt_c[kFNB];
  unsigned long long qmin[kFNB], dig[kFNB], pqmin[kFNB];
#pragma unroll
  for (int k = 0; k < kFNB; ++k) {
    cnt_a[k] = 0; cnt_b[k] = 0; cnt_c[k] = 0;
    qmin[k] = 0; dig[k] = 0; pqmin[k] = 0;
    FamSmem& S = FS(k, tidb);
    S.qmax = 0; S.pqmax = 0; S.pdig = 0; S.apos = -1; S.wa = -1; S.dwa = 0; S.pre_dec_a = 0;
  }
  uint32_t carry = hypm, seen = 0, va = 0;
  uint32_t Eprev = 0, ev = 0;
  // q_min / q_max summed over [t0, start of the current word) (the
  // carry-dependent prefix's stretch is G at its first action)
  unsigned long long Gb = 0, Gxb = 0;
  const bool want_dec = DEC && valid;
  uint64_t dec_row = want_dec ? reinterpret_cast<uint64_t>(wk.dec + (int64_t)c0 * wk.dec_cstride +
                                                           (int64_t)(wt0 - ws) * N + n)
                              : 0;
  const uint64_t dec_step = 4ull * (uint64_t)N;
  const uint32_t km_s = smem_u32(&s_km[bw][0][0]);
  const int32_t Ti = (int32_t)T;
  const int32_t w_tail = (Ti - 1) >> 5;
  const uint32_t tail_m = (Ti & 31) ? ((1u << (Ti & 31)) - 1u) : ~0u;

  for (int32_t j = 0; j < nwords; ++j) {
    const int b = j % kMB;
    const uint32_t mb_s = mbuf_s + (uint32_t)(b * sizeof(MaskBuf));
    mbar_wait(&mfull[b], (uint32_t)(j / kMB) & 1u);
    const int32_t w = w_first + j;
    const int32_t p0 = w * 32;
    const uint32_t incw = lds_u32(mb_s + inc_off), decw = lds_u32(mb_s + dec_off);
    const uint32_t warm = (p0 >= W) ? 0u : ((W - p0) >= 32 ? ~0u : ((1u << (W - p0)) - 1u));
    const uint32_t incv = incw & ~warm;          // p = +1
    const uint32_t decv = decw & ~warm & ~incv;  // p = -1 (line 4 before line 6)
    const uint32_t E = incv | decv;              // uncore_tune_ls.push_back(1)
    if (w >= wt0) {
      const uint32_t outm = (w == w_tail) ? tail_m : ~0u;
      // the position of the word's last decision: 31, or the trace's last interval
      const uint32_t lsh = (w == w_tail) ? (uint32_t)((Ti - 1) & 31) : 31u;
      const uint64_t M = lds_u64v(mb_s + (uint32_t)offsetof(MaskBuf, M));
      const uint32_t smin = lds_u32(mb_s + (uint32_t)offsetof(MaskBuf, smin) + 4u * lane);
      const uint32_t xmx = lds_u32(mb_s + (uint32_t)offsetof(MaskBuf, xmx) + 4u * lane);
      const uint32_t pcol = mb_s + (uint32_t)offsetof(MaskBuf, P) + 8u * lane;
      const uint32_t pxcol = mb_s + (uint32_t)offsetof(MaskBuf, Px) + 8u * lane;
      const unsigned long long Pw = smin ? lds_u64v(pcol + 256u * 31u) : 0ull;
      const unsigned long long Pxw = xmx ? lds_u64v(pxcol + 256u * 31u) : 0ull;
      ev += __popc(E & outm);
      uint32_t cnt[kNBits];
      Window<H_T>::count(E, Eprev, H, cnt);  // Alg. 2 (l.9), shared by the bundle
      // per config, branch-free: Alg. 2 >= k, Alg. 3 fill, counters, digest
      const uint32_t cin_w = carry, seen_w = seen;
      uint32_t Lvk[kFNB];
#pragma unroll
      for (int k = 0; k < kFNB; ++k) {
        const uint32_t ck = (cin_w >> k) & 1u;
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
        const uint32_t Dw = forward_fill(A, V, ck);
        const uint32_t Lv = (Dw << 1) | ck;          // interval level = dec[t-1]
        const uint32_t chm = (Dw ^ Lv) & outm;
        const uint32_t Dout = Dw & outm;
        cnt_a[k] += (uint32_t)__popc(HI & outm) | ((uint32_t)__popc(act & outm) << 16);
        cnt_b[k] += (uint32_t)__popc(Dout);   // (intervals at min: from the decisions, see the epilogue)
        cnt_c[k] += (uint32_t)__popc(chm);
        dig[k] += (unsigned long long)Dout * M;
        Lvk[k] = Lv;
        carry = (carry & ~(1u << k)) | (((Dw >> lsh) & 1u) << k);
        if constexpr (DEC) {  // words after the first action (earlier ones are deferred)
          if (valid && ((seen_w >> k) & 1u) && cfg[k] >= 0)
            reinterpret_cast<uint32_t*>(dec_row)[(int64_t)(cfg[k] - c0) * wk.dec_cstride] = Dout;
        }
      }
      if (seen_w != (1u << kFNB) - 1u) {  // some config has not acted yet in this segment (rare)
#pragma unroll
        for (int k = 0; k < kFNB; ++k) {
          if ((seen_w >> k) & 1u) continue;
          // the carry-dependent prefix (recomputed: off the common path)
          const uint32_t ck = (cin_w >> k) & 1u;
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
          const uint32_t A = HI | E | warm;
          const uint32_t V = decv & ~HI;
          const uint32_t Am = A & outm;
          uint32_t pre_dec;
          FamSmem& S = FS(k, tidb);
          if (Am) {
            const int i = __ffs(Am) - 1;
            seen |= 1u << k;
            va |= ((V >> i) & 1u) << k;
            pre_dec = (1u << i) - 1u;
            S.apos = (int32_t)(p0 + i - t0);
            S.wa = (int32_t)(w - wt0);
            S.dwa = forward_fill(A, V, ck) & outm;
            S.pre_dec_a = pre_dec;
            // stretch of the carry-dependent prefix [t0, first action]: G there
            pqmin[k] = Gb + (smin ? lds_u64v(pcol + 256u * (uint32_t)i) : 0ull);
            S.pqmax = Gxb + (xmx ? lds_u64v(pxcol + 256u * (uint32_t)i) : 0ull);
          } else {
            pre_dec = outm;
          }
          S.pdig += (unsigned long long)pre_dec * M;
        }
      }
      // model M stretch at min over the intervals run at min: sum of q over
      // Lv & smin (P is flat where smin is clear, and zero past T), one
      // shared load per run boundary
#pragma unroll
      for (int k = 0; k < kFNB; ++k) {
        const uint32_t lq = Lvk[k] & outm;
        if (lq & smin) qmin[k] += run_sum(forward_fill(smin, lq, 0u), pcol);
      }
      if (xmx) {  // some sample exceeds even the capacity at max (rare)
#pragma unroll
        for (int k = 0; k < kFNB; ++k) {
          const uint32_t lx = ~Lvk[k] & outm;
          if (lx & xmx) FS(k, tidb).qmax += run_sum(forward_fill(xmx, lx, 0u), pxcol);
        }
      }
      Gb += Pw;
      Gxb += Pxw;
      dec_row += dec_step;
    }
    Eprev = E;
    mbar_arrive(&mempty[b]);
  }

  // ---------------- epilogue: publish, look back, correct ----------------
  if (tidb == 0)
    if (unsigned long long* tr = trace_buf(wk)) trace_put(tr, 1, gtimer());
#pragma unroll
  for (int k = 0; k < kFNB; ++k) {
    const int32_t c = cfg[k];
    if (!valid || c < 0) continue;
    const uint32_t sk = (seen >> k) & 1u, last_min = (carry >> k) & 1u;
    uint32_t* status = wk.status + ((int64_t)c * nseg) * N + n;
    st_release(status + s * N, (wk.epoch << 3) | 1u | (sk << 1) | (last_min << 2));
  }
#pragma unroll
  for (int k = 0; k < kFNB; ++k) {
    const int32_t c = cfg[k];
    if (!valid || c < 0) continue;
    const bool sk = (seen >> k) & 1u;
    const FamSmem& S = FS(k, tidb);
    uint32_t* status = wk.status + ((int64_t)c * nseg) * N + n;
    const uint32_t hyp = (s > 0) ? 1u : (wk.carry ? (__ldg(wk.carry + (int64_t)c * N + n) & 1u) : 0u);
    uint32_t cin = hyp;
    if (s > 0) {
      cin = wk.carry ? (wk.carry[(int64_t)c * N + n] & 1u) : 0u;
      for (int64_t jj = s - 1; jj >= 0; --jj) {
        uint32_t v;
        while (((v = ld_acquire(status + jj * N)) >> 3) != wk.epoch) __nanosleep(MAGUS_LOOKBACK_SLEEP);
        if (v & 2u) { cin = (v >> 2) & 1u; break; }
      }
    }
    if (tidb == 0 && k == 0)
      if (unsigned long long* tr = trace_buf(wk)) trace_put(tr, 2, gtimer());
    if (wk.carry && s == nseg - 1)
      st_release(status + s * N, (wk.epoch << 3) | 3u | ((sk ? (carry >> k) & 1u : cin) << 2));
    uint32_t hi = cnt_a[k] & 0xFFFFu, msr = cnt_a[k] >> 16;
    uint32_t mdec = cnt_b[k];
    uint32_t ch = cnt_c[k];
    unsigned long long qn = qmin[k], qx = S.qmax, dg = dig[k];
    const unsigned long long pqn = sk ? pqmin[k] : Gb, pqx = sk ? S.pqmax : Gxb;  // no action: the whole segment
    if (cin != hyp) {
      const uint32_t n_dec = sk ? (uint32_t)S.apos : (uint32_t)(t1 - t0);
      if (hyp) {  // assumed min, truly max
        mdec -= n_dec;
        qn -= pqn; qx += pqx; dg -= S.pdig;
      } else {    // assumed max, truly min
        mdec += n_dec;
        qn += pqn; qx -= pqx; dg += S.pdig;
      }
      const uint32_t vak = (va >> k) & 1u;
      if (sk) ch += (uint32_t)((int)(vak != cin) - (int)(vak != hyp));
    }
    // intervals t0 .. t1-1 run at dec[t0-1] .. dec[t1-2]: the segment's min
    // decisions, plus the carry-in, minus its last decision (the hold of the
    // carry when nothing acted) -- the popcount of the interval mask, summed
    const uint32_t dlast = sk ? (carry >> k) & 1u : cin;
    const uint32_t mint = mdec + cin - dlast;
    if (want_dec) {  // deferred prefix decision words
      uint32_t* dec_out = wk.dec + (int64_t)c * wk.dec_cstride + n;
      const uint32_t fill = cin ? ~0u : 0u;
      const int32_t wlast = sk ? wt0 + S.wa : wend;
      for (int32_t w = wt0; w < wlast; ++w) dec_out[(w - ws) * N] = fill & tail_mask(w * 32, T);
      if (sk) dec_out[(wt0 + S.wa - ws) * N] = (S.dwa & ~S.pre_dec_a) | (fill & S.pre_dec_a);
    }
    unsigned long long* acc = wk.acc + (int64_t)c * kAccFields * N + n;
    atomicAdd(acc + 0 * N, (unsigned long long)ev);
    atomicAdd(acc + 1 * N, (unsigned long long)hi);
    atomicAdd(acc + 2 * N, (unsigned long long)msr);
    atomicAdd(acc + 3 * N, (unsigned long long)ch);
    atomicAdd(acc + 4 * N, (unsigned long long)mdec);
    atomicAdd(acc + 5 * N, (unsigned long long)mint);
    atomicAdd(acc + 6 * N, qn);
    atomicAdd(acc + 7 * N, qx);
    atomicAdd(acc + 8 * N, Gxb);  // q_base: q_max over every interval
    atomicAdd(acc + 9 * N, dg);
  }
  __threadfence();
  bar_named(1, nbt);
  if (tidb == 0) sh_last = (atomicAdd(wk.arrive + (int64_t)cfirst * ngroups + g, 1u) == (uint32_t)(nseg - 1));
  bar_named(1, nbt);
  if (sh_last) {  // every segment of this trace group is in: finalise its 32 traces x the family
    __threadfence();
#pragma unroll 1
    for (int k = 0; k < kFNB; ++k) {
      const int32_t c = cfg[k];
      if (c < 0) continue;  // uniform across the warp
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
        if (wk.carry)
          wk.carry[(int64_t)c * N + n] = (__ldcg(wk.status + ((int64_t)c * nseg + nseg - 1) * N + n) >> 2) & 1u;
        magus_summary sm_out;
        finalize_summary(plat, T, (int64_t)a[0], (int64_t)a[1], (int64_t)a[2], (int64_t)a[3], (int64_t)a[4],
                         (int64_t)a[5], a[6], a[7], a[8], a[9], (int64_t)a[10], (int64_t)a[11], &sm_out,
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
      if (wk.totals) {  // per-config fleet totals (exact integer sums): one warp = the group's 32 traces
#pragma unroll
        for (int q = 0; q < kTotAcc; ++q) {
          tv[q] = warp_sum_tot(tv[q], q);
        }
        if (lane == 0) {
          while (ld_acquire(wk.ticket + kTotalsFlagWord) == 0u) __nanosleep(MAGUS_LOOKBACK_SLEEP);
#pragma unroll
          for (int q = 0; q < kTotAcc; ++q) {
            const int word = q < 13 ? 1 + q : MAGUS_TOT_BURST_BASE + (q - 13);
            atomicAdd(reinterpret_cast<unsigned long long*>(wk.totals + (int64_t)c * MAGUS_TOT_WORDS + word), tv[q]);
          }
        }
      }
    }
    if (tidb == 0) wk.arrive[(int64_t)cfirst * ngroups + g] = 0;
  }
  // every bundle warp is past its totals (and their wait for the launch's
  // flag) before this CTA may be the one that re-arms the flag
  bar_named(1, nbt);
  if (tidb == 0) {
    if (unsigned long long* tr = trace_buf(wk)) {
      trace_put(tr, 3, gtimer());
      trace_put(tr, 7, sh_last);
    }
    __threadfence();
    if (atomicAdd(wk.done, 1u) == gridDim.x - 1) {  // the launch's last CTA re-arms the ticket
      *wk.ticket = 0;
      *wk.done = 0;
      wk.ticket[kTotalsFlagWord] = 0;
    }
  }
}

typedef void (*family_fn)(CUtensorMap, CUtensorMap, int64_t, int64_t, const DevPolicy*, const int32_t*,
                          DevPlatform, int64_t, int64_t, int32_t, int32_t, FamilyDev, StreamWork);

// DEC: decision words emitted (a compile-time flag: the sweeps emit none)
// NT = 4: the sweep grids' 4 tau_inc x 4 tau_dec thresholds, unrolled
family_fn pick_family(int32_t H, bool dec, int32_t ni, int32_t nd) {
  if (H == 10 && ni == 4 && nd == 4) return dec ? family_kernel<10, true, 4> : family_kernel<10, false, 4>;
  if (H == 10) return dec ? family_kernel<10, true, 0> : family_kernel<10, false, 0>;
  return dec ? family_kernel<0, true, 0> : family_kernel<0, false, 0>;
}

size_t family_smem(int32_t nbund) {
  return (size_t)kFStages * kFStageBytes + (size_t)kMB * sizeof(MaskBuf) +
         (size_t)kFNB * 32 * (size_t)nbund * sizeof(FamSmem);
}

}  // namespace

bool family_supported(int32_t W, int32_t H, int32_t NB, int32_t nbund, int32_t ni, int32_t nd) {
  return NB == kFNB && W >= 2 && W <= 33 && H >= 1 && H <= 32 && nbund >= 1 && nbund <= kFamMaxBund &&
         ni >= 1 && ni <= kFamMaxThr && nd >= 1 && nd <= kFamMaxThr;
}

int family_cta_traces() { return kFT; }

int family_ctas_per_sm(int32_t H, int32_t nbund) {
  family_fn f = pick_family(H, false, 4, 4);
  const size_t smem = family_smem(nbund);
  cudaFuncSetAttribute((const void*)f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, (const void*)f, 32 * (nbund + kMaskWarps), smem) !=
      cudaSuccess)
    return 0;
  return nb;
}

int launch_family(cudaStream_t st, const void* tmap32, const void* tmap_mul, int64_t N, int64_t T,
                  const DevPolicy* pol_dev, const int32_t* bundles_dev, int32_t nbund, int32_t H,
                  const FamilyDev& fam, const DevPlatform& plat, int64_t nseg, int64_t seg_len,
                  const StreamWork& wk, int* grid_out) {
  family_fn f = pick_family(H, wk.dec != nullptr, fam.ni, fam.nd);
  const size_t smem = family_smem(nbund);
  cudaFuncSetAttribute((const void*)f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  const int32_t ngroups = (int32_t)((N + kFT - 1) / kFT);
  const int64_t grid = (int64_t)ngroups * nseg;
  if (grid_out) *grid_out = (int)grid;
  const CUtensorMap* m = reinterpret_cast<const CUtensorMap*>(tmap32);
  const CUtensorMap* mm = reinterpret_cast<const CUtensorMap*>(tmap_mul);
  f<<<(unsigned)grid, 32 * (nbund + kMaskWarps), smem, st>>>(*m, *mm, N, T, pol_dev, bundles_dev, plat, nseg,
                                                                  seg_len, ngroups, nbund, fam, wk);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
