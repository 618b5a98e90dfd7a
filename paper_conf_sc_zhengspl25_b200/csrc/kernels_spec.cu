// kernels_spec.cu -- NEXT f3 (closed loop with the paper's jump rule) by
// speculative time segmentation.
//
// In the closed loop Alg. 1 observes the delivered throughput
// min(x_t, B(l_t)) (P@37360 / P@38709), so the state entering round t --
//   at_min  dec[t-1] == r_min (the level of interval t),
//   hist    the events of rounds t-H .. t-1 (uncore_tune_ls),
//   ring    the levels of intervals t-W+1 .. t-1 (their delivered samples
//           are still in the Alg. 1 window),
// -- depends on the whole past and no exact closed form segments it.  But
// the loop forgets: once the window's samples fit under the capacity at
// r_min, or a burst drives both histories to the same action, two runs
// from different states coincide.  So:
//   spec_kernel   one thread per (trace, segment, config): replay the R
//                 rounds before the segment from a guessed state (max, no
//                 events; exact when the run starts at t = 0), record the
//                 state reached at t0 (the speculation), replay the segment
//                 with full accounting into per-segment partial sums and
//                 outputs, record the final state;
//   spec_fix_kernel  one thread per (trace, config), in segment order: a
//                 segment whose speculated state equals the true state at
//                 its start (the exact final state of its predecessor) is
//                 exact -- the recurrence is deterministic -- and is
//                 accepted; otherwise it is replayed from the true state
//                 (rewriting its partials and outputs).  Then model M
//                 finalisation of the summed partials.
// Results are bit-identical to the sequential replay whatever the guess;
// only the amount of re-replay depends on how fast the loop forgets.
#include <algorithm>

#include "device_common.cuh"

namespace magus {
namespace {

constexpr int kSpecThreads = 128;
constexpr int kSpecChunk = 16;

enum { SF_EV, SF_HI, SF_MSR, SF_CH, SF_MDEC, SF_MINT, SF_QMIN, SF_QMAX, SF_QBASE, SF_DIG, SF_BB, SF_BM, kSpecFields };

struct SpecArgs {
  const float* x;
  int64_t N, ld;
  int32_t T, nw;
  const DevPolicy* pol;
  int32_t C, nseg, seg_len, warm;   // warm = R, the speculation's replay length
  unsigned long long* part;         // [C][nseg][kSpecFields][N]
  unsigned long long* s_hist;       // [C][nseg][N] speculated state at t0
  unsigned long long* s_ring;
  uint32_t* s_min;
  unsigned long long* f_hist;       // [C][nseg][N] state at t1 of the replay
  unsigned long long* f_ring;
  uint32_t* f_min;
  unsigned long long* g_hist;       // [C][nseg][N] the same after the retry pass
  unsigned long long* g_ring;
  uint32_t* g_min;
  magus_summary* summary;           // [C][N] (required)
  magus_base* base;                 // [N] or NULL
  uint32_t* dec;                    // [C][nw][N] or NULL
  uint8_t* levels;                  // [C][T][N] or NULL
  unsigned int* reruns;             // [1] segments replayed again (diagnostic)
};

template <typename ST>
struct SpecState {
  ST hist, ring;
  bool at_min;
};

struct SpecAcc {
  int32_t ev, hi, msr, ch, mdec, mint, bb, bm;
  unsigned long long qmin, qmax, qbase, dig;
};

// model-M / closed-loop constants of the platform (float thresholds are
// exact: x > fB <=> (double)x > B, x > xthr <=> RN(x * invB) > 1)
struct SpecPlat {
  double Bmin, Bmax, invB_min, invB_max;
  float fBmin, fBmax, xthr_min, xthr_max, xburst;
  int32_t bursts, min_keeps, r_min, r_max;
};

// Rounds [ta, tb) of trace n under config P from state st.  ACCT: meter
// model M, write outputs and accumulate (ta is then 32-aligned).  ST: the
// hist / ring shift registers (32-bit when H <= 32 and W <= 33).
template <bool ACCT, typename ST>
__device__ __forceinline__ void spec_run(const SpecArgs& a, const SpecPlat& sp, const DevPolicy& P, int32_t c,
                                         int64_t n, int32_t ta, int32_t tb, SpecState<ST>& st, SpecAcc& acc) {
  constexpr int kBits = 8 * (int)sizeof(ST);
  const ST hmask = P.H >= kBits ? (ST)~(ST)0 : (ST)(((ST)1 << P.H) - 1);
  const ST rmask = P.W - 1 >= kBits ? (ST)~(ST)0 : (ST)(((ST)1 << (P.W - 1)) - 1);
  const int sh = P.W - 2;           // ring bit of interval t-W+1 at round t
  uint32_t word = 0, half = 0;
  // one round t (i: its position in the chunk)
  auto round = [&](int i, int32_t t, float x, float xl) {
    const bool lm = st.at_min;      // interval t runs at dec[t-1] (reading R6)
    bool nm = lm;
    if (t >= P.W) {                 // MDFS rounds start at t = W (reading R5)
      // delivered throughput of interval t and of the lag interval (f3)
      const bool lmin = (st.ring >> sh) & 1;
      const bool ct = x > (lm ? sp.fBmin : sp.fBmax), cl = xl > (lmin ? sp.fBmin : sp.fBmax);
      const double yt = ct ? (lm ? sp.Bmin : sp.Bmax) : (double)x;
      const double yl = cl ? (lmin ? sp.Bmin : sp.Bmax) : (double)xl;
      const uint32_t hf = (__popc((uint32_t)st.hist) +
                           (kBits > 32 ? __popc((uint32_t)((uint64_t)st.hist >> 32)) : 0)) >= P.k ? 1u : 0u;
      const double D = yt - yl;     // Alg. 1 (host-inverted thresholds)
      const uint32_t pi = D > P.d_inc ? 1u : 0u;
      const uint32_t pd = (pi == 0u && D < P.d_dec) ? 1u : 0u;
      // l.10 / l.18-19: uncore_freq <- upper; l.23-25: <- lower (jump); else hold.
      // (Integer masks throughout: bool if/else and ternary forms of this
      // select gave wrong decisions and counts in this lambda under nvcc
      // 12.9 -- reproduced with device printf: pd = 1, nm unchanged.)
      const uint32_t ev = pi | pd, up = hf | pi;
      nm = ((up ^ 1u) & (pd | (uint32_t)lm)) != 0u;
      st.hist = (ST)(((st.hist << 1) | (ST)ev) & hmask);
      if (ACCT) {
        acc.ev += (int32_t)ev;
        acc.hi += (int32_t)hf;
        acc.msr += (int32_t)(hf | ev);
      }
    }
    st.ring = (ST)(((st.ring << 1) | (ST)lm) & rmask);
    if (ACCT) {
      acc.mint += lm;
      if (x > (lm ? sp.xthr_min : sp.xthr_max)) {   // stretch at dec[t-1] (sparse)
        if (lm) acc.qmin += q_literal(x, sp.invB_min);
        else acc.qmax += q_literal(x, sp.invB_max);
      }
      if (x > sp.xthr_max) acc.qbase += q_literal(x, sp.invB_max);
      if (sp.bursts && x > sp.xburst) {
        ++acc.bb;
        acc.bm += lm ? sp.min_keeps : 1;
      }
      acc.ch += (t >= 1 && nm != lm);
      half |= (uint32_t)nm << i;
      if (a.levels) a.levels[((int64_t)c * a.T + t) * a.N + n] = (uint8_t)(nm ? sp.r_min : sp.r_max);
    }
    st.at_min = nm;
  };
  auto flush = [&](int32_t t_last) {  // the word holding interval t_last is complete
    const int64_t w = t_last >> 5;
    acc.mdec += __popc(word);
    if (a.dec) a.dec[((int64_t)c * a.nw + w) * a.N + n] = word;
    acc.dig += (unsigned long long)word * digest_mul(w);
    word = 0;
  };
  // samples and lags of the next chunk are loaded while this one is replayed
  float nxs[kSpecChunk], nxl[kSpecChunk];
  const int ld32 = (int)a.ld;
  auto load = [&](int32_t tc) {
    const float* px = a.x + (int64_t)tc * a.ld + n;
    if (tc >= P.W && tc + kSpecChunk <= tb) {
      const float* pl = px - (int64_t)(P.W - 1) * a.ld;
#pragma unroll
      for (int i = 0; i < kSpecChunk; ++i) {
        nxs[i] = __ldg(px + i * ld32);
        nxl[i] = __ldg(pl + i * ld32);
      }
    } else {
#pragma unroll
      for (int i = 0; i < kSpecChunk; ++i) {
        const int32_t t = tc + i;
        nxs[i] = t < tb ? __ldg(a.x + (int64_t)t * a.ld + n) : 0.0f;
        nxl[i] = (t < tb && t >= P.W) ? __ldg(a.x + (int64_t)(t - P.W + 1) * a.ld + n) : 0.0f;
      }
    }
  };
  if (ta < tb) load(ta);
  for (int32_t tc = ta; tc < tb; tc += kSpecChunk) {
    float xs[kSpecChunk], xl[kSpecChunk];
#pragma unroll
    for (int i = 0; i < kSpecChunk; ++i) {
      xs[i] = nxs[i];
      xl[i] = nxl[i];
    }
    const int rem = min(kSpecChunk, tb - tc);
    if (tc + kSpecChunk < tb) load(tc + kSpecChunk);
    half = 0;
    if (rem == kSpecChunk) {
#pragma unroll
      for (int i = 0; i < kSpecChunk; ++i) round(i, tc + i, xs[i], xl[i]);
    } else {
      for (int i = 0; i < rem; ++i) round(i, tc + i, xs[i], xl[i]);
    }
    if (ACCT) {                     // ta is 32-aligned: a chunk is one half of a word
      word |= half << ((tc - ta) & 16);
      if (((tc - ta) & 16) || tc + kSpecChunk >= tb) flush(tc + rem - 1);
    }
  }
}

__device__ __forceinline__ void store_part(const SpecArgs& a, int32_t c, int32_t s, int64_t n, const SpecAcc& acc) {
  unsigned long long* p = a.part + ((int64_t)c * a.nseg + s) * kSpecFields * a.N + n;
  const unsigned long long v[kSpecFields] = {
      (unsigned long long)acc.ev, (unsigned long long)acc.hi, (unsigned long long)acc.msr,
      (unsigned long long)acc.ch, (unsigned long long)acc.mdec, (unsigned long long)acc.mint,
      acc.qmin, acc.qmax, acc.qbase, acc.dig, (unsigned long long)acc.bb, (unsigned long long)acc.bm};
#pragma unroll
  for (int f = 0; f < kSpecFields; ++f) p[(int64_t)f * a.N] = v[f];
}

template <typename ST>
__global__ void __launch_bounds__(kSpecThreads, 4) spec_kernel(SpecArgs a, SpecPlat sp) {
  const int64_t n = (int64_t)blockIdx.x * kSpecThreads + threadIdx.x;
  const int32_t s = blockIdx.y, c = blockIdx.z;
  if (n >= a.N) return;
  const DevPolicy P = a.pol[c];
  const int32_t t0 = s * a.seg_len, t1 = min(a.T, t0 + a.seg_len);
  SpecState<ST> st{0, 0, false};    // the state at t = 0 (max, H zeros); the guess otherwise
  SpecAcc acc{};
  const int32_t ts = max(0, t0 - a.warm);
  spec_run<false>(a, sp, P, c, n, ts, t0, st, acc);
  const int64_t ix = ((int64_t)c * a.nseg + s) * a.N + n;
  a.s_hist[ix] = (unsigned long long)st.hist;
  a.s_ring[ix] = (unsigned long long)st.ring;
  a.s_min[ix] = st.at_min | (ts == 0 ? 2u : 0u);  // bit 1: exact (the run started at t = 0)
  spec_run<true>(a, sp, P, c, n, t0, t1, st, acc);
  store_part(a, c, s, n, acc);
  a.f_hist[ix] = (unsigned long long)st.hist;
  a.f_ring[ix] = (unsigned long long)st.ring;
  a.f_min[ix] = st.at_min;
}

// One parallel retry pass: a segment whose speculation differs from its
// predecessor's (speculative) final state is replayed from that state.  An
// isolated miss -- predecessor right, this guess wrong -- becomes exact
// here instead of in the sequential fix pass.  Reads f_*, writes g_* (and
// the segment's speculation, partials and outputs when it replays).
template <typename ST>
__global__ void __launch_bounds__(kSpecThreads, 4) spec_retry_kernel(SpecArgs a, SpecPlat sp) {
  const int64_t n = (int64_t)blockIdx.x * kSpecThreads + threadIdx.x;
  const int32_t s = blockIdx.y, c = blockIdx.z;
  if (n >= a.N) return;
  const int64_t ix = ((int64_t)c * a.nseg + s) * a.N + n;
  const uint32_t sm = a.s_min[ix];
  bool same = s == 0 || (sm & 2u);
  SpecState<ST> st{0, 0, false};
  if (!same) {
    const int64_t ip = ix - a.N;      // segment s - 1
    st.hist = (ST)a.f_hist[ip];
    st.ring = (ST)a.f_ring[ip];
    st.at_min = a.f_min[ip] != 0;
    same = (ST)a.s_hist[ix] == st.hist && (ST)a.s_ring[ix] == st.ring && ((sm & 1u) != 0) == st.at_min;
  }
  if (same) {
    a.g_hist[ix] = a.f_hist[ix];
    a.g_ring[ix] = a.f_ring[ix];
    a.g_min[ix] = a.f_min[ix];
    return;
  }
  a.s_hist[ix] = (unsigned long long)st.hist;  // the new speculation
  a.s_ring[ix] = (unsigned long long)st.ring;
  a.s_min[ix] = st.at_min;
  const DevPolicy P = a.pol[c];
  const int32_t t0 = s * a.seg_len, t1 = min(a.T, t0 + a.seg_len);
  SpecAcc acc{};
  spec_run<true>(a, sp, P, c, n, t0, t1, st, acc);
  store_part(a, c, s, n, acc);
  a.g_hist[ix] = (unsigned long long)st.hist;
  a.g_ring[ix] = (unsigned long long)st.ring;
  a.g_min[ix] = st.at_min;
}

template <typename ST>
__global__ void __launch_bounds__(kSpecThreads) spec_fix_kernel(SpecArgs a, SpecPlat sp, DevPlatform plat) {
  const int64_t gid = (int64_t)blockIdx.x * kSpecThreads + threadIdx.x;
  if (gid >= a.N * a.C) return;
  const int32_t c = (int32_t)(gid / a.N);
  const int64_t n = gid - (int64_t)c * a.N;
  const DevPolicy P = a.pol[c];
  const int64_t i0 = (int64_t)c * a.nseg * a.N + n;  // segment 0 is exact
  SpecState<ST> tr{(ST)a.g_hist[i0], (ST)a.g_ring[i0], a.g_min[i0] != 0};
  unsigned int reruns = 0;
  for (int32_t s = 1; s < a.nseg; ++s) {
    const int64_t ix = ((int64_t)c * a.nseg + s) * a.N + n;
    const uint32_t sm = a.s_min[ix];
    const bool ok = (sm & 2u) || ((ST)a.s_hist[ix] == tr.hist && (ST)a.s_ring[ix] == tr.ring &&
                                  ((sm & 1u) != 0) == tr.at_min);
    if (ok) {
      tr.hist = (ST)a.g_hist[ix];
      tr.ring = (ST)a.g_ring[ix];
      tr.at_min = a.g_min[ix] != 0;
    } else {                          // replay the segment from the true state
      const int32_t t0 = s * a.seg_len, t1 = min(a.T, t0 + a.seg_len);
      SpecAcc acc{};
      spec_run<true>(a, sp, P, c, n, t0, t1, tr, acc);
      store_part(a, c, s, n, acc);
      ++reruns;
    }
  }
  if (reruns && a.reruns) atomicAdd(a.reruns, reruns);
  // sum the partials (integers: exact in any order) and finalise model M
  unsigned long long v[kSpecFields];
#pragma unroll
  for (int f = 0; f < kSpecFields; ++f) v[f] = 0ull;
  for (int32_t s = 0; s < a.nseg; ++s) {
    const unsigned long long* p = a.part + ((int64_t)c * a.nseg + s) * kSpecFields * a.N + n;
#pragma unroll
    for (int f = 0; f < kSpecFields; ++f) v[f] += p[(int64_t)f * a.N];
  }
  finalize_summary(plat, a.T, (int64_t)v[SF_EV], (int64_t)v[SF_HI], (int64_t)v[SF_MSR], (int64_t)v[SF_CH],
                   (int64_t)v[SF_MDEC], (int64_t)v[SF_MINT], v[SF_QMIN], v[SF_QMAX], v[SF_QBASE], v[SF_DIG],
                   (int64_t)v[SF_BB], (int64_t)v[SF_BM], a.summary + gid, (a.base && c == 0) ? a.base + n : nullptr);
}

}  // namespace

bool spec_supported(const magus_policy& p) {
  return p.variant == MAGUS_VARIANT_CLOSED_LOOP && p.window <= 65;
}

size_t spec_scratch_bytes(int64_t N, int32_t C, int64_t nseg) {
  auto al = [](size_t b) { return (b + 255) / 256 * 256; };
  const size_t cs = (size_t)C * nseg * N;
  return al(8 * cs * kSpecFields) + 6 * al(8 * cs) + 3 * al(4 * cs) + 256;
}

int launch_spec(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld, const DevPolicy* pol_dev,
                int32_t C, bool wide, const DevPlatform& plat, int64_t nseg, int64_t seg_len, int64_t warm, void* scratch,
                magus_summary* out_summary, magus_base* out_base, uint32_t* out_dec, uint8_t* out_levels,
                unsigned int** reruns_out) {
  auto al = [](size_t b) { return (b + 255) / 256 * 256; };
  const size_t cs = (size_t)C * nseg * N;
  char* sc = (char*)scratch;
  SpecArgs a;
  a.x = x;
  a.N = N;
  a.ld = ld;
  a.T = (int32_t)T;
  a.nw = (int32_t)((T + 31) / 32);
  a.pol = pol_dev;
  a.C = C;
  a.nseg = (int32_t)nseg;
  a.seg_len = (int32_t)seg_len;
  a.warm = (int32_t)warm;
  a.part = (unsigned long long*)sc;
  sc += al(8 * cs * kSpecFields);
  a.s_hist = (unsigned long long*)sc;
  sc += al(8 * cs);
  a.s_ring = (unsigned long long*)sc;
  sc += al(8 * cs);
  a.f_hist = (unsigned long long*)sc;
  sc += al(8 * cs);
  a.f_ring = (unsigned long long*)sc;
  sc += al(8 * cs);
  a.s_min = (uint32_t*)sc;
  sc += al(4 * cs);
  a.f_min = (uint32_t*)sc;
  sc += al(4 * cs);
  a.g_hist = (unsigned long long*)sc;
  sc += al(8 * cs);
  a.g_ring = (unsigned long long*)sc;
  sc += al(8 * cs);
  a.g_min = (uint32_t*)sc;
  sc += al(4 * cs);
  a.reruns = (unsigned int*)sc;
  if (reruns_out) *reruns_out = a.reruns;
  a.summary = out_summary;
  a.base = out_base;
  a.dec = out_dec;
  a.levels = out_levels;
  if (cudaMemsetAsync(a.reruns, 0, sizeof(unsigned int), s) != cudaSuccess) return -1;
  SpecPlat sp;
  sp.Bmin = plat.Bmin;
  sp.Bmax = plat.Bmax;
  sp.invB_min = plat.invB_min;
  sp.invB_max = plat.invB_max;
  sp.fBmin = above_threshold(plat.Bmin);  // largest float f with !((double)f > B)
  sp.fBmax = above_threshold(plat.Bmax);
  sp.xthr_min = plat.xthr_min;
  sp.xthr_max = plat.xthr_max;
  sp.xburst = plat.xburst;
  sp.bursts = plat.burst_on;
  sp.min_keeps = plat.burst_min_keeps;
  sp.r_min = plat.r_min;
  sp.r_max = plat.r_max;
  const dim3 grid((unsigned)((N + kSpecThreads - 1) / kSpecThreads), (unsigned)nseg, (unsigned)C);
  const unsigned fb = (unsigned)((N * C + kSpecThreads - 1) / kSpecThreads);
  if (wide) {
    spec_kernel<uint64_t><<<grid, kSpecThreads, 0, s>>>(a, sp);
    spec_retry_kernel<uint64_t><<<grid, kSpecThreads, 0, s>>>(a, sp);
    spec_fix_kernel<uint64_t><<<fb, kSpecThreads, 0, s>>>(a, sp, plat);
  } else {
    spec_kernel<uint32_t><<<grid, kSpecThreads, 0, s>>>(a, sp);
    spec_retry_kernel<uint32_t><<<grid, kSpecThreads, 0, s>>>(a, sp);
    spec_fix_kernel<uint32_t><<<fb, kSpecThreads, 0, s>>>(a, sp, plat);
  }
  return cudaGetLastError() == cudaSuccess ? 3 : -1;
}

}  // namespace magus
