/*
 * magus_gen.h -- seeded synthetic memory-throughput traces (INPUT GENERATOR).
 *
 * This is the one module shared by the CUDA path and the oracle's tests: it
 * produces inputs only and contains none of the method's arithmetic (no
 * Alg. 1-3, no accounting).  It is integer-exact (splitmix64 + integer
 * arithmetic, no libm, no floating point until the final exact int->float
 * store), so the host build (gen/gen_host.c, gcc) and the device build
 * (libmagus, nvcc) emit bit-identical traces.
 *
 * Shape (recipe in DESIGN.md section 5; an assumption modelled on the paper's
 * GPU-dominant workloads, P@28128-P@28927 Sec. 5):
 *   class mix  ALTIS-like 40 % | ML-training 30 % | MD 15 % | SRAD-like 15 %
 *   levels     compute/idle U[200,1500], transfer burst U[8000,24000],
 *              CPU-prep U[2000,8000]  (integer MB/s)
 *   phases     COMPUTE (geometric dwell, mean 100/20/250/40 by class),
 *              BURST (mean 2, widths 1..~8 straddle the k=4 and W-1=9
 *              boundaries), PREP (mean 10), OSC (SRAD's rapid oscillation,
 *              P@38243 / P@40055: alternate idle/burst every 1-2 samples,
 *              mean 15 samples ~ 3 s)
 *   noise      v = L + L*((u mod 2001) - 1000)/20000 + (u' mod 64)
 *              (+-5 % multiplicative, up to 63 MB/s additive), clamped to
 *              [0, 2^24-1] so the fp32 store is exact.
 *   adversarial (kind 1): 80 % square-wave oscillation with periods
 *              {2,4,3,9} (3 and 9 divide W-1 = 9: the lag blind spot) at
 *              amplitudes {2000,2001,5000,5001} (exact Alg. 1 ties at the
 *              paper defaults), 20 % isolated bursts of width {2,3,4,5};
 *              no noise.
 * One sample = one 0.2 s interval (P@44789).
 */
#ifndef MAGUS_GEN_H_
#define MAGUS_GEN_H_

#include <stdint.h>

#if defined(__CUDACC__)
#define MG_HD __host__ __device__ __forceinline__
#else
#define MG_HD static inline
#endif

#define MG_GOLDEN 0x9E3779B97F4A7C15ULL

enum { MG_KIND_MIX = 0, MG_KIND_ADVERSARIAL = 1 };
enum { MG_CLS_ALTIS = 0, MG_CLS_ML = 1, MG_CLS_MD = 2, MG_CLS_SRAD = 3,
       MG_CLS_ADV_OSC = 4, MG_CLS_ADV_BURST = 5 };
enum { MG_ST_COMPUTE = 0, MG_ST_BURST = 1, MG_ST_PREP = 2, MG_ST_OSC = 3 };

typedef struct {
  uint64_t s;        /* splitmix64 state                                   */
  int32_t cls;       /* class                                              */
  int32_t st;        /* phase state                                        */
  int32_t lv_idle, lv_burst, lv_prep;
  int32_t period;    /* ML loader period / adversarial wave period         */
  int32_t ctr;       /* samples since the phase (or period) started        */
  int32_t osc_hi;    /* OSC: currently on the high half                    */
  int32_t osc_left;  /* OSC: samples left on this half                     */
  int32_t amp;       /* adversarial amplitude                              */
  int32_t width;     /* adversarial burst width / ML burst width           */
  int32_t gap;       /* adversarial gap before the next burst              */
  int32_t noise;     /* 1 = add sampling noise                             */
} mg_state;

MG_HD uint64_t mg_next(uint64_t* s) {
  uint64_t z = (*s += MG_GOLDEN);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

/* uniform integer in [lo, hi] (modulo draw; the bias is part of the recipe) */
MG_HD int32_t mg_uniform(uint64_t* s, int32_t lo, int32_t hi) {
  return lo + (int32_t)(mg_next(s) % (uint64_t)(hi - lo + 1));
}

MG_HD void mg_init(mg_state* g, uint64_t seed, int64_t global_id, int32_t kind) {
  g->s = seed ^ ((uint64_t)(global_id + 1) * MG_GOLDEN);
  g->lv_idle = mg_uniform(&g->s, 200, 1500);
  g->lv_burst = mg_uniform(&g->s, 8000, 24000);
  g->lv_prep = mg_uniform(&g->s, 2000, 8000);
  g->ctr = 0;
  g->osc_hi = 0;
  g->osc_left = 1;
  g->width = 2;
  g->gap = 10;
  g->noise = 1;
  if (kind == MG_KIND_ADVERSARIAL) {
    const int32_t amps[4] = {2000, 2001, 5000, 5001};
    const int32_t pers[4] = {2, 4, 3, 9};
    g->noise = 0;
    g->cls = (mg_next(&g->s) % 10u) < 8u ? MG_CLS_ADV_OSC : MG_CLS_ADV_BURST;
    g->amp = amps[mg_next(&g->s) & 3u];
    g->period = pers[mg_next(&g->s) & 3u];
    g->st = MG_ST_COMPUTE;
    g->gap = mg_uniform(&g->s, 10, 30);
    g->width = 2 + (int32_t)(mg_next(&g->s) & 3u);
    g->lv_burst = g->lv_idle + g->amp;
    return;
  }
  {
    uint32_t c = (uint32_t)(mg_next(&g->s) % 100u);
    g->cls = c < 40u ? MG_CLS_ALTIS : c < 70u ? MG_CLS_ML : c < 85u ? MG_CLS_MD : MG_CLS_SRAD;
  }
  g->period = mg_uniform(&g->s, 5, 50);
  /* ALTIS-like apps open with the host->device transfer burst */
  g->st = (g->cls == MG_CLS_ALTIS) ? MG_ST_BURST : MG_ST_COMPUTE;
  g->amp = 0;
}

/* leave the current phase with probability 1/mean (geometric dwell) */
MG_HD int mg_leave(uint64_t u, uint32_t mean) { return (uint32_t)((u >> 32) % mean) == 0u; }

/* Emits one sample (integer MB/s) and advances the phase machine. */
MG_HD int32_t mg_step(mg_state* g) {
  uint64_t u = mg_next(&g->s);
  int32_t level;
  /* ----- value of the current phase ----- */
  if (g->cls == MG_CLS_ADV_OSC) {
    /* square wave: high for ceil(P/2), low for floor(P/2) samples */
    int32_t hi_len = (g->period + 1) / 2;
    level = (g->ctr < hi_len) ? g->lv_burst : g->lv_idle;
    g->ctr = (g->ctr + 1) % g->period;
    /* 1/64 chance per sample to re-draw the period (keeps all four mixed) */
    if (((u >> 40) & 63u) == 0u) {
      const int32_t pers[4] = {2, 4, 3, 9};
      g->period = pers[(u >> 50) & 3u];
      g->ctr = 0;
    }
    return level;
  }
  if (g->cls == MG_CLS_ADV_BURST) {
    if (g->st == MG_ST_BURST) {
      level = g->lv_burst;
      if (++g->ctr >= g->width) {
        g->st = MG_ST_COMPUTE; g->ctr = 0;
        g->gap = 10 + (int32_t)((u >> 32) % 21u);
      }
    } else {
      level = g->lv_idle;
      if (++g->ctr >= g->gap) {
        g->st = MG_ST_BURST; g->ctr = 0;
        g->width = 2 + (int32_t)((u >> 48) & 3u);
      }
    }
    return level;
  }
  switch (g->st) {
    case MG_ST_BURST: level = g->lv_burst; break;
    case MG_ST_PREP: level = g->lv_prep; break;
    case MG_ST_OSC: level = g->osc_hi ? g->lv_burst : g->lv_idle; break;
    default: level = g->lv_idle; break;
  }
  {
    int64_t v = level;
    if (g->noise) {
      int64_t m = (int64_t)(u % 2001u) - 1000;
      v = v + (v * m) / 20000 + (int64_t)((u >> 16) & 63u);
    }
    if (v < 0) v = 0;
    if (v > 16777215) v = 16777215;
    level = (int32_t)v;
  }
  /* ----- phase transition after this sample ----- */
  g->ctr++;
  switch (g->cls) {
    case MG_CLS_ALTIS:
      if (g->st == MG_ST_COMPUTE) {
        if (mg_leave(u, 100u)) { g->st = ((u >> 20) & 1u) ? MG_ST_BURST : MG_ST_PREP; g->ctr = 0; }
      } else if (g->st == MG_ST_BURST) {
        if (mg_leave(u, 2u)) { g->st = MG_ST_COMPUTE; g->ctr = 0; }
      } else {
        if (mg_leave(u, 10u)) { g->st = MG_ST_COMPUTE; g->ctr = 0; }
      }
      break;
    case MG_CLS_ML:
      /* data-loader burst every `period` samples, jitter -1/0/+1 */
      if (g->st == MG_ST_COMPUTE) {
        int32_t jit = (int32_t)((u >> 21) % 3u) - 1;
        if (g->ctr >= g->period + jit) {
          g->st = MG_ST_BURST; g->ctr = 0; g->width = 1 + (int32_t)((u >> 24) % 3u);
        } else if (((u >> 32) % 200u) == 0u) {
          g->st = MG_ST_PREP; g->ctr = 0;
        }
      } else if (g->st == MG_ST_BURST) {
        if (g->ctr >= g->width) { g->st = MG_ST_COMPUTE; g->ctr = 0; }
      } else {
        if (mg_leave(u, 10u)) { g->st = MG_ST_COMPUTE; g->ctr = 0; }
      }
      break;
    case MG_CLS_MD:
      if (g->st == MG_ST_COMPUTE) {
        if (mg_leave(u, 250u)) { g->st = MG_ST_BURST; g->ctr = 0; }
      } else {
        if (mg_leave(u, 2u)) { g->st = MG_ST_COMPUTE; g->ctr = 0; }
      }
      break;
    default: /* SRAD-like */
      if (g->st == MG_ST_COMPUTE) {
        if (mg_leave(u, 40u)) { g->st = MG_ST_OSC; g->ctr = 0; g->osc_hi = 1; g->osc_left = 1 + (int32_t)((u >> 20) & 1u); }
      } else {
        if (--g->osc_left <= 0) { g->osc_hi ^= 1; g->osc_left = 1 + (int32_t)((u >> 20) & 1u); }
        if (mg_leave(u, 15u)) { g->st = MG_ST_COMPUTE; g->ctr = 0; }
      }
      break;
  }
  return level;
}

#endif /* MAGUS_GEN_H_ */
