/*
 * oracle.h -- types of the CPU ORACLE (test infrastructure; see
 * magus_oracle.cpp).  Deliberately NOT include/magus.h: the oracle and the
 * CUDA path share no headers.  The Python test harness marshals between the
 * two field by field.
 */
#ifndef MAGUS_ORACLE_H_
#define MAGUS_ORACLE_H_
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int32_t W;        /* |mem_throughput_ls|                     */
  int32_t H;        /* |uncore_tune_ls|                        */
  double L;         /* direv_length                            */
  double tau_inc;   /* inc_threshold                           */
  double tau_dec;   /* dec_threshold (signed)                  */
  double t_hi;      /* high_freq_threshold                     */
  int32_t variant;  /* 0 paper; 1 closed loop (f3); 2 gradual step (f4) */
  int32_t step;     /* ratio step of the gradual variant       */
} or_policy;

typedef struct {
  int32_t r_min, r_max;
  double dt, bw_max, beta, p_other, p_unc_min, p_unc_max, e_sw, t_sw, bound;
  double burst;   /* Sec. 6.3 burst threshold theta (<= 0: not counted) */
} or_platform;

typedef struct {
  int64_t n_events, n_hi_rounds, n_msr_writes, n_changes, n_min_dec, n_min_int;
  uint64_t q_min, q_max, digest;
  double time, energy, slowdown;
  int32_t viol, reserved;
  int64_t n_burst_base;   /* |B|: bursts of the max-uncore run        */
  int64_t n_burst_magus;  /* |A|: bursts of the MAGUS run             */
  int64_t n_burst_inter;  /* |A and B|                                */
  int64_t n_burst_union;  /* |A or B|                                 */
} or_summary;

typedef struct {
  uint64_t q_base;
  double time, energy;
  uint64_t reserved;
} or_base;

#ifdef __cplusplus
}
#endif
#endif
