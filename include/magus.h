/*
 * magus.h -- C-ABI of libmagus: a B200 (sm_100a) batch replay of the MAGUS
 * uncore-frequency decision loop (Zheng, Sultanov, Papka, Lan, "Minimizing
 * Power Waste in Heterogenous Computing via Adaptive Uncore Scaling", SC'25).
 *
 * Citations are P@<byte offset> into the paper text (PAPER.md is one line, so
 * a byte offset is the only precise locator), plus the section / algorithm.
 *
 *   Alg. 1  Memory Throughput Trend Prediction ........ P@20631 (Sec. 3.1)
 *   Alg. 2  High Frequency Detection ................... P@21063 (Sec. 3.2)
 *   Alg. 3  MDFS (combination + step rule) ............. P@25445 (Sec. 3.3)
 *   init: uncore at max, 10-cycle fill, tune list = 10 zeros
 *                                              P@23755, P@23939, P@24182
 *   default thresholds 200 / 500 / 0.4, 0.2 s ........... P@25197 (Sec. 3.3)
 *   Pareto default 300 / 500 / 0.4 ...................... P@44170 (Sec. 6.4)
 *
 * Readings of the paper that the library implements (all listed with their
 * reasons in DESIGN.md section 3): dec_threshold is signed (-500); the first
 * MDFS round is t = W; Alg. 3's garbled lines 12-14 are "else status <- 0";
 * a decision made after sample t governs interval t+1; open loop.
 *
 * The energy / slowdown accounting ("model M") is an
 * ASSUMPTION: the paper measures energy with RAPL/NVML (P@31772) and does not
 * model it.
 *
 * Conventions for every call:
 *   - Returns magus_status; MAGUS_OK == 0.
 *   - All arguments are validated before anything is launched.  On error no
 *     output is written and magus_last_error(ctx) holds a one-line reason.
 *   - Device pointers are raw CUDA device addresses owned by the caller (the
 *     Python binding allocates them through torch).  The library never frees
 *     caller memory.  The context owns its scratch memory (grown on demand,
 *     freed by magus_destroy).
 *   - The CUDA stream given to magus_init (or magus_set_stream) is borrowed;
 *     device work is enqueued on it asynchronously.  Calls that return host
 *     values synchronise that stream and say so.
 *   - One context per host thread.
 */
#ifndef MAGUS_H_
#define MAGUS_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MAGUS_ABI_VERSION 1

typedef struct magus_ctx_s* magus_ctx;

typedef enum {
  MAGUS_OK = 0,
  MAGUS_ERR_INVALID_ARG = 1,
  MAGUS_ERR_NOT_INITIALIZED = 2,
  MAGUS_ERR_CUDA = 3,
  MAGUS_ERR_NCCL = 4,
  MAGUS_ERR_OOM = 5,
  MAGUS_ERR_UNSUPPORTED = 6,
  MAGUS_ERR_NO_FEASIBLE = 7
} magus_status;

/* One policy configuration = the parameters of Alg. 1-3.
 * Validation: window >= 2; 1 <= history <= 64; deriv_len finite and > 0;
 * tau_inc, tau_dec finite; t_hi > 0 and not NaN (t_hi > 1 disables Alg. 2). */
typedef struct {
  int32_t window;    /* W = |mem_throughput_ls|. Paper: not stated; reading 10
                        (filled during the 10-cycle init, P@23939-P@24050).   */
  int32_t history;   /* H = |uncore_tune_ls|. Paper: 10 zeros (P@24182).     */
  double  deriv_len; /* L = direv_length, the divisor of Alg. 1 line 3.
                        Paper: not stated; reading L = W (P@20695).          */
  double  tau_inc;   /* Alg. 1: d >  tau_inc -> +1. Paper 200 (P@25197).     */
  double  tau_dec;   /* Alg. 1: d <  tau_dec -> -1. SIGNED: paper "500" is
                        read as -500 (reading R1).                 */
  double  t_hi;      /* Alg. 2: s/H >= t_hi -> high-frequency. Paper 0.4.    */
  int32_t variant;   /* 0 = the paper's MAGUS.  NEXT rows:
                        MAGUS_VARIANT_CLOSED_LOOP: Alg. 1 observes delivered
                        throughput min(x_t, B(l_t)) instead of demand (f3);
                        MAGUS_VARIANT_GRADUAL: +-step ratio per event instead
                        of the jump to max/min (f4, the contrast of P@35554).
                        Non-zero variants run on the sequential (closed
                        loop) or the time-segmented walk (open loop)
                        kernels; see MAGUS_OPT_KERNEL.                       */
  int32_t step;      /* ratio step of MAGUS_VARIANT_GRADUAL (>= 1), else 0   */
} magus_policy;
enum { MAGUS_VARIANT_CLOSED_LOOP = 1, MAGUS_VARIANT_GRADUAL = 2 };

/* Platform + accounting model M (an assumption).
 * Validation: 1 <= ratio_min < ratio_max <= 127; dt_s > 0; bw_max_mbs > 0;
 * beta >= 0; all doubles finite; powers/energies >= 0. */
typedef struct {
  int32_t ratio_min;      /* uncore ratio, 100 MHz units: 8 (0.8 GHz)        */
  int32_t ratio_max;      /* 22 (2.2 GHz) Intel+A100, P@29320; 25 Max1550    */
  double  dt_s;           /* sampling interval, 0.2 s (P@44789)              */
  double  bw_max_mbs;     /* memory-path capacity at ratio_max (MB/s);
                             capacity at ratio l is bw_max * l / ratio_max   */
  double  beta;           /* memory-boundness of the stretch                 */
  double  p_other_w;      /* power not attributable to the uncore (W)       */
  double  p_unc_min_w;    /* uncore power at ratio_min (W)                   */
  double  p_unc_max_w;    /* uncore power at ratio_max (W); 82 W range from
                             Fig. 2 (P@12253)                                */
  double  e_switch_j;     /* energy per frequency change ("negligible", 0)   */
  double  t_switch_s;     /* time per frequency change (0)                   */
  double  slowdown_bound; /* 0.05, the "<5 % performance loss" (P@1715)      */
  double  burst_mbs;      /* Sec. 6.3 burst threshold theta for the Jaccard
                             accuracy (P@41094-P@41603; "predefined", value
                             not printed): an interval is a burst when the
                             delivered throughput min(x, B_l) exceeds it.
                             <= 0 disables the burst counters.               */
} magus_platform;

/* Result per (config, trace).  Integer counters are exact; time/energy are
 * model M evaluated from them in a fixed fp64 operation order.  120 bytes. */
typedef struct {
  int64_t  n_events;      /* rounds with trend != 0 (Alg. 3 l.17/22 push 1)  */
  int64_t  n_hi_rounds;   /* rounds with high_freq_status = 1 (l.10)         */
  int64_t  n_msr_writes;  /* tune_uncore_freq calls (l.11, l.19, l.25)       */
  int64_t  n_changes;     /* t in [1,T): dec[t] != dec[t-1]                  */
  int64_t  n_min_dec;     /* #t with dec[t] = ratio_min                      */
  int64_t  n_min_int;     /* #t whose interval ran at ratio_min (l_t = dec[t-1]) */
  uint64_t q_min;         /* sum of quantised stretch over intervals at min  */
  uint64_t q_max;         /* same over intervals at max                      */
  uint64_t digest;        /* sum_w word_w * (mix64(w)|1) mod 2^64 over the
                             32-step decision words          */
  double   time_s;        /* modelled runtime under MAGUS                    */
  double   energy_j;      /* modelled energy under MAGUS                     */
  double   slowdown;      /* time_s / base.time_s - 1 (>= 0 exactly)         */
  int32_t  viol;          /* slowdown > slowdown_bound                       */
  int32_t  reserved;
  int64_t  n_burst_base;  /* #t with min(x_t, B(ratio_max)) > burst_mbs      */
  int64_t  n_burst_magus; /* #t with min(x_t, B(l_t)) > burst_mbs (l_t =
                             dec[t-1]); Jaccard (Sec. 6.3) = |A and B| /
                             |A or B| = n_burst_magus / n_burst_base, since
                             B(l) <= B(max) makes the MAGUS bursts a subset  */
} magus_summary;

/* Config-independent baseline per trace: uncore pinned at ratio_max (the
 * Intel default for GPU-dominant apps, P@10496 / P@30503).  32 bytes. */
typedef struct {
  uint64_t q_base;        /* sum of quantised stretch at ratio_max           */
  double   time_s;
  double   energy_j;
  uint64_t reserved;
} magus_base;

/* Per-config totals over traces: exact integer sums (uint64[MAGUS_TOT_WORDS = 18]) so that the
 * cross-trace and cross-GPU reduction is order-free and bit-reproducible.
 * The q sums are split into 32-bit limbs (q = hi*2^32 + lo per trace) so that
 * each limb sum fits in 64 bits for any n_traces < 2^32, which also makes a
 * plain NCCL uint64 sum exact. */
enum {
  MAGUS_TOT_N_TRACES = 0,
  MAGUS_TOT_N_VIOL,
  MAGUS_TOT_EVENTS,
  MAGUS_TOT_HI_ROUNDS,
  MAGUS_TOT_MSR_WRITES,
  MAGUS_TOT_CHANGES,
  MAGUS_TOT_MIN_DEC,
  MAGUS_TOT_MIN_INT,
  MAGUS_TOT_QMIN_LO,
  MAGUS_TOT_QMIN_HI,
  MAGUS_TOT_QMAX_LO,
  MAGUS_TOT_QMAX_HI,
  MAGUS_TOT_QBASE_LO,
  MAGUS_TOT_QBASE_HI,
  MAGUS_TOT_N_STEPS,     /* sum over traces of T                            */
  MAGUS_TOT_BURST_BASE,  /* sum of n_burst_base                             */
  MAGUS_TOT_BURST_MAGUS, /* sum of n_burst_magus                            */
  MAGUS_TOT_RESERVED,
  MAGUS_TOT_WORDS = 18
};

/* fp64 quantities derived from one config's integer totals (host-side,
 * fixed operation order). */
typedef struct {
  double  energy_j;       /* fleet energy under MAGUS                         */
  double  time_s;         /* fleet runtime under MAGUS                        */
  double  base_energy_j;  /* fleet energy at ratio_max                        */
  double  base_time_s;
  double  saving;         /* 1 - energy_j / base_energy_j                     */
  double  slowdown;       /* time_s / base_time_s - 1                         */
  int64_t n_viol;         /* traces whose own slowdown exceeds the bound      */
  int64_t n_traces;
  double  jaccard;        /* fleet burst Jaccard, sum A and B / sum A or B
                             (1 when there is no burst at all)               */
} magus_derived;

/* ---- lifecycle -------------------------------------------------------- */

/* Creates a context bound to CUDA `device`, enqueuing on `cuda_stream`
 * (a cudaStream_t; NULL = legacy default stream).  Copies *plat. */
magus_status magus_init(magus_ctx* out, int device, void* cuda_stream,
                        const magus_platform* plat);
magus_status magus_destroy(magus_ctx ctx);
magus_status magus_set_stream(magus_ctx ctx, void* cuda_stream);
const char*  magus_status_string(magus_status s);
const char*  magus_last_error(magus_ctx ctx);
int32_t      magus_abi_version(void);

/* ---- presets (P@25197, P@44170, P@29320, P@29831, P@12253) ------------ */
enum { MAGUS_POLICY_PAPER_DEFAULT = 0, MAGUS_POLICY_PAPER_PARETO = 1 };
enum { MAGUS_PLATFORM_INTEL_A100 = 0, MAGUS_PLATFORM_INTEL_MAX1550 = 1 };
magus_status magus_policy_preset(int32_t id, magus_policy* out);
magus_status magus_platform_preset(int32_t id, magus_platform* out);
/* SWEEP256: tau_inc {100,200,300,400} x tau_dec {-250,-500,-750,-1000} x
 * t_hi {0.2,0.3,0.4,0.5} x W {4,6,10,16}; L = W, H = 10;
 * index = iInc + 4*(iDec + 4*(iHi + 4*iW)).  paper_default = 165.
 * FLEET64: same without the W axis, W = L = H = 10; paper_default = 37. */
magus_status magus_grid_sweep256(magus_policy out[256]);
magus_status magus_grid_fleet64(magus_policy out[64]);

/* ---- the hot path ------------------------------------------------------ */

/* Replays Alg. 1-3 over every interval of every trace for every config and
 * scores the decisions with model M.
 *   traces        device, fp32, TIME-MAJOR: sample t of trace n at
 *                 traces[t*ld + n] (MB/s per interval).  NaN samples behave
 *                 as "hold" (both Alg. 1 comparisons false).
 *   n_traces      N >= 1;  n_steps T in [1, 2^24];  ld >= N.
 *   params        HOST array of n_params (>= 1) configs.
 *   out_summary   device [n_params][n_traces] or NULL.
 *   out_base      device [n_traces] or NULL.
 *   out_decisions device uint32 [n_params][ceil(T/32)][n_traces] or NULL:
 *                 bit (t % 32) of word [c][t/32][n] is 1 iff dec[t] = ratio_min.
 *                 (Time-blocked, trace-minor: each warp stores 128 contiguous
 *                 bytes.)  Bits past T are 0.
 *   out_totals    device uint64 [n_params][MAGUS_TOT_WORDS] or NULL.
 * Asynchronous on the context stream. */
magus_status magus_replay(magus_ctx ctx, const float* traces, int64_t n_traces,
                          int64_t n_steps, int64_t ld,
                          const magus_policy* params, int32_t n_params,
                          magus_summary* out_summary, magus_base* out_base,
                          uint32_t* out_decisions, uint64_t* out_totals);

/* ---- time-chunked replay (SURVEY §8(b) magus_replay_resume, §8(e)) -----
 * Replays a long trace set in time chunks that need not fit in HBM together
 * (config 4: 262 GB on one GPU).  Exact by the closed form of Alg. 3
 * (DESIGN.md 6.3): p_t and the Alg. 2 history depend only on
 * x[t-W-H+1..t], and the only carried decision state is dec[t_start-1]; the
 * model-M accumulators are integers, so chunk sums are order-free.
 *
 *   state     caller-owned DEVICE buffer of magus_resume_state_bytes(N, C)
 *             bytes, 8-byte aligned, ALL ZERO before the first chunk (t = 0);
 *             one state per (trace set, params) sequence; not shared between
 *             concurrent calls.  Layout (opaque): integer accumulators
 *             [C][12][N] u64, then dec[t_start-1] [C][N] u32.
 *   traces    device, time-major like magus_replay: row r (< n_rows) holds
 *             global interval t_base + r.
 *   t_base    multiple of 32;  t_start multiple of 32 in [t_base,
 *             t_base + n_rows): the first interval this call decides; it MUST
 *             equal the end (t_base + n_rows) of the previous call on `state`
 *             (0 on a zeroed state).  Rows [t_base, t_start) are the halo:
 *             t_start - t_base >= min(t_start, magus_resume_halo(params)).
 *             Chunks other than the last must end on a multiple of 32.
 *   outputs   as magus_replay over the PREFIX [0, t_base + n_rows): summaries,
 *             base and totals are those of a one-shot replay of the first
 *             t_base + n_rows intervals (bit-identical); out_decisions holds
 *             the words of [t_start, t_base + n_rows) only:
 *             [n_params][ceil((t_base + n_rows - t_start)/32)][n_traces].
 * Runs the stream kernel only (variant 0, W <= 33, H <= 32, 16-B aligned
 * traces, ld % 4 == 0): MAGUS_ERR_UNSUPPORTED otherwise.  Asynchronous. */
magus_status magus_resume_state_bytes(int64_t n_traces, int32_t n_params, size_t* out);
magus_status magus_resume_halo(const magus_policy* params, int32_t n_params, int64_t* rows);
magus_status magus_replay_resume(magus_ctx ctx, const float* traces, int64_t n_traces,
                                 int64_t n_rows, int64_t ld, int64_t t_base, int64_t t_start,
                                 const magus_policy* params, int32_t n_params, void* state,
                                 magus_summary* out_summary, magus_base* out_base,
                                 uint32_t* out_decisions, uint64_t* out_totals);

/* Per-interval decisions as uncore ratios (needed for multi-level variants):
 * out_levels DEVICE uint8 [n_params][n_steps][n_traces], level[c][t][n] =
 * dec[t] of trace n under config c.  Runs the walk kernels (open loop) or
 * the sequential kernel (closed loop), never the stream kernel; other
 * outputs as in magus_replay.  Asynchronous. */
magus_status magus_replay_levels(magus_ctx ctx, const float* traces, int64_t n_traces,
                                 int64_t n_steps, int64_t ld, const magus_policy* params,
                                 int32_t n_params, uint8_t* out_levels,
                                 magus_summary* out_summary, uint64_t* out_totals);

/* NEXT f2: offline-optimal schedules under model M.
 * For every trace and every Lagrange weight lambda_j >= 0 (HOST array),
 * the schedule dec[0..T-1] over the level set (full_grid = 0: {ratio_min,
 * ratio_max}, MAGUS's decision space; 1: every ratio in between) that
 * minimises  energy + lambda * time  of model M, by an exact DP in time order
 * with deterministic tie-breaks (stay before move; lowest ratio first).
 * out DEVICE double [n_traces][n_lambda][3] = {minimal cost, energy, time}
 * of that schedule (energy/time summed along the path in time order).
 * lambda = 0 gives the least energy any schedule reaches: a lower bound MAGUS
 * cannot beat; max_j (cost_j - lambda_j * (1 + bound) * base_time) is the
 * Lagrangian lower bound of the slowdown-constrained problem.  Asynchronous. */
magus_status magus_offline_bound(magus_ctx ctx, const float* traces, int64_t n_traces,
                                 int64_t n_steps, int64_t ld, const double* lambdas,
                                 int32_t n_lambda, int32_t full_grid, double* out);

/* End-to-end variant: every pointer is HOST memory (pinned or pageable).
 * Stages traces host->device through context-owned buffers, runs
 * magus_replay, copies the requested outputs back.  Synchronises. */
magus_status magus_replay_host(magus_ctx ctx, const float* traces_host,
                               int64_t n_traces, int64_t n_steps, int64_t ld,
                               const magus_policy* params, int32_t n_params,
                               magus_summary* summary_host,
                               magus_base* base_host,
                               uint32_t* decisions_host,
                               uint64_t* totals_host);

/* Derives the fp64 fleet quantities of one config from its integer totals
 * (host memory, MAGUS_TOT_WORDS words) under the context's platform. */
magus_status magus_totals_derive(magus_ctx ctx, const uint64_t* totals_host,
                                 magus_derived* out);

/* Picks the config of least fleet energy among those with n_viol == 0
 * (the Sec. 6.4 choice on the energy/runtime front, P@44696, under the
 * <5 % loss bound, P@1715).  Ties -> lowest index.  `totals` is DEVICE
 * memory [n_params][MAGUS_TOT_WORDS] (already summed over ranks when
 * sharded).  If no config is feasible returns MAGUS_ERR_NO_FEASIBLE with
 * *best = argmin (n_viol, energy) and *best_row filled.  Synchronises. */
magus_status magus_sweep_best(magus_ctx ctx, const uint64_t* totals,
                              int32_t n_params, int32_t* best,
                              magus_derived* best_row);

/* Asynchronous form of magus_sweep_best: the derivation and the argmin run
 * on the device (bit-identical to the host derivation) and the result is
 * copied to host memory in ONE transfer without synchronising the stream;
 * *out is valid once the stream reaches this point (pinned host memory
 * keeps the copy asynchronous). */
typedef struct {
  int32_t best;           /* chosen config (argmin (n_viol, energy) if none feasible) */
  int32_t feasible;       /* 1 if some config has n_viol == 0                        */
  magus_derived row;      /* its fleet quantities                                    */
} magus_choice;
magus_status magus_sweep_best_async(magus_ctx ctx, const uint64_t* totals, int32_t n_params,
                                    magus_choice* out);

/* Host-only forms (no context, no GPU): the same derivation and choice from
 * host totals [n_params][MAGUS_TOT_WORDS] under *plat.  Used by the
 * multi-rank glue after the all-reduce and by CPU tests. */
magus_status magus_derive_host(const magus_platform* plat, const uint64_t* totals_host,
                               magus_derived* out);
magus_status magus_sweep_best_host(const magus_platform* plat, const uint64_t* totals_host,
                                   int32_t n_params, int32_t* best, magus_derived* best_row);

/* Energy/runtime Pareto front over the configs (Sec. 6.4, Fig. 7,
 * P@43971-P@44696): on_front[c] = 1 iff no config has fleet energy and
 * fleet runtime both <= config c's with at least one strictly less.
 * `totals` DEVICE [n_params][MAGUS_TOT_WORDS]; on_front HOST [n_params];
 * *n_front = number of configs on the front.  Synchronises. */
magus_status magus_pareto_front(magus_ctx ctx, const uint64_t* totals, int32_t n_params,
                                int32_t* on_front, int32_t* n_front);
magus_status magus_pareto_front_host(const magus_platform* plat, const uint64_t* totals_host,
                                     int32_t n_params, int32_t* on_front, int32_t* n_front);

/* ---- synthetic traces (input generator; gen/magus_gen.h) --------------- */
enum { MAGUS_GEN_MIX = 0, MAGUS_GEN_ADVERSARIAL = 1 };
/* Writes traces id0 .. id0+n_traces-1 of the seeded Markov phase model to
 * device memory out[t*ld + i] (fp32, integer-valued MB/s).  Bit-identical to
 * the host generator in gen/.  Asynchronous. */
magus_status magus_gen_traces(magus_ctx ctx, uint64_t seed, int64_t id0,
                              int64_t n_traces, int64_t n_steps, int64_t ld,
                              int32_t kind, float* out);
/* Time-chunked form (config 4 on one GPU: the traces never coexist in HBM):
 * writes intervals [t0, t0 + n_rows) of the same traces to out rows
 * 0..n_rows-1 (row stride ld).  `state` is a caller-owned DEVICE buffer of
 * magus_gen_state_bytes(n_traces) bytes holding each trace's phase machine:
 * t0 = 0 seeds it, later calls must continue at the previous t0 + n_rows.
 * Concatenated chunks equal magus_gen_traces bit for bit.  Asynchronous. */
magus_status magus_gen_state_bytes(int64_t n_traces, size_t* out);
magus_status magus_gen_traces_resume(magus_ctx ctx, uint64_t seed, int64_t id0, int64_t n_traces,
                                     int64_t t0, int64_t n_rows, int64_t ld, int32_t kind,
                                     void* state, float* out);

/* ---- diagnostics of the host precompute (no GPU needed) ----------------- */
/* The stream kernel never divides: Alg. 1's "d = delta/L > tau_inc" becomes
 * "delta > delta_inc" with delta_inc the largest double whose RN quotient by L
 * does not exceed tau_inc (exact because RN(delta/L) is monotone in delta);
 * likewise "delta < delta_dec"; Alg. 2's "s/H >= t_hi" becomes s >= k_hi
 * (k_hi = H+1: never).  Model M's "RN(x * (1/B_l)) > 1" becomes the float
 * comparison x > x_stretch_l. */
typedef struct {
  double  delta_inc;
  double  delta_dec;
  int32_t k_hi;
  int32_t reserved;
} magus_policy_consts;
typedef struct {
  float   x_stretch_min, x_stretch_max;
  double  inv_cap_min, inv_cap_max;   /* 1 / B_l in (MB/s)^-1 */
  double  p_min_w, p_max_w;           /* model-M power at ratio_min / max */
} magus_platform_consts;
magus_status magus_policy_inspect(const magus_policy* p, magus_policy_consts* out);
magus_status magus_platform_inspect(const magus_platform* p, magus_platform_consts* out);

/* ---- optional native NCCL path (SURVEY 8(b) magus_comm_init) ------------
 * The sweep's one collective (north_star (3)) without torch:
 * an in-place uint64 SUM all-reduce of the per-config totals over NVLink /
 * NVSwitch, exact and order-free (integer words).  libnccl.so.2 is opened
 * lazily on the first call (no link-time dependency); MAGUS_ERR_NCCL when it
 * is missing or an NCCL call fails (detail in magus_last_error). */
#define MAGUS_COMM_ID_BYTES 128
/* rank 0 creates the id and ships it to every rank by its own means */
magus_status magus_comm_unique_id(void* id_out /* host, MAGUS_COMM_ID_BYTES */);
/* one communicator per context (on ctx's device); collective over the
 * nranks processes: each must call it with the same id.  Replaces an
 * earlier communicator of ctx.  Synchronous. */
magus_status magus_comm_init(magus_ctx ctx, const void* id /* host, MAGUS_COMM_ID_BYTES */,
                             int32_t nranks, int32_t rank);
/* totals DEVICE uint64 [n_params][MAGUS_TOT_WORDS], summed over the ranks in
 * place on ctx's stream (asynchronous); a no-op without a communicator.
 * Call it between magus_replay and magus_sweep_best / _async on every rank
 * (every rank then takes the same deterministic choice, no broadcast). */
magus_status magus_allreduce_totals(magus_ctx ctx, uint64_t* totals, int32_t n_params);

/* ---- options, instrumentation ------------------------------------------ */
enum {
  MAGUS_OPT_KERNEL = 0,       /* 0 auto, 1 reference (per-sample, the printed
                                 divisions), 2 stream, 3 sequential (per-sample,
                                 latency-optimised: the auto choice for the
                                 closed loop with the gradual step), 4 walk
                                 (time-segmented open loop: the auto choice
                                 for f4 and level output; UNSUPPORTED for
                                 closed-loop configs), 5 spec (speculatively
                                 time-segmented closed loop, jump rule,
                                 W <= 65; opt-in)        */
  MAGUS_OPT_SEGMENTS = 1,     /* 0 auto, else the number of time segments    */
  MAGUS_OPT_TIMING = 2,       /* 1: record CUDA events around the main kernel */
  MAGUS_OPT_WAVES = 3,        /* auto segmentation: 0 (default) = wave model
                                 (segment count minimising the modelled
                                 rounds x segment length), else aim at this
                                 many waves of CTAs                          */
  MAGUS_OPT_BUNDLE = 4,       /* configs per thread sharing Alg. 1/2 work:
                                 0 auto, or force 1, 2 or 4                  */
  MAGUS_OPT_SPEC_WARM = 5,    /* kernel 5: rounds each segment's speculation
                                 replays before it (0 = auto, min(segment,
                                 1024)); any value gives the same results   */
  MAGUS_OPT_TRACE = 6,        /* 1: the stream kernel records a per-CTA
                                 timeline (diagnostics; magus_get_trace)     */
  MAGUS_OPT_NARROW = 7,       /* 1: the stream kernel's one-config path uses
                                 128-trace CTAs (4 per SM) instead of the
                                 default 512-trace CTA per SM (A/B option;
                                 results are identical)                      */
  MAGUS_OPT_WALK1 = 9,        /* 1: the open-loop walk (kernel 4) in ONE pass
                                 (segment map and replay in the same scan,
                                 the carry-dependent prefix replayed after a
                                 decoupled look-back) instead of the default
                                 two passes (maps, then the replay); measured
                                 slower on config 2; A/B
                                 option, results identical                  */
  MAGUS_OPT_FAMILY = 8        /* 0 (default): a (W, H) group of <= 16 bundles
                                 of 4 configs with <= 8 distinct tau_inc and
                                 tau_dec thresholds (a sweep grid, Sec. 6.4)
                                 runs on the family kernel, which compares
                                 each sample once for the whole group; 1: the
                                 per-bundle stream kernel (A/B option;
                                 results are identical)                      */
};
magus_status magus_set_option(magus_ctx ctx, int32_t key, int64_t value);

typedef struct {
  int64_t launches_total;     /* kernels launched by this context            */
  int64_t main_launches;      /* replay-kernel launches timed (OPT_TIMING)   */
  double  main_ms_total;      /* summed CUDA-event time of those launches    */
  int64_t last_segments;      /* time segments used by the last replay       */
  int64_t last_kernel;        /* 1 reference, 2 stream, 3 sequential         */
  int64_t last_grid;          /* CTAs of the last main launch                */
  int64_t last_reruns;        /* kernel 5: segments whose speculation missed
                                 and were replayed again, in the last replay
                                 (read with a device sync); else 0           */
  int64_t last_family;        /* stream path: launches of the last replay that
                                 ran on the family kernel (a sweep grid's
                                 (W, H) groups; MAGUS_OPT_FAMILY)            */
} magus_stats;
/* Per-CTA timeline of the last stream-kernel replay under MAGUS_OPT_TRACE
 * (diagnostics, not the hot path): out host uint64 [cap][8] per CTA (in
 * blockIdx order) = {start, scan end, look-back end, end} (%globaltimer ns),
 * SM id, time segment, trace group, 1 if this CTA finalised its group.
 * *n_out = CTAs recorded (<= cap).  Synchronises ctx's stream.
 * INVALID_ARG without a traced replay. */
magus_status magus_get_trace(magus_ctx ctx, uint64_t* out, int64_t cap, int64_t* n_out);
/* Synchronises when timing is on (reads the events). */
magus_status magus_get_stats(magus_ctx ctx, magus_stats* out);
magus_status magus_reset_stats(magus_ctx ctx);

#ifdef __cplusplus
}
#endif
#endif /* MAGUS_H_ */
