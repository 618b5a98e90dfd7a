// magus_internal.h -- device-side parameter blocks and launch plumbing shared
// by the libmagus translation units (NOT part of the C-ABI).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/magus.h"

namespace magus {

// Stretch metering of model M: the per-interval stretch
// sigma = max(0, x/B_l - 1) is capped at 2^15 intervals and metered in units
// of 2^-24 interval, so every accumulation is an exact integer sum.
constexpr double kQScale = 16777216.0;                 // 2^24
constexpr double kQCapScaled = 549755813888.0;         // 2^15 * 2^24 = 2^39
constexpr int64_t kMaxSteps = int64_t(1) << 24;       // keeps sum q < 2^63

// Per-config constants, precomputed on the host (precompute.cpp).
struct DevPolicy {
  // Alg. 1 literal form (reference kernel): d = delta / L
  double L, tau_inc, tau_dec;
  // Alg. 1 inverted form (stream kernel): delta > d_inc  <=> RN(delta/L) > tau_inc
  //                                        delta < d_dec  <=> RN(delta/L) < tau_dec
  double d_inc, d_dec;
  // Alg. 2 literal form: (double)s / (double)H >= t_hi
  double t_hi;
  // Alg. 2 inverted form: s >= k  (k = H+1: never)
  int32_t W, H, k, pad;
  int32_t variant, step;  // NEXT f3/f4 (per-sample kernel only)
};

// Platform / model-M constants.
struct DevPlatform {
  int32_t r_min, r_max;
  // literal form (reference kernel): r = x * invB; r > 1 -> s = r - 1 ...
  double invB_min, invB_max;
  // inverted form (stream kernel): x > xthr <=> RN(x*invB) > 1 ; r24 = x*invB24
  float xthr_min, xthr_max;
  double invB24_min, invB24_max;
  // finalisation (fp64, fixed order)
  double dt, cQ, P_max, P_min, e_sw, t_sw, bound;
  // Sec. 6.3 bursts: burst(t, l) <=> x_t > theta and B_l > theta
  double burst_mbs, Bmin, Bmax;  // literal form (reference kernel)
  float xburst;                  // x > xburst <=> (double)x > theta
  int32_t burst_on;              // theta > 0 and B_max > theta
  int32_t burst_min_keeps;       // B_min > theta: the level never hides a burst
  float xobs_max;                // x > xobs_max <=> (double)x > B_max (f3: delivered < x at r_max)
};

// Work/scratch block of the fused stream kernel (kernels_stream.cu).  The
// counters and accumulators are zero at allocation and self-cleaning (the
// last user of each resets it); the segment status words are tagged with a
// per-replay epoch, so nothing needs a memset between replays.
constexpr int kAccFields = 12;  // ev hi msr ch mdec mint qmin qmax qbase dig bbase bmagus
struct StreamWork {
  uint32_t* ticket;              // [1] launch-order work ticket
  uint32_t* done;                // [1] finished CTAs of the launch
  uint32_t* status;              // [C][nseg][N] epoch<<3 | last_min<<2 | seen<<1 | 1
  unsigned long long* acc;       // [C][kAccFields][N] segment sums
  uint32_t* arrive;              // [C][ngroups] finished segments
  unsigned long long* tacc;      // (unused since the finalisers add into the totals rows)
  uint32_t* tarrive;             // (unused)
  uint32_t epoch;
  magus_summary* summary;        // [C][N] or NULL
  magus_base* base;              // [N] or NULL
  uint32_t* dec;                 // [C][nw][N] or NULL
  int64_t dec_cstride;           // nw * N
  uint64_t* totals;              // [C][18] or NULL
  const unsigned long long* mul; // [ceil(T/32)][2] {mix64(w) | 1, 0}: 16-B bulk-copy rows
  // time-chunked replay (magus_replay_resume): the kernel works in global
  // intervals [ts, T); buffer row r (TMA coordinate) is interval tb + r.
  // Both are multiples of 32 (0, 0 for a one-shot replay).
  int32_t tb, ts;
  // resume state ([C][N] dec[t_start-1] bits, read at the start, rewritten by
  // the finaliser once every segment of the (bundle, group) is in); NULL =
  // one-shot replay.  In resume mode `acc` points into the caller's state and
  // is kept (not self-cleaned).
  uint32_t* carry;
};
// MAGUS_OPT_TRACE: the per-CTA timeline buffer's address lives in scratch
// right after the ticket words (ticket[2..3] as a u64, NULL = off), so the
// kernel's parameter block -- and its register allocation -- is unchanged.
constexpr int kTraceSlotWords = 2;
// ticket[4]: raised (1) once the launch's first CTA has initialised the
// totals rows; cleared with the ticket by the launch's last CTA
constexpr int kTotalsFlagWord = 4;
// resume state layout: acc [C][kAccFields][N] u64, then carry [C][N] u32
inline size_t resume_state_bytes(int64_t N, int32_t C) {
  return 8 * (size_t)kAccFields * (size_t)C * (size_t)N + 4 * (size_t)C * (size_t)N;
}

// Host precompute (precompute.cpp); returns false + message on invalid input.
bool validate_policy(const magus_policy& p, char* msg, size_t n);
bool validate_platform(const magus_platform& p, char* msg, size_t n);
DevPolicy make_dev_policy(const magus_policy& p);
DevPlatform make_dev_platform(const magus_platform& p);
double invert_inc(double L, double tau_inc);
double invert_dec(double L, double tau_dec);
float stretch_threshold(double invB);
float above_threshold(double theta);  // largest float f with !((double)f > theta)
constexpr int kTotAccWords = 15;      // totals words 1..13 + the two burst sums

// Launchers (each returns the number of kernels launched, or -1 on error).

// Per-sample kernel (kernels_ref.cu); multi = per-level accounting (gradual
// variant); out_levels optional uint8 [C][T][N].
int launch_reference(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
                     const DevPolicy* pol_dev, int32_t C, const DevPlatform& plat, double bw_max,
                     double p_lo, double p_span, bool multi, bool literal, magus_summary* out_summary,
                     magus_base* out_base, uint32_t* out_dec, uint8_t* out_levels);

// Sequential-variant kernel (kernels_seq.cu): one thread per (trace, config),
// cp.async-prefetched, latency-optimised chain; f3/f4 and level output.
bool seq_supported(const magus_policy& p);
bool seq_fits(const DevPlatform& plat, bool closed, bool multi);  // shared memory of the launch
int launch_seq(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
               const DevPolicy* pol_dev, int32_t C, const DevPlatform& plat, double bw_max,
               double p_lo, double p_span, bool closed, bool multi, magus_summary* out_summary,
               magus_base* out_base, uint32_t* out_dec, uint8_t* out_levels);

// Time-segmented open-loop kernel (kernels_walk.cu): f4 and level output;
// scratch = maps + accumulators (walk_scratch_bytes); out_summary required.
size_t walk_scratch_bytes(int64_t N, int32_t C, int64_t T, int64_t nseg, const DevPlatform& plat);
int launch_walk(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld, const DevPolicy* pol_dev,
                int32_t C, int32_t max_H, const DevPlatform& plat, double bw_max, double p_lo, double p_span,
                int64_t nseg, int64_t seg_len, void* scratch, magus_summary* out_summary, magus_base* out_base,
                uint32_t* out_dec, uint8_t* out_levels, bool fused,
                int32_t same_W /* W of every config, else 0: pass 1's compile-time lag window */);

// Speculatively time-segmented closed loop (kernels_spec.cu): f3 with the
// jump rule; scratch = spec_scratch_bytes; out_summary required.
bool spec_supported(const magus_policy& p);
size_t spec_scratch_bytes(int64_t N, int32_t C, int64_t nseg);
int launch_spec(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld, const DevPolicy* pol_dev,
                int32_t C, bool wide /* some H > 32 or W > 33 */, const DevPlatform& plat, int64_t nseg, int64_t seg_len, int64_t warm, void* scratch,
                magus_summary* out_summary, magus_base* out_base, uint32_t* out_dec, uint8_t* out_levels,
                unsigned int** reruns_out);

// Native NCCL (comm.cpp, dlopen'ed lazily); return 0 or an ncclResult_t /
// -1 when libnccl is unavailable.
bool nccl_available();
const char* nccl_error(int r);
int nccl_unique_id(void* out);
int nccl_comm_init(void** comm, const void* id_bytes, int nranks, int rank);
int nccl_comm_destroy(void* comm);
int nccl_allreduce_u64_sum(void* comm, uint64_t* buf, size_t count, cudaStream_t s);

// Configuration-family kernel (kernels_family.cu): one CTA = 32 traces x one
// time segment x every bundle of a (W, H) launch group (<= 16 bundles of 4
// configs), the per-sample Alg. 1 compares done once for all of them against
// the family's distinct inverted thresholds.
constexpr int kFamMaxThr = 8;   // distinct d_inc / d_dec values of a family
constexpr int kFamMaxBund = 16;
struct FamilyDev {
  double d_inc[kFamMaxThr], d_dec[kFamMaxThr];
  int32_t ni, nd;
  uint8_t bi[kFamMaxBund], bd[kFamMaxBund];  // bundle -> threshold indices
};
bool family_supported(int32_t W, int32_t H, int32_t NB, int32_t nbund, int32_t ni, int32_t nd);
int family_cta_traces();
int family_ctas_per_sm(int32_t H, int32_t nbund);
int launch_family(cudaStream_t s, const void* tmap32 /* CUtensorMap, box 32 x 32 */, const void* tmap_mul,
                  int64_t N, int64_t T, const DevPolicy* pol_dev, const int32_t* bundles_dev, int32_t nbund,
                  int32_t H, const FamilyDev& fam, const DevPlatform& plat, int64_t nseg, int64_t seg_len,
                  const StreamWork& wk, int* grid_out);

bool stream_supported(int32_t W, int32_t H);
// Fused stream kernel over nbund bundles of NB configs (bundles_dev:
// [nbund][NB] global config indices, -1 = padding).  All configs of a launch
// share (W, H); the configs of a bundle also share L, tau_inc and tau_dec.
// Replay + carry look-back + finalisation + totals in one launch.
int launch_stream(cudaStream_t s, const void* tmap /* CUtensorMap, host copy */,
                  const void* tmap_mul /* CUtensorMap over StreamWork::mul */, int64_t N,
                  int64_t T, const DevPolicy* pol_dev, const int32_t* bundles_dev, int32_t nbund,
                  int32_t NB, int32_t W, int32_t H, const DevPlatform& plat, int64_t nseg,
                  int64_t seg_len, const StreamWork& wk, bool narrow, int* grid_out);
int stream_ctas_per_sm(int32_t W, int32_t H, int32_t NB, bool burst, bool narrow);
int stream_cta_traces(int32_t W, int32_t H, int32_t NB, bool burst, bool narrow);  // traces per CTA

// NEXT f2 DP (kernels_bound.cu): out [N][nl][3] = {cost, energy, time}.
int launch_bound(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
                 const double* lambdas_dev, int32_t nl, bool full_grid, const DevPlatform& plat,
                 double bw_max, double p_lo, double p_span, double* out);

int launch_totals(cudaStream_t s, const magus_summary* summary, const magus_base* base, int64_t N,
                  int64_t T, int32_t C, uint64_t* totals);

// device sweep choice (kernels_post.cu), bit-identical to the host form
typedef magus_choice SweepResult;
int launch_sweep_best(cudaStream_t s, const uint64_t* totals, int32_t C, const DevPlatform& plat,
                      SweepResult* res);

// digest multiplier table mul[w] = mix64(w) | 1 for w < nw (kernels_post.cu)
int launch_digest_table(cudaStream_t s, unsigned long long* mul, int64_t nw);

int launch_gen(cudaStream_t s, uint64_t seed, int64_t id0, int64_t N, int64_t T, int64_t ld,
               int32_t kind, float* out);
int launch_gen_resume(cudaStream_t s, uint64_t seed, int64_t id0, int64_t N, int64_t t0, int64_t R,
                      int64_t ld, int32_t kind, void* state, float* out);
size_t gen_state_bytes(int64_t N);

// host-side derivation of fleet quantities (api.cu)
void derive_totals(const DevPlatform& p, const uint64_t* w, magus_derived* out);

}  // namespace magus
