// api.cu -- libmagus C-ABI (include/magus.h): validation, per-config host
// precompute, scratch management, kernel dispatch, totals, sweep choice.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <utility>
#include <vector>

#include "magus_internal.h"

using namespace magus;

struct magus_ctx_s {
  int device = 0;
  cudaStream_t stream = nullptr;
  magus_platform plat{};
  DevPlatform dplat{};
  std::string err;
  int sms = 148;
  // options
  int64_t opt_kernel = 0, opt_segments = 0, opt_timing = 0, opt_waves = 0, opt_trace = 0, opt_narrow = 0;
  int64_t opt_walk1 = 0;   // 1: the one-pass walk kernel (A/B)
  int64_t opt_family = 0;  // 0: family kernel for the groups it takes; 1: bundle kernels only
  void* trace_dev = nullptr;   // MAGUS_OPT_TRACE timeline [trace_cap][8]
  int64_t trace_cap = 0, trace_n = 0;
  bool trace_armed = false;          // scratch holds a timeline address
  void* trace_slot_host[2] = {nullptr, nullptr};  // [0] the address, [1] NULL
  // device scratch
  void* scratch = nullptr;
  size_t scratch_bytes = 0;
  uint64_t work_sig = 0;   // layout of the fused kernel's counters in scratch
  uint32_t epoch = 0;      // per-replay tag of the segment status words
  // policy upload cache
  std::vector<magus_policy> last_params;
  void* pol_dev = nullptr;
  size_t pol_dev_bytes = 0;
  void* pol_host = nullptr;  // pinned staging
  size_t pol_host_bytes = 0;
  cudaEvent_t pol_copied = nullptr;
  std::vector<uint64_t> best_host;   // sweep_best staging (size marker)
  void* best_pinned = nullptr;
  struct LaunchGroup {
    int32_t W, H, NB;   // kernel specialisation
    int64_t off;        // first bundle (rows of NB config indices) in the device table
    int32_t nbund;
    bool fam_ok;        // the family kernel can take the whole group (kernels_family.cu)
    FamilyDev fam;
  };
  std::vector<LaunchGroup> groups;  // one stream launch each
  int64_t opt_bundle = 0;           // 0 auto, else force NB in {1, 2, 4}
  int64_t opt_spec_warm = 0;
  unsigned int* spec_reruns = nullptr;  // device counter of the last spec replay (in scratch)
  void* comm = nullptr;                 // ncclComm_t of magus_comm_init (optional)        // spec kernel: rounds replayed before a segment (0 auto)
  int64_t uploaded_bundle_opt = -1;
  // e2e staging (device)
  void* sweep_dev = nullptr;  // SweepResult of magus_sweep_best_async
  void* mul_dev = nullptr;  // digest multiplier table mix64(w) | 1, w < mul_nw
  int64_t mul_nw = 0;
  void* lam_dev = nullptr;  // NEXT f2 lambda grid
  size_t lam_bytes = 0;
  void* stage_dev = nullptr;
  size_t stage_bytes = 0;
  // stats
  int64_t launches = 0, main_launches = 0, last_segments = 0, last_kernel = 0, last_grid = 0, last_family = 0;
  double main_ms = 0.0;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> pending;
  std::vector<cudaEvent_t> event_pool;
  std::map<std::pair<int, int>, int> ctas_cache;
  PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
};

namespace {

magus_status fail(magus_ctx ctx, magus_status st, const char* fmt, ...) {
  if (ctx) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    std::vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    ctx->err = buf;
  }
  return st;
}

magus_status cuda_fail(magus_ctx ctx, cudaError_t e, const char* what) {
  return fail(ctx, MAGUS_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CK(call)                                   \
  do {                                             \
    cudaError_t e_ = (call);                       \
    if (e_ != cudaSuccess) return cuda_fail(ctx, e_, #call); \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

magus_status ensure_scratch(magus_ctx ctx, size_t bytes) {
  if (bytes <= ctx->scratch_bytes) return MAGUS_OK;
  ctx->work_sig = 0;
  // the stream may still use the old buffer
  CK(cudaStreamSynchronize(ctx->stream));
  if (ctx->scratch) cudaFree(ctx->scratch);
  ctx->scratch = nullptr;
  ctx->scratch_bytes = 0;
  const size_t want = align_up(bytes + bytes / 8, 1 << 20);
  cudaError_t e = cudaMalloc(&ctx->scratch, want);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(ctx, MAGUS_ERR_OOM, "scratch allocation of %zu bytes failed", want);
  }
  ctx->scratch_bytes = want;
  CK(cudaMemsetAsync(ctx->scratch, 0, want, ctx->stream));  // counters start at zero
  return MAGUS_OK;
}

cudaEvent_t take_event(magus_ctx ctx) {
  if (!ctx->event_pool.empty()) {
    cudaEvent_t e = ctx->event_pool.back();
    ctx->event_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

bool same_params(const std::vector<magus_policy>& a, const magus_policy* b, int32_t n) {
  if ((int32_t)a.size() != n) return false;
  return std::memcmp(a.data(), b, sizeof(magus_policy) * (size_t)n) == 0;
}

// Uploads DevPolicy[C] and the bundle table.  Configs are grouped by (W, H)
// (one kernel specialisation per group), and inside a group into bundles of
// NB configs with bit-identical inverted Alg. 1 thresholds (same L, tau_inc,
// tau_dec up to rounding): a bundle shares Delta, the event word and the Alg. 2
// window count, and differs only in k (t_hi).
magus_status upload_policies(magus_ctx ctx, const magus_policy* params, int32_t C) {
  if (same_params(ctx->last_params, params, C) && ctx->pol_dev &&
      ctx->uploaded_bundle_opt == ctx->opt_bundle)
    return MAGUS_OK;
  std::vector<DevPolicy> dp((size_t)C);
  std::map<std::pair<int, int>, std::map<std::pair<uint64_t, uint64_t>, std::vector<int32_t>>> g;
  for (int32_t c = 0; c < C; ++c) {
    dp[c] = make_dev_policy(params[c]);
    uint64_t ki, kd;
    std::memcpy(&ki, &dp[c].d_inc, 8);
    std::memcpy(&kd, &dp[c].d_dec, 8);
    g[{params[c].window, params[c].history}][{ki, kd}].push_back(c);
  }
  ctx->groups.clear();
  std::vector<int32_t> table;
  for (auto& wh : g) {
    size_t maxsz = 1;
    for (auto& b : wh.second) maxsz = std::max(maxsz, b.second.size());
    int32_t NB = ctx->opt_bundle ? (int32_t)ctx->opt_bundle : (maxsz >= 3 ? 4 : (int32_t)maxsz);
    magus_ctx_s::LaunchGroup lg{wh.first.first, wh.first.second, NB, 0, 0, false, {}};
    lg.off = (int64_t)table.size();
    // family: the distinct inverted thresholds of the group's bundles
    std::vector<uint64_t> dinc, ddec;
    std::vector<uint8_t> bi, bd;
    for (auto& b : wh.second) {
      const auto& v = b.second;
      auto idx = [](std::vector<uint64_t>& tab, uint64_t key) {
        for (size_t i = 0; i < tab.size(); ++i)
          if (tab[i] == key) return (uint8_t)i;
        tab.push_back(key);
        return (uint8_t)(tab.size() - 1);
      };
      const uint8_t ii = idx(dinc, b.first.first), id = idx(ddec, b.first.second);
      for (size_t i = 0; i < v.size(); i += (size_t)NB) {
        for (int32_t k = 0; k < NB; ++k) table.push_back(i + k < v.size() ? v[i + k] : -1);
        lg.nbund++;
        bi.push_back(ii);
        bd.push_back(id);
      }
    }
    lg.fam_ok = family_supported(lg.W, lg.H, NB, lg.nbund, (int32_t)dinc.size(), (int32_t)ddec.size());
    if (lg.fam_ok) {
      lg.fam.ni = (int32_t)dinc.size();
      lg.fam.nd = (int32_t)ddec.size();
      for (size_t i = 0; i < dinc.size(); ++i) std::memcpy(&lg.fam.d_inc[i], &dinc[i], 8);
      for (size_t i = 0; i < ddec.size(); ++i) std::memcpy(&lg.fam.d_dec[i], &ddec[i], 8);
      for (int32_t b = 0; b < lg.nbund; ++b) {
        lg.fam.bi[b] = bi[(size_t)b];
        lg.fam.bd[b] = bd[(size_t)b];
      }
    }
    ctx->groups.push_back(lg);
  }
  std::vector<int32_t>& cidx = table;
  const size_t pol_bytes = align_up(sizeof(DevPolicy) * (size_t)C, 256);
  const size_t need = pol_bytes + sizeof(int32_t) * cidx.size();
  if (ctx->pol_copied) CK(cudaEventSynchronize(ctx->pol_copied));  // pinned buffer reuse
  if (need > ctx->pol_dev_bytes) {
    CK(cudaStreamSynchronize(ctx->stream));
    if (ctx->pol_dev) cudaFree(ctx->pol_dev);
    ctx->pol_dev = nullptr;
    CK(cudaMalloc(&ctx->pol_dev, need));
    ctx->pol_dev_bytes = need;
  }
  if (need > ctx->pol_host_bytes) {
    if (ctx->pol_host) cudaFreeHost(ctx->pol_host);
    ctx->pol_host = nullptr;
    CK(cudaMallocHost(&ctx->pol_host, need));
    ctx->pol_host_bytes = need;
  }
  std::memcpy(ctx->pol_host, dp.data(), sizeof(DevPolicy) * (size_t)C);
  std::memcpy((char*)ctx->pol_host + pol_bytes, cidx.data(), sizeof(int32_t) * cidx.size());
  CK(cudaMemcpyAsync(ctx->pol_dev, ctx->pol_host, need, cudaMemcpyHostToDevice, ctx->stream));
  if (!ctx->pol_copied) CK(cudaEventCreateWithFlags(&ctx->pol_copied, cudaEventDisableTiming));
  CK(cudaEventRecord(ctx->pol_copied, ctx->stream));
  ctx->last_params.assign(params, params + C);
  ctx->uploaded_bundle_opt = ctx->opt_bundle;
  return MAGUS_OK;
}

const DevPolicy* dev_policies(magus_ctx ctx) { return (const DevPolicy*)ctx->pol_dev; }
const int32_t* dev_cidx(magus_ctx ctx, int64_t off) {
  const size_t pol_bytes = align_up(sizeof(DevPolicy) * ctx->last_params.size(), 256);
  return (const int32_t*)((const char*)ctx->pol_dev + pol_bytes) + off;
}

int ctas_per_sm(magus_ctx ctx, int W, int H, int NB) {
  const bool burst = ctx->dplat.burst_on != 0, narrow = ctx->opt_narrow != 0;
  auto key = std::make_pair((W * 8 + NB) * 4 + (burst ? 2 : 0) + (narrow ? 1 : 0), H);
  auto it = ctx->ctas_cache.find(key);
  if (it != ctx->ctas_cache.end()) return it->second;
  int v = stream_ctas_per_sm(W, H, NB, burst, narrow);
  ctx->ctas_cache[key] = v;
  return v;
}

int64_t stream_groups(magus_ctx ctx, int64_t N, int W, int H, int NB) {  // CTAs per (segment, bundle)
  const int tr = stream_cta_traces(W, H, NB, ctx->dplat.burst_on != 0, ctx->opt_narrow != 0);
  return (N + tr - 1) / tr;
}

// the family kernel takes the group: every bundle in one CTA (no burst counters there)
bool use_family(magus_ctx ctx, const magus_ctx_s::LaunchGroup& g) {
  return g.fam_ok && ctx->opt_family == 0 && ctx->dplat.burst_on == 0;
}
int64_t group_ctas(magus_ctx ctx, int64_t N, const magus_ctx_s::LaunchGroup& g, int64_t nseg) {
  if (use_family(ctx, g)) return (N + family_cta_traces() - 1) / family_cta_traces() * nseg;
  return stream_groups(ctx, N, g.W, g.H, g.NB) * g.nbund * nseg;
}
int group_ctas_per_sm(magus_ctx ctx, const magus_ctx_s::LaunchGroup& g) {
  if (use_family(ctx, g)) {
    auto key = std::make_pair(-1 - g.nbund, g.H == 10 ? 10 : 0);
    auto it = ctx->ctas_cache.find(key);
    if (it != ctx->ctas_cache.end()) return it->second;
    const int v = family_ctas_per_sm(g.H, g.nbund);
    ctx->ctas_cache[key] = v;
    return v;
  }
  return ctas_per_sm(ctx, g.W, g.H, g.NB);
}

magus_status encode_tmap(magus_ctx ctx, CUtensorMap* map, const float* x, int64_t N, int64_t T,
                         int64_t ld, uint32_t box_traces = 128) {
  if (!ctx->encode) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    if (!fn || q != cudaDriverEntryPointSuccess)
      return fail(ctx, MAGUS_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    ctx->encode = (PFN_cuTensorMapEncodeTiled_v12000)fn;
  }
  cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)T};
  cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
  cuuint32_t box[2] = {box_traces, 32};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = ctx->encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)x, dims, strides, box,
                           estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(ctx, MAGUS_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return MAGUS_OK;
}

// 1-D map over the digest table: one 16-B box (2 x u64) per decision word
magus_status encode_mul_tmap(magus_ctx ctx, CUtensorMap* map) {
  cuuint64_t dims[1] = {(cuuint64_t)(2 * ctx->mul_nw)};
  cuuint64_t strides[1] = {(cuuint64_t)(2 * ctx->mul_nw) * 8};  // rank 1: not read
  cuuint32_t box[1] = {2};
  cuuint32_t estr[1] = {1};
  CUresult r = ctx->encode(map, CU_TENSOR_MAP_DATA_TYPE_UINT64, 1, ctx->mul_dev, dims, strides, box, estr,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                           CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(ctx, MAGUS_ERR_CUDA, "digest tensor map failed (%d)", (int)r);
  return MAGUS_OK;
}

magus_status validate_replay(magus_ctx ctx, const float* traces, int64_t N, int64_t T, int64_t ld,
                             const magus_policy* params, int32_t C) {
  if (!traces) return fail(ctx, MAGUS_ERR_INVALID_ARG, "traces is NULL");
  if (N < 1 || N > ((int64_t)1 << 31) - 1) return fail(ctx, MAGUS_ERR_INVALID_ARG, "n_traces %lld out of range", (long long)N);
  if (T < 1 || T > kMaxSteps) return fail(ctx, MAGUS_ERR_INVALID_ARG, "n_steps %lld not in [1, 2^24]", (long long)T);
  if (ld < N) return fail(ctx, MAGUS_ERR_INVALID_ARG, "ld %lld < n_traces %lld", (long long)ld, (long long)N);
  if (!params || C < 1) return fail(ctx, MAGUS_ERR_INVALID_ARG, "no params");
  char msg[256];
  for (int32_t c = 0; c < C; ++c)
    if (!validate_policy(params[c], msg, sizeof msg))
      return fail(ctx, MAGUS_ERR_INVALID_ARG, "params[%d]: %s", c, msg);
  return MAGUS_OK;
}

}  // namespace

namespace magus {

static double u128_to_double(unsigned __int128 v) { return (double)v; }

void derive_totals(const DevPlatform& p, const uint64_t* w, magus_derived* out) {
  const uint64_t NT = w[MAGUS_TOT_N_STEPS];
  const uint64_t mint = w[MAGUS_TOT_MIN_INT];
  const unsigned __int128 qmin =
      ((unsigned __int128)w[MAGUS_TOT_QMIN_HI] << 32) + (unsigned __int128)w[MAGUS_TOT_QMIN_LO];
  const unsigned __int128 qmax =
      ((unsigned __int128)w[MAGUS_TOT_QMAX_HI] << 32) + (unsigned __int128)w[MAGUS_TOT_QMAX_LO];
  const unsigned __int128 qbase =
      ((unsigned __int128)w[MAGUS_TOT_QBASE_HI] << 32) + (unsigned __int128)w[MAGUS_TOT_QBASE_LO];
  const double ch = (double)w[MAGUS_TOT_CHANGES];
  const double time_max = p.dt * (double)(NT - mint) + p.cQ * u128_to_double(qmax);
  const double time_min = p.dt * (double)mint + p.cQ * u128_to_double(qmin);
  const double time = (p.dt * (double)NT + p.cQ * u128_to_double(qmin + qmax)) + p.t_sw * ch;
  const double energy = (p.P_max * time_max + p.P_min * time_min) + p.e_sw * ch;
  const double base_time = p.dt * (double)NT + p.cQ * u128_to_double(qbase);
  const double base_energy = p.P_max * base_time;
  out->energy_j = energy;
  out->time_s = time;
  out->base_energy_j = base_energy;
  out->base_time_s = base_time;
  out->saving = 1.0 - energy / base_energy;
  out->slowdown = time / base_time - 1.0;
  out->n_viol = (int64_t)w[MAGUS_TOT_N_VIOL];
  out->n_traces = (int64_t)w[MAGUS_TOT_N_TRACES];
  // Sec. 6.3: |A and B| / |A or B| with A = MAGUS bursts, B = max-uncore
  // bursts; A is a subset of B (B_l <= B_max), so this is sum A / sum B.
  const uint64_t uni = w[MAGUS_TOT_BURST_BASE], inter = w[MAGUS_TOT_BURST_MAGUS];
  out->jaccard = uni ? (double)inter / (double)uni : 1.0;
}

}  // namespace magus

extern "C" {

int32_t magus_abi_version(void) { return MAGUS_ABI_VERSION; }

const char* magus_status_string(magus_status s) {
  switch (s) {
    case MAGUS_OK: return "ok";
    case MAGUS_ERR_INVALID_ARG: return "invalid argument";
    case MAGUS_ERR_NOT_INITIALIZED: return "not initialized";
    case MAGUS_ERR_CUDA: return "CUDA error";
    case MAGUS_ERR_NCCL: return "NCCL error";
    case MAGUS_ERR_OOM: return "out of device memory";
    case MAGUS_ERR_UNSUPPORTED: return "unsupported";
    case MAGUS_ERR_NO_FEASIBLE: return "no feasible config";
  }
  return "unknown status";
}

const char* magus_last_error(magus_ctx ctx) { return ctx ? ctx->err.c_str() : "NULL context"; }

magus_status magus_policy_preset(int32_t id, magus_policy* out) {
  if (!out) return MAGUS_ERR_INVALID_ARG;
  magus_policy p;
  p.window = 10;        // reading R4
  p.history = 10;       // P@24182
  p.deriv_len = 10.0;   // reading R4: L = W
  p.tau_dec = -500.0;   // P@25197 "500", signed per reading R1
  p.t_hi = 0.4;         // P@25197
  p.variant = 0;        // the paper's MAGUS
  p.step = 0;
  if (id == MAGUS_POLICY_PAPER_DEFAULT) p.tau_inc = 200.0;       // P@25197 (Sec. 3.3)
  else if (id == MAGUS_POLICY_PAPER_PARETO) p.tau_inc = 300.0;   // P@44170 (Sec. 6.4)
  else return MAGUS_ERR_INVALID_ARG;
  *out = p;
  return MAGUS_OK;
}

magus_status magus_platform_preset(int32_t id, magus_platform* out) {
  if (!out) return MAGUS_ERR_INVALID_ARG;
  magus_platform p;
  p.ratio_min = 8;            // 0.8 GHz (P@29320 / P@29831)
  if (id == MAGUS_PLATFORM_INTEL_A100) p.ratio_max = 22;          // 2.2 GHz, P@29320
  else if (id == MAGUS_PLATFORM_INTEL_MAX1550) p.ratio_max = 25;  // 2.5 GHz, P@29831
  else return MAGUS_ERR_INVALID_ARG;
  p.dt_s = 0.2;               // P@44789
  p.bw_max_mbs = 32000.0;     // model-M assumption
  p.beta = 1.0;               // model-M assumption
  p.p_other_w = 218.0;        // 118 W CPU at min uncore (Fig. 2) + 100 W board (assumption)
  p.p_unc_min_w = 0.0;
  p.p_unc_max_w = 82.0;       // Fig. 2: 200 W -> 120 W (P@12253)
  p.e_switch_j = 0.0;         // "negligible" (P@27899)
  p.t_switch_s = 0.0;
  p.slowdown_bound = 0.05;    // P@1715
  p.burst_mbs = 0.0;          // Sec. 6.3 Jaccard counters off by default (theta not printed)
  *out = p;
  return MAGUS_OK;
}

static const double kGridInc[4] = {100.0, 200.0, 300.0, 400.0};
static const double kGridDec[4] = {-250.0, -500.0, -750.0, -1000.0};
static const double kGridHi[4] = {0.2, 0.3, 0.4, 0.5};
static const int32_t kGridW[4] = {4, 6, 10, 16};

magus_status magus_grid_sweep256(magus_policy out[256]) {
  if (!out) return MAGUS_ERR_INVALID_ARG;
  for (int iW = 0; iW < 4; ++iW)
    for (int iHi = 0; iHi < 4; ++iHi)
      for (int iDec = 0; iDec < 4; ++iDec)
        for (int iInc = 0; iInc < 4; ++iInc) {
          magus_policy& p = out[iInc + 4 * (iDec + 4 * (iHi + 4 * iW))];
          p.window = kGridW[iW];
          p.history = 10;
          p.deriv_len = (double)kGridW[iW];
          p.tau_inc = kGridInc[iInc];
          p.tau_dec = kGridDec[iDec];
          p.t_hi = kGridHi[iHi];
        p.variant = 0;
        p.step = 0;
        }
  return MAGUS_OK;
}

magus_status magus_grid_fleet64(magus_policy out[64]) {
  if (!out) return MAGUS_ERR_INVALID_ARG;
  for (int iHi = 0; iHi < 4; ++iHi)
    for (int iDec = 0; iDec < 4; ++iDec)
      for (int iInc = 0; iInc < 4; ++iInc) {
        magus_policy& p = out[iInc + 4 * (iDec + 4 * iHi)];
        p.window = 10;
        p.history = 10;
        p.deriv_len = 10.0;
        p.tau_inc = kGridInc[iInc];
        p.tau_dec = kGridDec[iDec];
        p.t_hi = kGridHi[iHi];
        p.variant = 0;
        p.step = 0;
      }
  return MAGUS_OK;
}

magus_status magus_policy_inspect(const magus_policy* p, magus_policy_consts* out) {
  char msg[256];
  if (!p || !out || !validate_policy(*p, msg, sizeof msg)) return MAGUS_ERR_INVALID_ARG;
  const DevPolicy d = make_dev_policy(*p);
  out->delta_inc = d.d_inc;
  out->delta_dec = d.d_dec;
  out->k_hi = d.k;
  out->reserved = 0;
  return MAGUS_OK;
}

magus_status magus_platform_inspect(const magus_platform* p, magus_platform_consts* out) {
  char msg[256];
  if (!p || !out || !validate_platform(*p, msg, sizeof msg)) return MAGUS_ERR_INVALID_ARG;
  const DevPlatform d = make_dev_platform(*p);
  out->x_stretch_min = d.xthr_min;
  out->x_stretch_max = d.xthr_max;
  out->inv_cap_min = d.invB_min;
  out->inv_cap_max = d.invB_max;
  out->p_min_w = d.P_min;
  out->p_max_w = d.P_max;
  return MAGUS_OK;
}

magus_status magus_init(magus_ctx* out, int device, void* cuda_stream, const magus_platform* plat) {
  if (!out || !plat) return MAGUS_ERR_INVALID_ARG;
  *out = nullptr;
  char msg[256];
  if (!validate_platform(*plat, msg, sizeof msg)) return MAGUS_ERR_INVALID_ARG;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    return MAGUS_ERR_CUDA;
  }
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return MAGUS_ERR_CUDA;
  if (prop.major != 10) return MAGUS_ERR_UNSUPPORTED;  // built for sm_100a only
  magus_ctx ctx = new magus_ctx_s();
  ctx->device = device;
  ctx->stream = (cudaStream_t)cuda_stream;
  ctx->plat = *plat;
  ctx->dplat = make_dev_platform(*plat);
  ctx->sms = prop.multiProcessorCount;
  *out = ctx;
  return MAGUS_OK;
}

magus_status magus_destroy(magus_ctx ctx) {
  if (!ctx) return MAGUS_ERR_INVALID_ARG;
  {
    DeviceGuard dg(ctx->device);
    cudaStreamSynchronize(ctx->stream);
    if (ctx->scratch) cudaFree(ctx->scratch);
    if (ctx->pol_dev) cudaFree(ctx->pol_dev);
    if (ctx->pol_host) cudaFreeHost(ctx->pol_host);
    if (ctx->best_pinned) cudaFreeHost(ctx->best_pinned);
    if (ctx->lam_dev) cudaFree(ctx->lam_dev);
    if (ctx->mul_dev) cudaFree(ctx->mul_dev);
    if (ctx->trace_dev) cudaFree(ctx->trace_dev);
    if (ctx->sweep_dev) cudaFree(ctx->sweep_dev);
    if (ctx->stage_dev) cudaFree(ctx->stage_dev);
    if (ctx->pol_copied) cudaEventDestroy(ctx->pol_copied);
    for (auto& pr : ctx->pending) {
      cudaEventDestroy(pr.first);
      cudaEventDestroy(pr.second);
    }
    for (auto e : ctx->event_pool) cudaEventDestroy(e);
    if (ctx->comm) nccl_comm_destroy(ctx->comm);
  }
  delete ctx;
  return MAGUS_OK;
}

magus_status magus_set_stream(magus_ctx ctx, void* cuda_stream) {
  if (!ctx) return MAGUS_ERR_INVALID_ARG;
  ctx->stream = (cudaStream_t)cuda_stream;
  return MAGUS_OK;
}

magus_status magus_set_option(magus_ctx ctx, int32_t key, int64_t value) {
  if (!ctx) return MAGUS_ERR_INVALID_ARG;
  switch (key) {
    case MAGUS_OPT_KERNEL:
      if (value < 0 || value > 5) return fail(ctx, MAGUS_ERR_INVALID_ARG, "kernel option %lld", (long long)value);
      ctx->opt_kernel = value;
      return MAGUS_OK;
    case MAGUS_OPT_SEGMENTS:
      if (value < 0) return fail(ctx, MAGUS_ERR_INVALID_ARG, "segments < 0");
      ctx->opt_segments = value;
      return MAGUS_OK;
    case MAGUS_OPT_TIMING:
      ctx->opt_timing = value ? 1 : 0;
      return MAGUS_OK;
    case MAGUS_OPT_SPEC_WARM:
      if (value < 0 || value > (int64_t(1) << 24)) return fail(ctx, MAGUS_ERR_INVALID_ARG, "spec warm-up out of range");
      ctx->opt_spec_warm = value;
      return MAGUS_OK;
    case MAGUS_OPT_BUNDLE:
      if (value != 0 && value != 1 && value != 2 && value != 4)
        return fail(ctx, MAGUS_ERR_INVALID_ARG, "bundle option must be 0, 1, 2 or 4");
      ctx->opt_bundle = value;
      return MAGUS_OK;
    case MAGUS_OPT_TRACE:
      ctx->opt_trace = value ? 1 : 0;
      return MAGUS_OK;
    case MAGUS_OPT_NARROW:
      ctx->opt_narrow = value ? 1 : 0;
      return MAGUS_OK;
    case MAGUS_OPT_WALK1:
      ctx->opt_walk1 = value ? 1 : 0;
      return MAGUS_OK;
    case MAGUS_OPT_FAMILY:
      ctx->opt_family = value ? 1 : 0;
      return MAGUS_OK;
    case MAGUS_OPT_WAVES:
      if (value < 0 || value > 64) return fail(ctx, MAGUS_ERR_INVALID_ARG, "waves not in [0, 64]");
      ctx->opt_waves = value;
      return MAGUS_OK;
  }
  return fail(ctx, MAGUS_ERR_INVALID_ARG, "unknown option %d", key);
}

// time-chunked replay (magus_replay_resume): buffer row r = global interval
// tb + r, output from row ts on, state = caller's resume state
struct ResumeArgs {
  int64_t tb, ts;
  void* state;
};

static magus_status replay_impl(magus_ctx ctx, const float* traces, int64_t N, int64_t T,
                                int64_t ld, const magus_policy* params, int32_t C,
                                magus_summary* out_summary, magus_base* out_base,
                                uint32_t* out_decisions, uint64_t* out_totals, uint8_t* out_levels,
                                const ResumeArgs* rs = nullptr) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  magus_status st = validate_replay(ctx, traces, N, T, ld, params, C);
  if (st != MAGUS_OK) return st;
  const int64_t tb = rs ? rs->tb : 0, ts = rs ? rs->ts : 0;
  if (tb + T > kMaxSteps)
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "t_base + n_rows %lld exceeds 2^24", (long long)(tb + T));
  DeviceGuard dg(ctx->device);
  cudaGetLastError();

  // kernel choice: the stream kernel runs the paper's MAGUS (variant 0) with
  // W <= 33, H <= 32 on TMA-addressable traces; everything else, and any
  // per-interval level output, runs the per-sample kernel
  bool all_stream = out_levels == nullptr, multi = false, closed = false, all_seq = true, all_spec = true;
  for (int32_t c = 0; c < C; ++c) {
    all_stream = all_stream && params[c].variant == 0 &&
                 stream_supported(params[c].window, params[c].history);
    multi = multi || (params[c].variant & MAGUS_VARIANT_GRADUAL) != 0;
    closed = closed || (params[c].variant & MAGUS_VARIANT_CLOSED_LOOP) != 0;
    all_seq = all_seq && seq_supported(params[c]);
    all_spec = all_spec && spec_supported(params[c]);
  }
  const bool tma_ok = ((uintptr_t)traces % 16 == 0) && (ld % 4 == 0);
  all_seq = all_seq && ld < (int64_t(1) << 26)  // the sequential kernel's 32-bit row offsets
            && seq_fits(ctx->dplat, closed, multi);  // per-ratio rows of wide ratio ranges
  int kernel = (int)ctx->opt_kernel;
  // open loop (no closed-loop config): the time-segmented walk kernel
  const bool walk_ok = !closed && ld < (int64_t(1) << 26);  // 32-bit row offsets of a 32-step word
  // closed loop: the sequential kernel (the speculative kernel 5 is opt-in:
  // at config 2 it measured 3.7 ms vs 3.1 ms)
  if (kernel == 0) kernel = (all_stream && tma_ok) ? 2 : (walk_ok ? 4 : (all_seq ? 3 : (all_spec ? 5 : 1)));
  if (kernel == 5 && !all_spec)
    return fail(ctx, MAGUS_ERR_UNSUPPORTED,
                "speculative kernel: closed-loop jump configs only (variant 1), W <= 65");
  if (kernel == 4 && !walk_ok)
    return fail(ctx, MAGUS_ERR_UNSUPPORTED,
                "walk kernel: closed-loop configs (variant 1, 3) have no exact time segmentation; ld < 2^26");
  if (kernel == 3 && !all_seq)
    return fail(ctx, MAGUS_ERR_UNSUPPORTED,
                "sequential kernel: closed-loop configs need W <= 64 (jump) or W <= 128 (gradual), "
                "ld < 2^26, and a ratio range whose per-ratio rows fit in shared memory");
  if (kernel == 2 && !(all_stream && tma_ok))
    return fail(ctx, MAGUS_ERR_UNSUPPORTED,
                "stream kernel needs W in [2,33], H in [1,32], 16-B aligned traces and ld %% 4 == 0");
  if (rs && kernel != 2)
    return fail(ctx, MAGUS_ERR_UNSUPPORTED,
                "time-chunked replay runs on the stream kernel only (variant 0, W in [2,33], "
                "H in [1,32], 16-B aligned traces, ld %% 4 == 0)");

  st = upload_policies(ctx, params, C);
  if (st != MAGUS_OK) return st;

  const int64_t Tr = T - ts;            // rows this call replays
  const int64_t nw = (Tr + 31) / 32;     // decision words written
  int64_t nseg = 1, seg_len = ((Tr + 31) / 32) * 32;
  if (kernel == 2) {
    const int64_t ngroups = (N + 127) / 128;
    bool packed = false;  // NB > 1 packs per-segment counters in 16 bits
    for (auto& g : ctx->groups) packed = packed || g.NB > 1;
    if (ctx->opt_segments > 0) {
      nseg = ctx->opt_segments;
    } else if (ctx->opt_waves == 0) {
      // Wave model: the launches of the W groups run back to back and every
      // CTA of a launch streams one segment, so a launch takes
      // ceil(CTAs / resident slots) rounds of (segment + halo + fixed epilogue)
      // steps.  Pick the segment count with the smallest modelled total
      // (fewer segments on ties: less halo re-read and look-back).
      const int64_t words = (Tr + 31) / 32;
      const int64_t lo = packed ? (words * 32 + 65503) / 65504 : 1;
      const int64_t hi = std::max<int64_t>(lo, std::min<int64_t>(words / 16, 4096));  // >= 512 steps
      double best_cost = 0.0;
      nseg = lo;
      for (int64_t cand = lo; cand <= hi; ++cand) {
        const int64_t len = ((Tr + cand - 1) / cand + 31) / 32 * 32;
        if ((Tr + len - 1) / len != cand) continue;  // not realisable with 32-step segments
        double cost = 0.0;
        for (auto& g : ctx->groups) {
          const int64_t slots = (int64_t)ctx->sms * std::max(1, group_ctas_per_sm(ctx, g));
          const int64_t ctas = group_ctas(ctx, N, g, cand);
          const int64_t halo = cand > 1 ? ((g.W + g.H - 1 + 31) / 32) * 32 : 0;
          cost += (double)((ctas + slots - 1) / slots) * (double)(len + halo + 96);
        }
        if (cand == lo || cost < best_cost * 0.999) {
          best_cost = cost;
          nseg = cand;
        }
      }
    } else {
      int per_sm = 1 << 30;
      int64_t nbund = 0;
      for (auto& g : ctx->groups) {
        per_sm = std::min(per_sm, group_ctas_per_sm(ctx, g));
        nbund += g.nbund;
      }
      if (per_sm < 1) per_sm = 1;
      const int64_t slots = (int64_t)ctx->sms * per_sm * ctx->opt_waves;
      nseg = std::max<int64_t>(1, (slots + ngroups * nbund - 1) / (ngroups * nbund));
    }
    seg_len = ((Tr + nseg - 1) / nseg + 31) / 32 * 32;
    if (packed && seg_len > 65504) seg_len = 65504;
    const int64_t min_len = 512;  // keeps the halo re-read below ~6 %
    if (ctx->opt_segments == 0 && seg_len < min_len) seg_len = std::min<int64_t>(min_len, ((Tr + 31) / 32) * 32);
    nseg = (Tr + seg_len - 1) / seg_len;
  }
  const int64_t ngroups = (N + 127) / 128;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  if (ctx->opt_timing) {
    ev0 = take_event(ctx);
    ev1 = take_event(ctx);
  }
  int launched = 0;
  if (kernel == 5) {
    // segments: ~2 waves of resident threads, each >= 1024 rounds; each
    // speculation replays `warm` rounds before its segment
    if (ctx->opt_segments > 0) {
      nseg = ctx->opt_segments;
    } else {
      const int64_t target = (int64_t)ctx->sms * 1024 * 2;
      nseg = std::max<int64_t>(1, (target + N * C - 1) / (N * C));
      nseg = std::min<int64_t>(nseg, std::max<int64_t>(1, T / 1024));
    }
    nseg = std::min<int64_t>(std::max<int64_t>(nseg, 1), 65535);
    seg_len = ((T + nseg - 1) / nseg + 31) / 32 * 32;
    nseg = (T + seg_len - 1) / seg_len;
    const int64_t warm = ctx->opt_spec_warm > 0 ? ctx->opt_spec_warm : std::min<int64_t>(seg_len, 1024);  // measured best
    const size_t sum_bytes = out_summary ? 0 : align_up(sizeof(magus_summary) * (size_t)(N * C), 256);
    const size_t base_bytes = (out_base || !out_totals) ? 0 : align_up(sizeof(magus_base) * (size_t)N, 256);
    st = ensure_scratch(ctx, sum_bytes + base_bytes + spec_scratch_bytes(N, C, nseg) + 256);
    if (st != MAGUS_OK) return st;
    ctx->work_sig = 0;  // scratch reused: the stream path must re-zero its counters
    char* sp = (char*)ctx->scratch;
    magus_summary* summ = out_summary;
    if (!summ) { summ = (magus_summary*)sp; sp += sum_bytes; }
    magus_base* base = out_base;
    if (!base && out_totals) { base = (magus_base*)sp; sp += base_bytes; }
    if (ctx->opt_timing) CK(cudaEventRecord(ev0, ctx->stream));
    bool wide = false;
    for (int32_t c = 0; c < C; ++c) wide = wide || params[c].history > 32 || params[c].window > 33;
    int r = launch_spec(ctx->stream, traces, N, T, ld, dev_policies(ctx), C, wide, ctx->dplat, nseg, seg_len, warm, sp,
                        summ, base, out_decisions, out_levels, &ctx->spec_reruns);
    if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "spec kernel launch");
    launched += r;
    ctx->last_grid = ((N + 127) / 128) * nseg * C;
    if (ctx->opt_timing) CK(cudaEventRecord(ev1, ctx->stream));
    if (out_totals) {
      r = launch_totals(ctx->stream, summ, base, N, T, C, out_totals);
      if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "totals kernel launch");
      launched += r;
    }
  } else if (kernel == 4) {
    // segments: enough independent (trace, segment, config) chains for about
    // two full waves of resident threads, each >= 256 steps (halo re-read
    // and map composition stay a few per cent)
    if (ctx->opt_segments > 0) {
      nseg = ctx->opt_segments;
    } else {
      const int64_t target = (int64_t)ctx->sms * 2048 * 2;
      nseg = std::max<int64_t>(1, (target + N * C - 1) / (N * C));
      nseg = std::min<int64_t>(nseg, std::max<int64_t>(1, T / 256));
    }
    nseg = std::min<int64_t>(std::max<int64_t>(nseg, 1), 65535);
    seg_len = ((T + nseg - 1) / nseg + 31) / 32 * 32;
    nseg = (T + seg_len - 1) / seg_len;
    const size_t sum_bytes = out_summary ? 0 : align_up(sizeof(magus_summary) * (size_t)(N * C), 256);
    const size_t base_bytes = (out_base || !out_totals) ? 0 : align_up(sizeof(magus_base) * (size_t)N, 256);
    const size_t walk_bytes = walk_scratch_bytes(N, C, T, nseg, ctx->dplat);
    int32_t max_H = 1, same_W = params[0].window;
    for (int32_t c = 0; c < C; ++c) {
      max_H = std::max(max_H, params[c].history);
      if (params[c].window != same_W) same_W = 0;
    }
    st = ensure_scratch(ctx, sum_bytes + base_bytes + walk_bytes + 256);
    if (st != MAGUS_OK) return st;
    ctx->work_sig = 0;  // scratch reused: the stream path must re-zero its counters
    char* sp = (char*)ctx->scratch;
    magus_summary* summ = out_summary;
    if (!summ) { summ = (magus_summary*)sp; sp += sum_bytes; }
    magus_base* base = out_base;
    if (!base && out_totals) { base = (magus_base*)sp; sp += base_bytes; }
    if (ctx->opt_timing) CK(cudaEventRecord(ev0, ctx->stream));
    const double p_lo = ctx->plat.p_other_w + ctx->plat.p_unc_min_w;
    const double p_span = ctx->plat.p_unc_max_w - ctx->plat.p_unc_min_w;
    int r = launch_walk(ctx->stream, traces, N, T, ld, dev_policies(ctx), C, max_H, ctx->dplat, ctx->plat.bw_max_mbs,
                        p_lo, p_span, nseg, seg_len, sp, summ, base, out_decisions, out_levels, ctx->opt_walk1 != 0, same_W);
    if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "walk kernel launch");
    launched += r;
    ctx->last_grid = ((N + 127) / 128) * nseg * C;
    if (ctx->opt_timing) CK(cudaEventRecord(ev1, ctx->stream));
    if (out_totals) {
      r = launch_totals(ctx->stream, summ, base, N, T, C, out_totals);
      if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "totals kernel launch");
      launched += r;
    }
  } else if (kernel == 1 || kernel == 3) {
    // the per-sample kernels write summaries directly; totals need them
    const size_t sum_bytes = (out_summary || !out_totals) ? 0 : align_up(sizeof(magus_summary) * (size_t)(N * C), 256);
    const size_t base_bytes = (out_base || !out_totals) ? 0 : align_up(sizeof(magus_base) * (size_t)N, 256);
    st = ensure_scratch(ctx, sum_bytes + base_bytes + 256);
    if (st != MAGUS_OK) return st;
    ctx->work_sig = 0;  // scratch reused: the stream path must re-zero its counters
    char* sp = (char*)ctx->scratch;
    magus_summary* summ = out_summary;
    if (!summ && out_totals) { summ = (magus_summary*)sp; sp += sum_bytes; }
    magus_base* base = out_base;
    if (!base && out_totals) base = (magus_base*)sp;
    if (ctx->opt_timing) CK(cudaEventRecord(ev0, ctx->stream));
    const double p_lo = ctx->plat.p_other_w + ctx->plat.p_unc_min_w;
    const double p_span = ctx->plat.p_unc_max_w - ctx->plat.p_unc_min_w;
    int r;
    if (kernel == 3) {
      r = launch_seq(ctx->stream, traces, N, T, ld, dev_policies(ctx), C, ctx->dplat,
                     ctx->plat.bw_max_mbs, p_lo, p_span, closed, multi, summ, base, out_decisions,
                     out_levels);
      ctx->last_grid = (N * C + 31) / 32;
    } else {
      r = launch_reference(ctx->stream, traces, N, T, ld, dev_policies(ctx), C, ctx->dplat,
                           ctx->plat.bw_max_mbs, p_lo, p_span, multi,
                           /*literal=*/ctx->opt_kernel == 1, summ, base, out_decisions, out_levels);
      ctx->last_grid = (N * C + 127) / 128;
    }
    if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "per-sample kernel launch");
    launched += r;
    if (ctx->opt_timing) CK(cudaEventRecord(ev1, ctx->stream));
    if (out_totals) {
      r = launch_totals(ctx->stream, summ, base, N, T, C, out_totals);
      if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "totals kernel launch");
      launched += r;
    }
  } else {
    // scratch of the fused kernel: counters + accumulators (zero, self-cleaning)
    // followed by the epoch-tagged segment status words
    const size_t off_arrive = 256;
    const size_t off_tarrive = off_arrive + align_up(4 * (size_t)(C * ((N + 31) / 32)), 256);  // any CTA width
    const size_t off_tacc = off_tarrive + align_up(4 * (size_t)C, 256);
    const size_t off_acc = off_tacc + align_up(8 * kTotAccWords * (size_t)C, 256);
    const size_t off_status = off_acc + align_up(8 * (size_t)kAccFields * (size_t)(C * N), 256);
    const size_t total = off_status + align_up(4 * (size_t)(C * nseg) * (size_t)N, 256);
    st = ensure_scratch(ctx, total);
    if (st != MAGUS_OK) return st;
    const uint64_t sig = ((uint64_t)C * 1000003ULL + (uint64_t)N) * 1000033ULL + (uint64_t)nseg + 1;
    if (sig != ctx->work_sig) {
      // the whole region, status words included: another kernel path (walk,
      // seq, reference) may have left arbitrary words in this scratch, and a
      // look-back accepts any word whose tag equals the epoch
      CK(cudaMemsetAsync(ctx->scratch, 0, total, ctx->stream));
      ctx->work_sig = sig;
    }
    if (++ctx->epoch >= (1u << 29)) {
      CK(cudaMemsetAsync(ctx->scratch, 0, total, ctx->stream));
      ctx->epoch = 1;
    }
    char* sp = (char*)ctx->scratch;
    StreamWork wk;
    wk.ticket = (uint32_t*)sp;
    wk.done = (uint32_t*)sp + 1;
    wk.arrive = (uint32_t*)(sp + off_arrive);
    wk.tarrive = (uint32_t*)(sp + off_tarrive);
    wk.tacc = (unsigned long long*)(sp + off_tacc);
    wk.acc = (unsigned long long*)(sp + off_acc);
    wk.status = (uint32_t*)(sp + off_status);
    wk.epoch = ctx->epoch;
    wk.summary = out_summary;
    wk.base = out_base;
    wk.dec = out_decisions;
    wk.dec_cstride = nw * N;
    wk.totals = out_totals;
    wk.tb = (int32_t)tb;       // global interval of buffer row 0
    wk.ts = (int32_t)(tb + ts);  // first interval decided (global)
    wk.carry = nullptr;
    ctx->trace_n = 0;
    if (ctx->opt_trace || ctx->trace_armed) {  // the timeline address (or NULL) in scratch
      void* tp = nullptr;
      if (ctx->opt_trace) {
        int64_t grid_all = 0;
        for (auto& g : ctx->groups) grid_all += group_ctas(ctx, N, g, nseg);
        if (grid_all > ctx->trace_cap) {
          CK(cudaStreamSynchronize(ctx->stream));
          if (ctx->trace_dev) cudaFree(ctx->trace_dev);
          ctx->trace_dev = nullptr;
          ctx->trace_cap = 0;
          CK(cudaMalloc(&ctx->trace_dev, 64 * (size_t)grid_all));
          ctx->trace_cap = grid_all;
        }
        tp = ctx->trace_dev;
        ctx->trace_n = grid_all;
      }
      ctx->trace_slot_host[0] = tp;   // (a pageable source is staged before the call returns)
      CK(cudaMemcpyAsync((uint32_t*)sp + kTraceSlotWords, &ctx->trace_slot_host[ctx->opt_trace ? 0 : 1],
                         sizeof(void*), cudaMemcpyHostToDevice, ctx->stream));
      ctx->trace_armed = ctx->opt_trace != 0;
    }
    if (rs) {  // accumulators and carries live in the caller's state
      wk.acc = (unsigned long long*)rs->state;
      wk.carry = (uint32_t*)((char*)rs->state + 8 * (size_t)kAccFields * (size_t)(C * N));
    }
    const int64_t nw_glob = (tb + T + 31) / 32;  // digest words are global
    if (nw_glob > ctx->mul_nw) {  // the table depends on w only: grow it once, keep it
      CK(cudaStreamSynchronize(ctx->stream));
      if (ctx->mul_dev) cudaFree(ctx->mul_dev);
      ctx->mul_dev = nullptr;
      ctx->mul_nw = 0;
      const int64_t cap = std::max<int64_t>(nw_glob, 4096);
      CK(cudaMalloc(&ctx->mul_dev, 2 * sizeof(unsigned long long) * (size_t)cap));
      if (launch_digest_table(ctx->stream, (unsigned long long*)ctx->mul_dev, cap) < 0)
        return cuda_fail(ctx, cudaGetLastError(), "digest table launch");
      ctx->launches += 1;
      ctx->mul_nw = cap;
    }
    wk.mul = (const unsigned long long*)ctx->mul_dev;
    CUtensorMap map, map_mul, map32;
    st = encode_tmap(ctx, &map, traces, N, T, ld);
    if (st != MAGUS_OK) return st;
    bool any_family = false;
    for (auto& g : ctx->groups) any_family = any_family || use_family(ctx, g);
    if (any_family) {
      st = encode_tmap(ctx, &map32, traces, N, T, ld, (uint32_t)family_cta_traces());
      if (st != MAGUS_OK) return st;
    }
    st = encode_mul_tmap(ctx, &map_mul);
    if (st != MAGUS_OK) return st;
    if (ctx->opt_timing) CK(cudaEventRecord(ev0, ctx->stream));
    int64_t grid_total = 0;
    ctx->last_family = 0;
    for (auto& g : ctx->groups)  // one launch per group: its CTAs index grid.x
      if (group_ctas(ctx, N, g, nseg) > (int64_t)INT32_MAX)
        return fail(ctx, MAGUS_ERR_UNSUPPORTED, "%lld CTAs in one launch exceed the grid limit; replay fewer traces",
                    (long long)group_ctas(ctx, N, g, nseg));
    for (size_t gi = 0; gi < ctx->groups.size(); ++gi) {
      auto& g = ctx->groups[gi];
      int grid = 0;
      int r = use_family(ctx, g)
                  ? launch_family(ctx->stream, &map32, &map_mul, N, tb + T, dev_policies(ctx), dev_cidx(ctx, g.off),
                                  g.nbund, g.H, g.fam, ctx->dplat, nseg, seg_len, wk, &grid)
                  : launch_stream(ctx->stream, &map, &map_mul, N, tb + T, dev_policies(ctx), dev_cidx(ctx, g.off),
                                  g.nbund, g.NB, g.W, g.H, ctx->dplat, nseg, seg_len, wk, ctx->opt_narrow != 0, &grid);
      if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "stream kernel launch");
      launched += r;
      grid_total += grid;
      if (use_family(ctx, g)) ctx->last_family += 1;
    }
    ctx->last_grid = grid_total;
    if (ctx->opt_timing) CK(cudaEventRecord(ev1, ctx->stream));
  }
  if (ctx->opt_timing) ctx->pending.push_back({ev0, ev1});
  ctx->launches += launched;
  ctx->last_segments = nseg;
  ctx->last_kernel = kernel;
  if (kernel != 2) ctx->last_family = 0;
  return MAGUS_OK;
}

magus_status magus_replay(magus_ctx ctx, const float* traces, int64_t N, int64_t T, int64_t ld,
                          const magus_policy* params, int32_t C, magus_summary* out_summary,
                          magus_base* out_base, uint32_t* out_decisions, uint64_t* out_totals) {
  return replay_impl(ctx, traces, N, T, ld, params, C, out_summary, out_base, out_decisions,
                     out_totals, nullptr);
}

static int64_t resume_halo_rows(const magus_policy* params, int32_t C) {
  int64_t h = 0;
  for (int32_t c = 0; c < C; ++c)
    h = std::max<int64_t>(h, ((int64_t)params[c].window + params[c].history - 1 + 31) / 32 * 32);
  return h;
}

magus_status magus_resume_state_bytes(int64_t n_traces, int32_t n_params, size_t* out) {
  if (!out || n_traces < 1 || n_params < 1) return MAGUS_ERR_INVALID_ARG;
  *out = resume_state_bytes(n_traces, n_params);
  return MAGUS_OK;
}

magus_status magus_resume_halo(const magus_policy* params, int32_t n_params, int64_t* rows) {
  if (!params || n_params < 1 || !rows) return MAGUS_ERR_INVALID_ARG;
  char msg[256];
  for (int32_t c = 0; c < n_params; ++c)
    if (!validate_policy(params[c], msg, sizeof msg)) return MAGUS_ERR_INVALID_ARG;
  *rows = resume_halo_rows(params, n_params);
  return MAGUS_OK;
}

magus_status magus_replay_resume(magus_ctx ctx, const float* traces, int64_t N, int64_t n_rows,
                                 int64_t ld, int64_t t_base, int64_t t_start,
                                 const magus_policy* params, int32_t C, void* state,
                                 magus_summary* out_summary, magus_base* out_base,
                                 uint32_t* out_decisions, uint64_t* out_totals) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!state || (uintptr_t)state % 8 != 0)
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "state must be a non-NULL, 8-byte aligned device buffer");
  if (t_base < 0 || t_base % 32 != 0 || t_start % 32 != 0)
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "t_base and t_start must be non-negative multiples of 32");
  if (t_start < t_base || t_start >= t_base + n_rows)
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "t_start %lld outside the buffer [%lld, %lld)",
                (long long)t_start, (long long)t_base, (long long)(t_base + n_rows));
  if (params && C >= 1) {
    const int64_t halo = std::min<int64_t>(t_start, resume_halo_rows(params, C));
    if (t_start - t_base < halo)
      return fail(ctx, MAGUS_ERR_INVALID_ARG,
                  "the buffer must hold the %lld rows before t_start (t_base <= %lld)",
                  (long long)halo, (long long)(t_start - halo));
  }
  const ResumeArgs rs{t_base, t_start - t_base, state};
  return replay_impl(ctx, traces, N, n_rows, ld, params, C, out_summary, out_base, out_decisions,
                     out_totals, nullptr, &rs);
}

magus_status magus_replay_levels(magus_ctx ctx, const float* traces, int64_t N, int64_t T,
                                 int64_t ld, const magus_policy* params, int32_t C,
                                 uint8_t* out_levels, magus_summary* out_summary,
                                 uint64_t* out_totals) {
  if (ctx && !out_levels) return fail(ctx, MAGUS_ERR_INVALID_ARG, "out_levels is NULL");
  if (ctx && ctx->opt_kernel == 2)
    return fail(ctx, MAGUS_ERR_UNSUPPORTED, "per-interval levels come from the per-sample kernel");
  return replay_impl(ctx, traces, N, T, ld, params, C, out_summary, nullptr, nullptr, out_totals,
                     out_levels);
}

magus_status magus_offline_bound(magus_ctx ctx, const float* traces, int64_t N, int64_t T,
                                 int64_t ld, const double* lambdas, int32_t nl, int32_t full_grid,
                                 double* out) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!traces || !out || !lambdas || nl < 1 || N < 1 || T < 1 || T > kMaxSteps || ld < N)
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "bad offline_bound arguments");
  for (int32_t j = 0; j < nl; ++j)
    if (!(lambdas[j] >= 0.0) || !std::isfinite(lambdas[j]))
      return fail(ctx, MAGUS_ERR_INVALID_ARG, "lambda[%d] must be finite and >= 0", j);
  if (full_grid && ctx->plat.ratio_max - ctx->plat.ratio_min + 1 > 32)
    return fail(ctx, MAGUS_ERR_UNSUPPORTED, "the full grid supports at most 32 levels");
  DeviceGuard dg(ctx->device);
  const size_t need = sizeof(double) * (size_t)nl;
  if (need > ctx->lam_bytes) {
    CK(cudaStreamSynchronize(ctx->stream));
    if (ctx->lam_dev) cudaFree(ctx->lam_dev);
    ctx->lam_dev = nullptr;
    CK(cudaMalloc(&ctx->lam_dev, need));
    ctx->lam_bytes = need;
  }
  // pageable source: returns once staged, so `lambdas` may be reused at once
  CK(cudaMemcpyAsync(ctx->lam_dev, lambdas, need, cudaMemcpyHostToDevice, ctx->stream));
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  if (ctx->opt_timing) {  // the DP kernel alone (MAGUS_OPT_TIMING)
    ev0 = take_event(ctx);
    ev1 = take_event(ctx);
    CK(cudaEventRecord(ev0, ctx->stream));
  }
  const int r = launch_bound(ctx->stream, traces, N, T, ld, (const double*)ctx->lam_dev, nl, full_grid != 0,
                             ctx->dplat, ctx->plat.bw_max_mbs, ctx->plat.p_other_w + ctx->plat.p_unc_min_w,
                             ctx->plat.p_unc_max_w - ctx->plat.p_unc_min_w, out);
  if (r < 0) return cuda_fail(ctx, cudaGetLastError(), "bound kernel launch");
  if (ctx->opt_timing) {
    CK(cudaEventRecord(ev1, ctx->stream));
    ctx->pending.push_back({ev0, ev1});
  }
  ctx->launches += r;
  return MAGUS_OK;
}

magus_status magus_replay_host(magus_ctx ctx, const float* traces_host, int64_t N, int64_t T,
                               int64_t ld, const magus_policy* params, int32_t C,
                               magus_summary* summary_host, magus_base* base_host,
                               uint32_t* decisions_host, uint64_t* totals_host) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  magus_status st = validate_replay(ctx, traces_host, N, T, ld, params, C);
  if (st != MAGUS_OK) return st;
  DeviceGuard dg(ctx->device);
  const int64_t ldd = (N + 3) / 4 * 4;
  const int64_t nw = (T + 31) / 32;
  const size_t x_bytes = align_up(sizeof(float) * (size_t)(ldd * T), 256);
  const size_t s_bytes = summary_host ? align_up(sizeof(magus_summary) * (size_t)(N * C), 256) : 0;
  const size_t b_bytes = base_host ? align_up(sizeof(magus_base) * (size_t)N, 256) : 0;
  const size_t d_bytes = decisions_host ? align_up(sizeof(uint32_t) * (size_t)(C * nw * N), 256) : 0;
  const size_t t_bytes = totals_host ? align_up(sizeof(uint64_t) * (size_t)(C * MAGUS_TOT_WORDS), 256) : 0;
  const size_t need = x_bytes + s_bytes + b_bytes + d_bytes + t_bytes;
  if (need > ctx->stage_bytes) {
    CK(cudaStreamSynchronize(ctx->stream));
    if (ctx->stage_dev) cudaFree(ctx->stage_dev);
    ctx->stage_dev = nullptr;
    ctx->stage_bytes = 0;
    cudaError_t e = cudaMalloc(&ctx->stage_dev, need);
    if (e != cudaSuccess) { cudaGetLastError(); return fail(ctx, MAGUS_ERR_OOM, "staging allocation failed"); }
    ctx->stage_bytes = need;
  }
  char* p = (char*)ctx->stage_dev;
  float* xd = (float*)p; p += x_bytes;
  magus_summary* sd = summary_host ? (magus_summary*)p : nullptr; p += s_bytes;
  magus_base* bd = base_host ? (magus_base*)p : nullptr; p += b_bytes;
  uint32_t* dd = decisions_host ? (uint32_t*)p : nullptr; p += d_bytes;
  uint64_t* td = totals_host ? (uint64_t*)p : nullptr;
  CK(cudaMemcpy2DAsync(xd, ldd * 4, traces_host, ld * 4, N * 4, T, cudaMemcpyHostToDevice, ctx->stream));
  st = magus_replay(ctx, xd, N, T, ldd, params, C, sd, bd, dd, td);
  if (st != MAGUS_OK) return st;
  if (summary_host) CK(cudaMemcpyAsync(summary_host, sd, sizeof(magus_summary) * N * C, cudaMemcpyDeviceToHost, ctx->stream));
  if (base_host) CK(cudaMemcpyAsync(base_host, bd, sizeof(magus_base) * N, cudaMemcpyDeviceToHost, ctx->stream));
  if (decisions_host) CK(cudaMemcpyAsync(decisions_host, dd, sizeof(uint32_t) * C * nw * N, cudaMemcpyDeviceToHost, ctx->stream));
  if (totals_host) CK(cudaMemcpyAsync(totals_host, td, sizeof(uint64_t) * C * MAGUS_TOT_WORDS, cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  return MAGUS_OK;
}

magus_status magus_totals_derive(magus_ctx ctx, const uint64_t* totals_host, magus_derived* out) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!totals_host || !out) return fail(ctx, MAGUS_ERR_INVALID_ARG, "NULL argument");
  derive_totals(ctx->dplat, totals_host, out);
  return MAGUS_OK;
}

static magus_status choose_best(const DevPlatform& dp, const uint64_t* h, int32_t C, int32_t* best,
                                magus_derived* best_row) {
  std::vector<magus_derived> d((size_t)C);
  for (int32_t c = 0; c < C; ++c) derive_totals(dp, h + (size_t)c * MAGUS_TOT_WORDS, &d[c]);
  int32_t b = -1;
  for (int32_t c = 0; c < C; ++c)
    if (d[c].n_viol == 0 && (b < 0 || d[c].energy_j < d[b].energy_j)) b = c;
  magus_status st = MAGUS_OK;
  if (b < 0) {
    st = MAGUS_ERR_NO_FEASIBLE;
    b = 0;
    for (int32_t c = 1; c < C; ++c)
      if (d[c].n_viol < d[b].n_viol || (d[c].n_viol == d[b].n_viol && d[c].energy_j < d[b].energy_j)) b = c;
  }
  *best = b;
  if (best_row) *best_row = d[b];
  return st;
}

magus_status magus_sweep_best(magus_ctx ctx, const uint64_t* totals, int32_t C, int32_t* best,
                              magus_derived* best_row) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!totals || C < 1 || !best) return fail(ctx, MAGUS_ERR_INVALID_ARG, "bad sweep_best arguments");
  DeviceGuard dg(ctx->device);
  if (ctx->best_host.size() < (size_t)C * MAGUS_TOT_WORDS) {
    if (ctx->best_pinned) cudaFreeHost(ctx->best_pinned);
    ctx->best_pinned = nullptr;
    CK(cudaMallocHost(&ctx->best_pinned, sizeof(uint64_t) * (size_t)C * MAGUS_TOT_WORDS));
    ctx->best_host.resize((size_t)C * MAGUS_TOT_WORDS);
  }
  CK(cudaMemcpyAsync(ctx->best_pinned, totals, sizeof(uint64_t) * (size_t)C * MAGUS_TOT_WORDS,
                     cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  magus_status st = choose_best(ctx->dplat, (const uint64_t*)ctx->best_pinned, C, best, best_row);
  if (st == MAGUS_ERR_NO_FEASIBLE) ctx->err = "no config keeps every trace within the slowdown bound";
  return st;
}

static void pareto(const DevPlatform& dp, const uint64_t* h, int32_t C, int32_t* on_front,
                   int32_t* n_front) {
  std::vector<magus_derived> d((size_t)C);
  for (int32_t c = 0; c < C; ++c) derive_totals(dp, h + (size_t)c * MAGUS_TOT_WORDS, &d[c]);
  int32_t nf = 0;
  for (int32_t i = 0; i < C; ++i) {
    bool dominated = false;
    for (int32_t j = 0; j < C && !dominated; ++j)
      dominated = (d[j].energy_j <= d[i].energy_j && d[j].time_s <= d[i].time_s) &&
                  (d[j].energy_j < d[i].energy_j || d[j].time_s < d[i].time_s);
    on_front[i] = dominated ? 0 : 1;
    nf += on_front[i];
  }
  if (n_front) *n_front = nf;
}

magus_status magus_pareto_front(magus_ctx ctx, const uint64_t* totals, int32_t C, int32_t* on_front,
                                int32_t* n_front) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!totals || C < 1 || !on_front) return fail(ctx, MAGUS_ERR_INVALID_ARG, "bad pareto arguments");
  DeviceGuard dg(ctx->device);
  std::vector<uint64_t> h((size_t)C * MAGUS_TOT_WORDS);
  CK(cudaMemcpyAsync(h.data(), totals, h.size() * 8, cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  pareto(ctx->dplat, h.data(), C, on_front, n_front);
  return MAGUS_OK;
}

magus_status magus_pareto_front_host(const magus_platform* plat, const uint64_t* totals_host,
                                     int32_t C, int32_t* on_front, int32_t* n_front) {
  char msg[256];
  if (!plat || !totals_host || C < 1 || !on_front || !validate_platform(*plat, msg, sizeof msg))
    return MAGUS_ERR_INVALID_ARG;
  pareto(make_dev_platform(*plat), totals_host, C, on_front, n_front);
  return MAGUS_OK;
}

magus_status magus_comm_unique_id(void* id_out) {
  if (!id_out) return MAGUS_ERR_INVALID_ARG;
  return magus::nccl_unique_id(id_out) == 0 ? MAGUS_OK : MAGUS_ERR_NCCL;
}

magus_status magus_comm_init(magus_ctx ctx, const void* id, int32_t nranks, int32_t rank) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!id || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "comm_init: need an id and 0 <= rank < nranks");
  if (!magus::nccl_available()) return fail(ctx, MAGUS_ERR_NCCL, "libnccl.so.2 could not be opened");
  DeviceGuard dg(ctx->device);
  if (ctx->comm) {
    CK(cudaStreamSynchronize(ctx->stream));
    magus::nccl_comm_destroy(ctx->comm);
    ctx->comm = nullptr;
  }
  void* c = nullptr;
  const int r = magus::nccl_comm_init(&c, id, nranks, rank);
  if (r != 0) return fail(ctx, MAGUS_ERR_NCCL, "ncclCommInitRank: %s", magus::nccl_error(r));
  ctx->comm = c;
  return MAGUS_OK;
}

magus_status magus_allreduce_totals(magus_ctx ctx, uint64_t* totals, int32_t C) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!totals || C < 1) return fail(ctx, MAGUS_ERR_INVALID_ARG, "bad allreduce_totals arguments");
  if (!ctx->comm) return MAGUS_OK;
  DeviceGuard dg(ctx->device);
  const int r = magus::nccl_allreduce_u64_sum(ctx->comm, totals, (size_t)C * MAGUS_TOT_WORDS, ctx->stream);
  if (r != 0) return fail(ctx, MAGUS_ERR_NCCL, "ncclAllReduce: %s", magus::nccl_error(r));
  return MAGUS_OK;
}

magus_status magus_sweep_best_async(magus_ctx ctx, const uint64_t* totals, int32_t C,
                                    magus_choice* out) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!totals || C < 1 || !out) return fail(ctx, MAGUS_ERR_INVALID_ARG, "bad sweep_best_async arguments");
  DeviceGuard dg(ctx->device);
  if (!ctx->sweep_dev) CK(cudaMalloc(&ctx->sweep_dev, sizeof(SweepResult)));
  SweepResult* r = (SweepResult*)ctx->sweep_dev;
  if (launch_sweep_best(ctx->stream, totals, C, ctx->dplat, r) < 0)
    return cuda_fail(ctx, cudaGetLastError(), "sweep_best kernel launch");
  ctx->launches += 1;
  CK(cudaMemcpyAsync(out, r, sizeof(magus_choice), cudaMemcpyDeviceToHost, ctx->stream));
  return MAGUS_OK;
}

magus_status magus_derive_host(const magus_platform* plat, const uint64_t* totals_host,
                               magus_derived* out) {
  char msg[256];
  if (!plat || !totals_host || !out || !validate_platform(*plat, msg, sizeof msg)) return MAGUS_ERR_INVALID_ARG;
  derive_totals(make_dev_platform(*plat), totals_host, out);
  return MAGUS_OK;
}

magus_status magus_sweep_best_host(const magus_platform* plat, const uint64_t* totals_host,
                                   int32_t C, int32_t* best, magus_derived* best_row) {
  char msg[256];
  if (!plat || !totals_host || C < 1 || !best || !validate_platform(*plat, msg, sizeof msg))
    return MAGUS_ERR_INVALID_ARG;
  return choose_best(make_dev_platform(*plat), totals_host, C, best, best_row);
}

magus_status magus_gen_traces(magus_ctx ctx, uint64_t seed, int64_t id0, int64_t N, int64_t T,
                              int64_t ld, int32_t kind, float* out) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!out || N < 1 || T < 1 || ld < N || id0 < 0 || (kind != MAGUS_GEN_MIX && kind != MAGUS_GEN_ADVERSARIAL))
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "bad gen arguments");
  DeviceGuard dg(ctx->device);
  if (launch_gen(ctx->stream, seed, id0, N, T, ld, kind, out) < 0)
    return cuda_fail(ctx, cudaGetLastError(), "gen kernel launch");
  ctx->launches += 1;
  return MAGUS_OK;
}

magus_status magus_gen_state_bytes(int64_t n_traces, size_t* out) {
  if (!out || n_traces < 1) return MAGUS_ERR_INVALID_ARG;
  *out = gen_state_bytes(n_traces);
  return MAGUS_OK;
}

magus_status magus_gen_traces_resume(magus_ctx ctx, uint64_t seed, int64_t id0, int64_t N, int64_t t0,
                                     int64_t n_rows, int64_t ld, int32_t kind, void* state, float* out) {
  if (!ctx) return MAGUS_ERR_NOT_INITIALIZED;
  if (!out || !state || (uintptr_t)state % 8 != 0 || N < 1 || n_rows < 1 || t0 < 0 || ld < N || id0 < 0 ||
      (kind != MAGUS_GEN_MIX && kind != MAGUS_GEN_ADVERSARIAL))
    return fail(ctx, MAGUS_ERR_INVALID_ARG, "bad gen_traces_resume arguments");
  DeviceGuard dg(ctx->device);
  if (launch_gen_resume(ctx->stream, seed, id0, N, t0, n_rows, ld, kind, state, out) < 0)
    return cuda_fail(ctx, cudaGetLastError(), "gen kernel launch");
  ctx->launches += 1;
  return MAGUS_OK;
}

magus_status magus_get_trace(magus_ctx ctx, uint64_t* out, int64_t cap, int64_t* n_out) {
  if (!ctx || !out || cap < 0 || !n_out) return MAGUS_ERR_INVALID_ARG;
  if (!ctx->trace_dev || ctx->trace_n == 0) return fail(ctx, MAGUS_ERR_INVALID_ARG, "no traced replay");
  DeviceGuard dg(ctx->device);
  const int64_t n = std::min(cap, ctx->trace_n);
  CK(cudaMemcpyAsync(out, ctx->trace_dev, 64 * (size_t)n, cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  *n_out = n;
  return MAGUS_OK;
}

magus_status magus_get_stats(magus_ctx ctx, magus_stats* out) {
  if (!ctx || !out) return MAGUS_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  for (auto& pr : ctx->pending) {
    CK(cudaEventSynchronize(pr.second));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, pr.first, pr.second));
    ctx->main_ms += ms;
    ctx->main_launches += 1;
    ctx->event_pool.push_back(pr.first);
    ctx->event_pool.push_back(pr.second);
  }
  ctx->pending.clear();
  out->launches_total = ctx->launches;
  out->main_launches = ctx->main_launches;
  out->main_ms_total = ctx->main_ms;
  out->last_segments = ctx->last_segments;
  out->last_kernel = ctx->last_kernel;
  out->last_grid = ctx->last_grid;
  out->last_reruns = 0;
  out->last_family = ctx->last_family;
  if (ctx->last_kernel == 5 && ctx->spec_reruns) {
    unsigned int r = 0;
    CK(cudaMemcpyAsync(&r, ctx->spec_reruns, sizeof(r), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    out->last_reruns = r;
  }
  return MAGUS_OK;
}

magus_status magus_reset_stats(magus_ctx ctx) {
  if (!ctx) return MAGUS_ERR_INVALID_ARG;
  magus_stats tmp;
  magus_status st = magus_get_stats(ctx, &tmp);  // drains pending events
  ctx->launches = 0;
  ctx->main_launches = 0;
  ctx->main_ms = 0.0;
  return st;
}

}  // extern "C"
