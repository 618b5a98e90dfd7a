// kernels_bound.cu -- NEXT f2: offline-optimal schedules under model M.
//
// For each (trace, lambda) the DP over the level set finds the schedule
// dec[0..T-1] minimising energy + lambda * time of model M:
//   interval t runs at l_t = dec[t-1] (l_0 = r_max, reading R6);
//   cost of interval t at level l: c = e + lambda * tau with
//     tau = dt + cQ * q(x_t, l),  e = P_l * tau   (model M 4.2-4.3);
//   a change dec[t-1] != dec[t-2] (t >= 2, model M counts changes from t = 1)
//   costs e_sw + lambda * t_sw.
// V_t(i) = c(t, i) + min(V_{t-1}(i), min_{i' != i} V_{t-1}(i') + switch);
// ties: stay before move, lowest level index first.  Energy and time are
// summed along the chosen path in time order.  One thread per (trace,
// lambda); the level states live in registers (binary set) or local memory.
#include "device_common.cuh"

namespace magus {

constexpr int kBoundThreads = 128;

template <int MAXL>
__global__ void __launch_bounds__(kBoundThreads)
bound_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
             const double* __restrict__ lambdas, int32_t nl, int32_t L, int32_t l0, int32_t lstep,
             DevPlatform plat, double bw_max, double p_lo, double p_span, double* __restrict__ out) {
  __shared__ double s_invB[32], s_P[32];
  __shared__ float s_x[32][kBoundThreads];
  for (int i = threadIdx.x; i < L; i += blockDim.x) {
    const int l = l0 + i * lstep;
    const double B = (bw_max * (double)l) / (double)plat.r_max;
    s_invB[i] = 1.0 / B;
    s_P[i] = p_lo + (p_span * (double)(l - plat.r_min)) / (double)(plat.r_max - plat.r_min);
  }
  __syncthreads();
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool active = gid < N * nl;
  const int32_t j = active ? (int32_t)(gid / N) : 0;
  const int64_t n = active ? gid - (int64_t)j * N : 0;
  const double lam = lambdas[j];
  const double sw_c = plat.e_sw + lam * plat.t_sw;
  const int imax = L - 1;  // the level set is ascending and ends at r_max

  double V[MAXL], E[MAXL], Tm[MAXL];
  for (int i = 0; i < L; ++i) { V[i] = INFINITY; E[i] = 0.0; Tm[i] = 0.0; }

  for (int64_t t = 0; t < T; ++t) {
    const int jj = (int)(t & 31);
    if (jj == 0) {  // stage the next 32 samples of this trace (independent loads)
      __syncwarp();
#pragma unroll 8
      for (int i = 0; i < 32; ++i)
        s_x[i][threadIdx.x] = (active && t + i < T) ? x[(t + i) * ld + n] : 0.0f;
      __syncwarp();
    }
    const float xt = s_x[jj][threadIdx.x];
    if (t == 0) {
      const double tau = plat.dt + plat.cQ * (double)q_literal(xt, s_invB[imax]);
      const double e = s_P[imax] * tau;
      V[imax] = e + lam * tau;
      E[imax] = e;
      Tm[imax] = tau;
      continue;
    }
    // best and second best previous state (lowest index on ties)
    int a1 = 0;
    double m1 = V[0];
    for (int i = 1; i < L; ++i)
      if (V[i] < m1) { m1 = V[i]; a1 = i; }
    int a2 = -1;
    double m2 = INFINITY;
    for (int i = 0; i < L; ++i)
      if (i != a1 && (a2 < 0 || V[i] < m2)) { m2 = V[i]; a2 = i; }
    const bool sw = t >= 2;
    double nV[MAXL], nE[MAXL], nT[MAXL];
    for (int i = 0; i < L; ++i) {
      const int oi = (i == a1) ? a2 : a1;
      const double other = (i == a1) ? m2 : m1;
      const double move = sw ? other + sw_c : other;
      double v, e0, t0;
      if (oi < 0 || V[i] <= move) {
        v = V[i]; e0 = E[i]; t0 = Tm[i];
      } else {
        v = move;
        e0 = sw ? E[oi] + plat.e_sw : E[oi];
        t0 = sw ? Tm[oi] + plat.t_sw : Tm[oi];
      }
      const double tau = plat.dt + plat.cQ * (double)q_literal(xt, s_invB[i]);
      const double e = s_P[i] * tau;
      nV[i] = v + (e + lam * tau);
      nE[i] = e0 + e;
      nT[i] = t0 + tau;
    }
    for (int i = 0; i < L; ++i) { V[i] = nV[i]; E[i] = nE[i]; Tm[i] = nT[i]; }
  }
  if (!active) return;
  int b = 0;
  for (int i = 1; i < L; ++i)
    if (V[i] < V[b]) b = i;
  double* o = out + ((int64_t)n * nl + j) * 3;
  o[0] = V[b];
  o[1] = E[b];
  o[2] = Tm[b];
}

// (double)q_literal(x, invB) from the widened sample xd = (double)x, with
// floor(s * 2^24) formed in fp64 (RZ add of 2^52: exact for 0 < s * 2^24 <=
// 2^39) -- bit-identical, without an XU conversion per level.
__device__ __forceinline__ double q_as_double(double xd, double invB) {
  const double r = xd * invB;
  double s24 = (r - 1.0 < 32768.0 ? r - 1.0 : 32768.0) * kQScale;
  s24 = __dsub_rn(__dadd_rz(s24, 4503599627370496.0), 4503599627370496.0);
  return r > 1.0 ? s24 : 0.0;
}

// The binary level set {r_min, r_max}: the same recurrence with the two
// states in scalar registers (the generic kernel's arrays live in local
// memory) and the samples of 32 intervals loaded ahead.  For L = 2 the
// "other" state of each level is always the opposite one, so the
// best / second-best search reduces to it.  Same fp64 operations in the
// same order as bound_kernel (and the oracle DP).  (A branch skipping the
// stretch arithmetic for samples below the capacity measured slower:
// divergence across the warp's traces.)
__global__ void __launch_bounds__(kBoundThreads)
bound_binary_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
                    const double* __restrict__ lambdas, int32_t nl, DevPlatform plat, double bw_max,
                    double p_lo, double p_span, double* __restrict__ out) {
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= N * nl) return;
  const int32_t j = (int32_t)(gid / N);
  const int64_t n = gid - (int64_t)j * N;
  const double lam = lambdas[j];
  const double sw_c = plat.e_sw + lam * plat.t_sw;
  const int lmin = plat.r_min, lmax = plat.r_max;
  const double invB0 = 1.0 / ((bw_max * (double)lmin) / (double)lmax);
  const double invB1 = 1.0 / ((bw_max * (double)lmax) / (double)lmax);
  const double P0 = p_lo + (p_span * (double)(lmin - lmin)) / (double)(lmax - lmin);
  const double P1 = p_lo + (p_span * (double)(lmax - lmin)) / (double)(lmax - lmin);
  const double dt = plat.dt, cQ = plat.cQ, e_sw = plat.e_sw, t_sw = plat.t_sw;
  double V0 = INFINITY, E0 = 0.0, T0 = 0.0, V1 = INFINITY, E1 = 0.0, T1 = 0.0;
  const float* px = x + n;
  for (int64_t tc = 0; tc < T; tc += 32) {
    float xs[32];
    const int rem = (int)(T - tc < 32 ? T - tc : 32);
#pragma unroll
    for (int i = 0; i < 32; ++i) xs[i] = i < rem ? __ldg(px + (tc + i) * ld) : 0.0f;
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (i < rem) {
        const int64_t t = tc + i;
        // model M stretch (q_literal) with the sample widened
        // once and floor(s * 2^24) formed in fp64 (RZ add of 2^52: exact for
        // 0 < s * 2^24 <= 2^39), so no XU conversion per level; the value
        // equals (double)q_literal(x, invB) bit for bit
        const double xd = (double)xs[i];
        const double tau0 = dt + cQ * q_as_double(xd, invB0);
        const double tau1 = dt + cQ * q_as_double(xd, invB1);
        const double e0 = P0 * tau0, e1 = P1 * tau1;
        if (t == 0) {            // interval 0 runs at r_max (reading R6)
          V1 = e1 + lam * tau1;
          E1 = e1;
          T1 = tau1;
          continue;
        }
        const bool sw = t >= 2;
        const double mv0 = sw ? V1 + sw_c : V1, mv1 = sw ? V0 + sw_c : V0;
        const bool st0 = V0 <= mv0, st1 = V1 <= mv1;  // stay before move
        const double nV0 = (st0 ? V0 : mv0) + (e0 + lam * tau0);
        const double nE0 = (st0 ? E0 : (sw ? E1 + e_sw : E1)) + e0;
        const double nT0 = (st0 ? T0 : (sw ? T1 + t_sw : T1)) + tau0;
        const double nV1 = (st1 ? V1 : mv1) + (e1 + lam * tau1);
        const double nE1 = (st1 ? E1 : (sw ? E0 + e_sw : E0)) + e1;
        const double nT1 = (st1 ? T1 : (sw ? T0 + t_sw : T0)) + tau1;
        V0 = nV0; E0 = nE0; T0 = nT0;
        V1 = nV1; E1 = nE1; T1 = nT1;
      }
    }
  }
  const bool b1 = V1 < V0;  // lowest index on ties
  double* o = out + ((int64_t)n * nl + j) * 3;
  o[0] = b1 ? V1 : V0;
  o[1] = b1 ? E1 : E0;
  o[2] = b1 ? T1 : T0;
}


// ---------------------------------------------------------------------------
// bound_dp_kernel<L>: the same DP, restructured for throughput.
// Every result is bit-identical to bound_kernel / the oracle DP: the same fp64
// operations on the same operands in the same order; only which of them are
// evaluated, and where the operands are kept, changes.
//
// * No second minimum.  The move candidate of level i is the lowest-index
//   minimum a1 of the previous values for every i != a1, and a1 itself always
//   stays: V[a1] = m1 <= V[o] <= RN(V[o] + sw_c) for any other o, because
//   sw_c = e_sw + lambda * t_sw >= 0 (validated finite and >= 0, so no NaN)
//   and RN is monotone.  So every level compares against ONE move value
//   mv = m1 (+ sw_c) and inherits (E1, T1) = (E, T)[a1] when it moves.
// * Two passes per 32-step chunk.  Pass 1 runs the value chain only (V per
//   level, the lowest-index minimum, which levels stayed); pass 2 the path
//   sums.  When no level other than a1 stays in a step (always, up to exact
//   ties, when switches are free: e_sw = t_sw = 0, the paper's "negligible"
//   MSR writes), every level's new (E, T) is (E1, T1) or (Eb, Tb) plus its
//   own (e, tau), so only (E1, T1) are followed: E1' = (a1' == a1 ? E1 : Eb)
//   + e[a1'] (mode A).  A step where another level stays (a tie, or
//   sw_c > 0) keeps per-level (E, T) (mode B), rebuilt first from the last
//   mode-A step's record (its sample, the level that stayed, the two bases)
//   -- again the operations the oracle did.  Modes are warp-uniform.
// * Two lanes per (trace, lambda) chain, each owning half of the levels
//   (16 chains per warp), so a sub-partition holds ~2 warps of independent
//   work; a chain's minimum is its lanes' local trees merged by one shuffle
//   (the lower half wins ties: the lowest-index rule).
// * Stretch work only where it exists: the thresholds x*_l (x > x*_l <=>
//   RN(x * invB_l) > 1, host-inverted) rise with the level, so the levels with
//   a stretch at step t are a prefix [0, s) (warp max).  Their costs are
//   written to a per-lane row in shared memory; otherwise the q = 0 costs
//   (tau = dt, e = P_l * dt, e + lambda * dt: the same operations with q = 0)
//   are register constants.
// * Lanes are (trace, lambda) with lambda fastest; one warp per CTA; a rolled
//   step loop; samples staged per warp by cp.async, double-buffered.
// ---------------------------------------------------------------------------
struct BoundThr {
  float x[32];  // x*_l per level of the DP's level set (stretch_threshold)
};

constexpr int kDpChunk = 32;

__device__ __forceinline__ void cp_async4(float* dst, const float* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
               "l"(src)
               : "memory");
}

// V' = (V <= mv ? V : mv) + c, stay bit `bit` set when V <= mv
__device__ __forceinline__ void v_update(double& v, uint32_t& stay, double mv, uint32_t bit, double c) {
  asm("{\n.reg .pred p;\n"
      "setp.le.f64 p, %0, %2;\n"
      "@p or.b32 %1, %1, %3;\n"
      "selp.f64 %0, %0, %2, p;\n"
      "add.rn.f64 %0, %0, %4;\n}"
      : "+d"(v), "+r"(stay)
      : "d"(mv), "r"(bit), "d"(c));
}

template <int L>
__global__ void __launch_bounds__(32)
bound_dp_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
                const double* __restrict__ lambdas, int32_t nl, int32_t lstep, DevPlatform plat,
                double bw_max, double p_lo, double p_span, const __grid_constant__ BoundThr thr,
                double* __restrict__ out) {
  static_assert(L >= 4 && L <= 18, "level set");
  constexpr int H = (L + 1) / 2;  // levels per lane: [0, H) and [H, L)
  __shared__ double s_invB[2 * H], s_P[2 * H], s_Pdt[2 * H];
  __shared__ double s_c[H * 32];  // [local level][lane]: this step's stretched costs
  __shared__ float s_thr[32];
  __shared__ float s_x[2][kDpChunk][32];
  __shared__ uint8_t s_a1[kDpChunk][32];    // pass 1 -> 2: argmin of each step
  __shared__ uint32_t s_stay[kDpChunk][32];  // pass 1 -> 2: this lane's levels that stayed
  const int lane = threadIdx.x;
  const int h = lane & 1;          // which half of the levels
  const int base = h * H;          // first level of this lane
  for (int i = lane; i < 2 * H; i += 32) {
    if (i < L) {
      const int l = plat.r_min + i * lstep;
      const double B = (bw_max * (double)l) / (double)plat.r_max;
      s_invB[i] = 1.0 / B;
      s_P[i] = p_lo + (p_span * (double)(l - plat.r_min)) / (double)(plat.r_max - plat.r_min);
      s_Pdt[i] = s_P[i] * plat.dt;  // e at q = 0: P_l * (dt + cQ * 0) = P_l * dt
    } else {  // the padding level of an odd L: never reachable
      s_invB[i] = 0.0;
      s_P[i] = 0.0;
      s_Pdt[i] = 0.0;
    }
  }
  s_thr[lane] = lane < L ? thr.x[lane] : INFINITY;
  __syncwarp();
  const int64_t chain = (int64_t)blockIdx.x * 16 + (lane >> 1);
  const bool active = chain < N * nl;
  const int64_t n = active ? chain / nl : 0;
  const int32_t j = active ? (int32_t)(chain - n * nl) : 0;
  const double lam = lambdas[j];
  const double dt = plat.dt, cQ = plat.cQ, e_sw = plat.e_sw, t_sw = plat.t_sw;
  const double sw_c = e_sw + lam * t_sw;
  const double lt0 = lam * dt;  // lambda * tau at q = 0
  double cf[H];                 // this lane's costs at q = 0 (+inf: the padding level)
#pragma unroll
  for (int i = 0; i < H; ++i) cf[i] = (base + i < L) ? s_Pdt[base + i] + lt0 : INFINITY;

  double V[H], E[H], Tm[H];
  const float* px = x + n;
  // t = 0: every level's (e, tau); only r_max (the last level) is reachable
  {
    const double xd = (double)(active ? __ldg(px) : 0.0f);
#pragma unroll
    for (int i = 0; i < H; ++i) {
      const int g = base + i;
      const double tau = dt + cQ * q_as_double(xd, s_invB[g]);
      const double e = s_P[g] * tau;
      V[i] = (g == L - 1) ? e + lam * tau : INFINITY;
      E[i] = e;
      Tm[i] = tau;
    }
  }
  // the chain's scalars (identical in both lanes)
  double m1, E1, T1;
  {
    const int o = (L - 1) - H;  // r_max is local level L-1-H of the upper lane
    const double v = h ? V[o] : 0.0, e = h ? E[o] : 0.0, t = h ? Tm[o] : 0.0;
    m1 = __shfl_sync(0xFFFFFFFFu, v, lane | 1);
    E1 = __shfl_sync(0xFFFFFFFFu, e, lane | 1);
    T1 = __shfl_sync(0xFFFFFFFFu, t, lane | 1);
  }
  int a1 = L - 1;
  bool inB = true;  // the per-level (E, T) arrays are current
  // mode-A record of the last step: its sample, the level that stayed, the bases
  double r_x = 0.0, r_E1 = 0.0, r_Eb = 0.0, r_T1 = 0.0, r_Tb = 0.0;
  int r_a1 = L - 1;
  int prev_ns = 0;  // the last step stretched levels [0, prev_ns)
  // samples t = 1 + c * 32 + k in chunk c, staged into s_x[c & 1][k][lane]
  const int64_t nch = (T - 1 + kDpChunk - 1) / kDpChunk;
  auto stage = [&](int64_t c) {
    const int64_t t0 = 1 + c * kDpChunk;
    const int kmax = (int)(T - t0 < kDpChunk ? T - t0 : kDpChunk);
    const float* src = px + (active ? t0 * ld : 0);
    const int64_t step = active ? ld : 0;
    float* dst = &s_x[c & 1][0][lane];
#pragma unroll 8
    for (int k = 0; k < kmax; ++k) {
      cp_async4(dst + k * 32, src);
      src += step;
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  if (nch > 0) stage(0);
  for (int64_t c = 0; c < nch; ++c) {
    if (c + 1 < nch) {
      stage(c + 1);
      asm volatile("cp.async.wait_group 1;" ::: "memory");
    } else {
      asm volatile("cp.async.wait_group 0;" ::: "memory");
    }
    __syncwarp();
    const int64_t t0 = 1 + c * kDpChunk;
    const int kn = (int)(T - t0 < kDpChunk ? T - t0 : kDpChunk);
    const float* xs = &s_x[c & 1][0][lane];
    // ---- pass 1: the value chain (V per level, m1, argmin, stay bits) ----
#pragma unroll 1
    for (int k = 0; k < kn; ++k) {
      const bool sw = t0 + k >= 2;
      const double mv = sw ? m1 + sw_c : m1;
      const float xf = xs[k * 32];
      // levels with a stretch at this step: a prefix [0, ns) (NaN: none)
      int ns = 0;
      if (__any_sync(0xFFFFFFFFu, xf > s_thr[0])) {
#pragma unroll
        for (int w = 16; w > 0; w >>= 1)
          if (ns + w <= L && xf > s_thr[ns + w - 1]) ns += w;
        ns = __reduce_max_sync(0xFFFFFFFFu, ns);
      }
      uint32_t stay = 0;
      if (ns == 0) {  // every cost is its q = 0 constant
#pragma unroll
        for (int i = 0; i < H; ++i) v_update(V[i], stay, mv, 1u << i, cf[i]);
      } else {
        // this lane's stretched levels [base, ns) get the full model-M cost
        const double xd = (double)xf;
        const int nloc = ns - base;
#pragma unroll 1
        for (int i = 0; i < nloc && i < H; ++i) {
          const double tau = dt + cQ * q_as_double(xd, s_invB[base + i]);
          const double e = s_P[base + i] * tau;
          s_c[i * 32 + lane] = e + lam * tau;
        }
#pragma unroll
        for (int i = 0; i < H; ++i) v_update(V[i], stay, mv, 1u << i, i < nloc ? s_c[i * 32 + lane] : cf[i]);
      }
      (void)prev_ns;
      // lowest-index minimum: local pairwise tree, then the two halves
      double tv[H];
      int ti[H];
#pragma unroll
      for (int i = 0; i < H; ++i) { tv[i] = V[i]; ti[i] = base + i; }
#pragma unroll
      for (int w = 1; w < H; w *= 2) {
#pragma unroll
        for (int i = 0; i + w < H; i += 2 * w) {
          const bool r = tv[i + w] < tv[i];
          tv[i] = r ? tv[i + w] : tv[i];
          ti[i] = r ? ti[i + w] : ti[i];
        }
      }
      const double vo = __shfl_xor_sync(0xFFFFFFFFu, tv[0], 1);
      const int io = __shfl_xor_sync(0xFFFFFFFFu, ti[0], 1);
      // the partner wins if strictly smaller, or equal and lower (h = 1 takes an equal lower half)
      const bool take = h ? (vo <= tv[0]) : (vo < tv[0]);
      m1 = take ? vo : tv[0];
      s_a1[k][lane] = (uint8_t)(take ? io : ti[0]);
      s_stay[k][lane] = stay;
    }
    // ---- pass 2: the path sums (E, T) along the chosen predecessors ----
    // A step where a level other than the previous argmin stayed needs the
    // per-level histories (mode B); find out for the whole chunk first
    uint32_t other = 0;
    {
      int pa = a1;
#pragma unroll 1
      for (int k = 0; k < kn; ++k) {
        const int lb = pa - base;  // the argmin's bit in this lane's mask, if it is here
        other |= s_stay[k][lane] & ~((lb >= 0 && lb < H) ? (1u << lb) : 0u);
        pa = s_a1[k][lane];
      }
    }
    if (!__any_sync(0xFFFFFFFFu, other != 0u)) {
      // mode A throughout: every level but the argmin moved, so (E1, T1)
      // follow the argmin: E1' = (a1' == a1 ? E1 : Eb) + e[a1']
      double pE1 = E1, pEb = E1, pT1 = T1, pTb = T1, px_ = r_x;
      int pa1 = a1;
#pragma unroll 4
      for (int k = 0; k < kn; ++k) {
        const bool sw = t0 + k >= 2;
        const double Eb = sw ? E1 + e_sw : E1;
        const double Tb = sw ? T1 + t_sw : T1;
        const int na = s_a1[k][lane];
        const double xd = (double)xs[k * 32];
        const double tau_a = dt + cQ * q_as_double(xd, s_invB[na]);  // q = 0: dt, P * dt
        const double e_a = s_P[na] * tau_a;
        pE1 = E1; pEb = Eb; pT1 = T1; pTb = Tb; px_ = xd; pa1 = a1;
        E1 = (na == a1 ? E1 : Eb) + e_a;
        T1 = (na == a1 ? T1 : Tb) + tau_a;
        a1 = na;
      }
      if (kn > 0) {
        r_x = px_; r_a1 = pa1; r_E1 = pE1; r_Eb = pEb; r_T1 = pT1; r_Tb = pTb;
        inB = false;
      }
    } else {
#pragma unroll 1
      for (int k = 0; k < kn; ++k) {
        const bool sw = t0 + k >= 2;
        const double Eb = sw ? E1 + e_sw : E1;
        const double Tb = sw ? T1 + t_sw : T1;
        const int na = s_a1[k][lane];
        const uint32_t stay = s_stay[k][lane];
        const double xd = (double)xs[k * 32];
        const int lb = a1 - base;
        if (__any_sync(0xFFFFFFFFu, (stay & ~((lb >= 0 && lb < H) ? (1u << lb) : 0u)) != 0u)) {
          // mode B: per-level (E, T)
          if (!inB) {  // rebuild (E, T) of the last step from its record
#pragma unroll
            for (int i = 0; i < H; ++i) {
              const double tau = dt + cQ * q_as_double(r_x, s_invB[base + i]);
              const double e = s_P[base + i] * tau;
              E[i] = (base + i == r_a1 ? r_E1 : r_Eb) + e;
              Tm[i] = (base + i == r_a1 ? r_T1 : r_Tb) + tau;
            }
            inB = true;
          }
          double eo = 0.0, to = 0.0;
#pragma unroll
          for (int i = 0; i < H; ++i) {
            const double tau = dt + cQ * q_as_double(xd, s_invB[base + i]);
            const double e = s_P[base + i] * tau;
            const bool st = (stay >> i) & 1u;
            E[i] = (st ? E[i] : Eb) + e;
            Tm[i] = (st ? Tm[i] : Tb) + tau;
            if (base + i == na) { eo = E[i]; to = Tm[i]; }
          }
          const int owner = (lane & ~1) | (na >= H ? 1 : 0);
          E1 = __shfl_sync(0xFFFFFFFFu, eo, owner);
          T1 = __shfl_sync(0xFFFFFFFFu, to, owner);
        } else {
          const double tau_a = dt + cQ * q_as_double(xd, s_invB[na]);
          const double e_a = s_P[na] * tau_a;
          r_x = xd; r_a1 = a1; r_E1 = E1; r_Eb = Eb; r_T1 = T1; r_Tb = Tb;
          E1 = (na == a1 ? E1 : Eb) + e_a;
          T1 = (na == a1 ? T1 : Tb) + tau_a;
          inB = false;
        }
        a1 = na;
      }
    }
    __syncwarp();  // s_x[c & 1] is restaged by chunk c + 2
  }
  if (!active || h) return;
  double* o = out + chain * 3;  // [n][nl][3]: chain = n * nl + j
  o[0] = m1;
  o[1] = E1;
  o[2] = T1;
}

// ---------------------------------------------------------------------------
// bound_binary_free_kernel: the binary DP when switches are free (e_sw =
// t_sw = 0, the paper's "negligible" MSR writes -- the default platform).
// Then mv = m1 and a level stays only if V == m1, so without a tie every
// level's new value is m1 + c (stay or move alike: V = m1 when it stays),
// the new minimum is the smaller sum (the lower level on equality), and the
// path sums follow the argmin: E1 += e[a1'], T1 += tau[a1'] (Eb = E1 + 0 =
// E1).  Per step: two adds, a compare, three selects and two adds.  A tie
// (s0 == s1: both levels minimal) gives the levels different histories, so
// the warp rebuilds the per-level state of that step -- V_i = s_i,
// E_i = E1 + e_i, T_i = T1 + tau_i, the oracle's own sums -- and finishes
// with the general per-level recurrence (bound_binary_kernel's step).
// Lanes are (trace, lambda) with lambda fastest, so the stretch branch (a
// warp-wide vote on x > x*_min, host-inverted) is rarely taken; samples are
// staged per warp by cp.async, double-buffered; one warp per CTA.
// ---------------------------------------------------------------------------
constexpr int kBinChunk = 32;  // steps per staged chunk

__global__ void __launch_bounds__(32)
bound_binary_free_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
                         const double* __restrict__ lambdas, int32_t nl, DevPlatform plat, double bw_max,
                         double p_lo, double p_span, float xthr0, float xthr_max, double* __restrict__ out) {
  __shared__ float s_x[2][kBinChunk][32];
  const int lane = threadIdx.x;
  const int64_t gid = (int64_t)blockIdx.x * 32 + lane;
  const bool active = gid < N * nl;
  const int64_t n = active ? gid / nl : 0;
  const int32_t j = active ? (int32_t)(gid - n * nl) : 0;
  const double lam = lambdas[j];
  const int lmin = plat.r_min, lmax = plat.r_max;
  const double invB0 = 1.0 / ((bw_max * (double)lmin) / (double)lmax);
  const double invB1 = 1.0 / ((bw_max * (double)lmax) / (double)lmax);
  const double P0 = p_lo + (p_span * (double)(lmin - lmin)) / (double)(lmax - lmin);
  const double P1 = p_lo + (p_span * (double)(lmax - lmin)) / (double)(lmax - lmin);
  const double dt = plat.dt, cQ = plat.cQ;
  const double Pdt0 = P0 * dt, Pdt1 = P1 * dt;         // e at q = 0
  const double cf0 = Pdt0 + lam * dt, cf1 = Pdt1 + lam * dt;  // e + lambda * tau at q = 0
  const float* px = x + n;
  // t = 0 runs at r_max
  double m1, E1, T1;
  {
    const double xd = (double)(active ? __ldg(px) : 0.0f);
    const double tau1 = dt + cQ * q_as_double(xd, invB1);
    const double e1 = P1 * tau1;
    m1 = e1 + lam * tau1;
    E1 = e1;
    T1 = tau1;
  }
  bool general = false;  // warp-uniform: per-level recurrence after a tie
  double V0 = 0.0, V1 = 0.0, E0 = 0.0, Ea = 0.0, T0 = 0.0, Ta = 0.0;  // its per-level state
  const int64_t nch = (T - 1 + kBinChunk - 1) / kBinChunk;
  auto stage = [&](int64_t c) {
    const int64_t t0 = 1 + c * kBinChunk;
    const int kmax = (int)(T - t0 < kBinChunk ? T - t0 : kBinChunk);
    const float* src = px + (active ? t0 * ld : 0);
    const int64_t step = active ? ld : 0;
    float* dst = &s_x[c & 1][0][lane];
#pragma unroll 8
    for (int k = 0; k < kmax; ++k) {
      cp_async4(dst + k * 32, src);
      src += step;
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  if (nch > 0) stage(0);
  for (int64_t c = 0; c < nch; ++c) {
    if (c + 1 < nch) {
      stage(c + 1);
      asm volatile("cp.async.wait_group 1;" ::: "memory");
    } else {
      asm volatile("cp.async.wait_group 0;" ::: "memory");
    }
    __syncwarp();
    const int64_t t0 = 1 + c * kBinChunk;
    const int kn = (int)(T - t0 < kBinChunk ? T - t0 : kBinChunk);
    const float* xs = &s_x[c & 1][0][lane];
    // (c, e, tau) of both levels at a sample: full model M
    auto costs = [&](float xf, double& c0, double& c1, double& e0, double& e1, double& tau0, double& tau1) {
      const double xd = (double)xf;
      tau0 = dt + cQ * q_as_double(xd, invB0);
      tau1 = dt + cQ * q_as_double(xd, invB1);
      e0 = P0 * tau0;
      e1 = P1 * tau1;
      c0 = e0 + lam * tau0;
      c1 = e1 + lam * tau1;
    };
    bool redo = false;
    if (!general) {
      // fast sweep over the chunk; a tie anywhere sends the warp back to the
      // chunk's start for the careful sweep below
      const double m1s = m1, E1s = E1, T1s = T1;
      bool tie = false;
      // branch-free steps (so consecutive steps overlap): the r_min level's
      // model-M cost is computed for every sample (q = 0 below its capacity
      // gives exactly the q = 0 constants), the r_max level's only in chunks
      // where some lane's sample exceeds even that capacity (warp-uniform)
      bool over_max = false;
#pragma unroll 8
      for (int k = 0; k < kn; ++k) over_max |= xs[k * 32] > xthr_max;
      if (__any_sync(0xFFFFFFFFu, over_max)) {
#pragma unroll 4
        for (int k = 0; k < kn; ++k) {
          double c0, c1, e0, e1, tau0, tau1;
          costs(xs[k * 32], c0, c1, e0, e1, tau0, tau1);
          // without a tie, RN(m1 + c1) < RN(m1 + c0) <=> c1 < c0 (RN is
          // monotone): the step's choice does not depend on m1, and the
          // dependent chain is one add (the tie test runs beside it)
          const bool up = c1 < c0;
          tie |= (m1 + c0) == (m1 + c1);
          m1 = m1 + (up ? c1 : c0);
          E1 = E1 + (up ? e1 : e0);
          T1 = T1 + (up ? tau1 : tau0);
        }
      } else {
#pragma unroll 8
        for (int k = 0; k < kn; ++k) {
          const double xd = (double)xs[k * 32];
          const double tau0 = dt + cQ * q_as_double(xd, invB0);
          const double e0 = P0 * tau0;
          const double c0 = e0 + lam * tau0;
          const bool up = cf1 < c0;
          tie |= (m1 + c0) == (m1 + cf1);
          m1 = m1 + (up ? cf1 : c0);
          E1 = E1 + (up ? Pdt1 : e0);
          T1 = T1 + (up ? dt : tau0);
        }
      }
      if (__any_sync(0xFFFFFFFFu, tie)) {
        m1 = m1s; E1 = E1s; T1 = T1s;
        redo = true;
      }
    }
    if (general || redo) {
#pragma unroll 1
      for (int k = 0; k < kn; ++k) {
        double c0, c1, e0, e1, tau0, tau1;
        costs(xs[k * 32], c0, c1, e0, e1, tau0, tau1);
        if (!general) {
          const double s0 = m1 + c0, s1 = m1 + c1;
          if (__any_sync(0xFFFFFFFFu, s0 == s1)) {
            // a tie: rebuild every lane's per-level state of this step
            V0 = s0; V1 = s1;
            E0 = E1 + e0; Ea = E1 + e1;
            T0 = T1 + tau0; Ta = T1 + tau1;
            general = true;
          } else {
            const bool up = s1 < s0;
            m1 = up ? s1 : s0;
            E1 = E1 + (up ? e1 : e0);
            T1 = T1 + (up ? tau1 : tau0);
          }
        } else {  // the general recurrence (free switches: mv = the other level's V)
          const bool st0 = V0 <= V1, st1 = V1 <= V0;  // stay before move
          const double nV0 = (st0 ? V0 : V1) + c0, nE0 = (st0 ? E0 : Ea) + e0, nT0 = (st0 ? T0 : Ta) + tau0;
          const double nV1 = (st1 ? V1 : V0) + c1, nE1 = (st1 ? Ea : E0) + e1, nT1 = (st1 ? Ta : T0) + tau1;
          V0 = nV0; E0 = nE0; T0 = nT0;
          V1 = nV1; Ea = nE1; Ta = nT1;
        }
      }
    }
    __syncwarp();  // s_x[c & 1] is restaged by chunk c + 2
  }
  if (general) {
    const bool b1 = V1 < V0;  // lowest index on ties
    m1 = b1 ? V1 : V0;
    E1 = b1 ? Ea : E0;
    T1 = b1 ? Ta : T0;
  }
  if (!active) return;
  double* o = out + gid * 3;
  o[0] = m1;
  o[1] = E1;
  o[2] = T1;
}

// ---------------------------------------------------------------------------
// bound_binary_shared_kernel: bound_binary_free_kernel when nl divides 32 (a
// warp holds 32 / nl whole traces, lanes = (trace slot, lambda)).  The
// lambda-independent model-M terms of a step (tau, e = P tau of both levels)
// are computed once per (trace, step) into shared memory by the whole warp
// and read by the trace's nl lanes; samples are staged [step][trace slot]
// (one copy per trace, not per lane).  A lane's step is then c = e + lam tau,
// the choice (c1 < c0: no tie), the tie test and three adds.  Same fp64
// operations as the free kernel (and the oracle DP), bit for bit.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void cp_async4z(float* dst, const float* src, bool valid) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
               "l"(src), "r"(valid ? 4 : 0)
               : "memory");
}

__global__ void __launch_bounds__(32)
bound_binary_shared_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
                           const double* __restrict__ lambdas, int32_t nl, DevPlatform plat, double bw_max,
                           double p_lo, double p_span, float xthr_max, double* __restrict__ out) {
  __shared__ float s_x[2][kBinChunk][16];     // [buffer][step][trace slot]
  __shared__ double2 s_te[kBinChunk][16][2];  // [step][trace slot][level] {tau, e}
  const int lane = threadIdx.x;
  const int lgnl = __ffs(nl) - 1, lgtpw = 5 - lgnl, tpw = 1 << lgtpw;
  const int slot = lane >> lgnl, j = lane & (nl - 1);
  const int64_t n0 = (int64_t)blockIdx.x * tpw;  // the warp's first trace
  const int64_t n = n0 + slot;
  const bool active = n < N;
  const double lam = lambdas[j];
  const int lmin = plat.r_min, lmax = plat.r_max;
  const double invB0 = 1.0 / ((bw_max * (double)lmin) / (double)lmax);
  const double invB1 = 1.0 / ((bw_max * (double)lmax) / (double)lmax);
  const double P0 = p_lo + (p_span * (double)(lmin - lmin)) / (double)(lmax - lmin);
  const double P1 = p_lo + (p_span * (double)(lmax - lmin)) / (double)(lmax - lmin);
  const double dt = plat.dt, cQ = plat.cQ;
  const double Pdt1 = P1 * dt;
  const double cf1 = Pdt1 + lam * dt;  // e + lambda * tau at r_max, q = 0
  double m1, E1, T1;
  {
    const double xd = (double)(active ? __ldg(x + n) : 0.0f);
    const double tau1 = dt + cQ * q_as_double(xd, invB1);
    const double e1 = P1 * tau1;
    m1 = e1 + lam * tau1;
    E1 = e1;
    T1 = tau1;
  }
  bool general = false;
  double V0 = 0.0, V1 = 0.0, E0 = 0.0, Ea = 0.0, T0 = 0.0, Ta = 0.0;
  const int64_t nch = (T - 1 + kBinChunk - 1) / kBinChunk;
  // a lane's (step, slot) items of a chunk: slot r_l, steps k_l + i * kstride
  const int r_l = lane & (tpw - 1), k_l = lane >> lgtpw, kstride = 32 >> lgtpw;
  const bool r_ok = n0 + r_l < N;
  const float* xl = x + (r_ok ? n0 + r_l : 0);
  const int64_t ldk = (int64_t)kstride * ld;
  auto stage = [&](int64_t c) {
    const int64_t t0 = 1 + c * kBinChunk;
    const float* src = xl + (t0 + k_l) * ld;
    float* dst = &s_x[c & 1][k_l][r_l];
    int64_t t = t0 + k_l;
    for (int i = 0; i < tpw; ++i) {
      const bool ok = r_ok && t < T;
      cp_async4z(dst, ok ? src : x, ok);
      src += ldk;
      dst += kstride * 16;
      t += kstride;
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  if (nch > 0) stage(0);
  for (int64_t c = 0; c < nch; ++c) {
    if (c + 1 < nch) {
      stage(c + 1);
      asm volatile("cp.async.wait_group 1;" ::: "memory");
    } else {
      asm volatile("cp.async.wait_group 0;" ::: "memory");
    }
    __syncwarp();
    const int64_t t0 = 1 + c * kBinChunk;
    const int kn = (int)(T - t0 < kBinChunk ? T - t0 : kBinChunk);
    auto costs = [&](float xf, double& c0, double& c1, double& e0, double& e1, double& tau0, double& tau1) {
      const double xd = (double)xf;
      tau0 = dt + cQ * q_as_double(xd, invB0);
      tau1 = dt + cQ * q_as_double(xd, invB1);
      e0 = P0 * tau0;
      e1 = P1 * tau1;
      c0 = e0 + lam * tau0;
      c1 = e1 + lam * tau1;
    };
    bool redo = false;
    if (!general) {
      // the chunk's (tau, e) at r_min per (step, slot), once for the warp
      bool over = false;
      for (int k = k_l; k < kn; k += kstride) {
        const float xf = s_x[c & 1][k][r_l];
        const double tau0 = dt + cQ * q_as_double((double)xf, invB0);
        s_te[k][r_l][0] = make_double2(tau0, P0 * tau0);
        over |= xf > xthr_max;
      }
      const bool omax = __any_sync(0xFFFFFFFFu, over);
      if (omax) {  // some sample exceeds even the capacity at r_max (rare): that level's terms too
        for (int k = k_l; k < kn; k += kstride) {
          const double tau1 = dt + cQ * q_as_double((double)s_x[c & 1][k][r_l], invB1);
          s_te[k][r_l][1] = make_double2(tau1, P1 * tau1);
        }
      }
      __syncwarp();
      const double m1s = m1, E1s = E1, T1s = T1;
      bool tie = false;
      if (omax) {
#pragma unroll 4
        for (int k = 0; k < kn; ++k) {
          const double2 a = s_te[k][slot][0], b = s_te[k][slot][1];
          const double c0 = a.y + lam * a.x, c1 = b.y + lam * b.x;
          const bool up = c1 < c0;  // without a tie <=> RN(m1 + c1) < RN(m1 + c0)
          tie |= (m1 + c0) == (m1 + c1);
          m1 = m1 + (up ? c1 : c0);
          E1 = E1 + (up ? b.y : a.y);
          T1 = T1 + (up ? b.x : a.x);
        }
      } else {
        auto step0 = [&](int k) {
          const double2 a = s_te[k][slot][0];
          const double c0 = a.y + lam * a.x;
          const bool up = cf1 < c0;
          tie |= (m1 + c0) == (m1 + cf1);
          m1 = m1 + (up ? cf1 : c0);
          E1 = E1 + (up ? Pdt1 : a.y);
          T1 = T1 + (up ? dt : a.x);
        };
        if (kn == kBinChunk) {  // every chunk but the last: straight-line code
#pragma unroll
          for (int k = 0; k < kBinChunk; ++k) step0(k);
        } else {
#pragma unroll 8
          for (int k = 0; k < kn; ++k) step0(k);
        }
      }
      if (__any_sync(0xFFFFFFFFu, tie)) {
        m1 = m1s; E1 = E1s; T1 = T1s;
        redo = true;
      }
    }
    if (general || redo) {
#pragma unroll 1
      for (int k = 0; k < kn; ++k) {
        double c0, c1, e0, e1, tau0, tau1;
        costs(s_x[c & 1][k][slot], c0, c1, e0, e1, tau0, tau1);
        if (!general) {
          const double s0 = m1 + c0, s1 = m1 + c1;
          if (__any_sync(0xFFFFFFFFu, s0 == s1)) {
            V0 = s0; V1 = s1;
            E0 = E1 + e0; Ea = E1 + e1;
            T0 = T1 + tau0; Ta = T1 + tau1;
            general = true;
          } else {
            const bool up = s1 < s0;
            m1 = up ? s1 : s0;
            E1 = E1 + (up ? e1 : e0);
            T1 = T1 + (up ? tau1 : tau0);
          }
        } else {
          const bool st0 = V0 <= V1, st1 = V1 <= V0;
          const double nV0 = (st0 ? V0 : V1) + c0, nE0 = (st0 ? E0 : Ea) + e0, nT0 = (st0 ? T0 : Ta) + tau0;
          const double nV1 = (st1 ? V1 : V0) + c1, nE1 = (st1 ? Ea : E0) + e1, nT1 = (st1 ? Ta : T0) + tau1;
          V0 = nV0; E0 = nE0; T0 = nT0;
          V1 = nV1; Ea = nE1; Ta = nT1;
        }
      }
    }
    __syncwarp();  // s_x[c & 1] is restaged by chunk c + 2, s_te by the next chunk
  }
  if (general) {
    const bool b1 = V1 < V0;
    m1 = b1 ? V1 : V0;
    E1 = b1 ? Ea : E0;
    T1 = b1 ? Ta : T0;
  }
  if (!active) return;
  double* o = out + (n * nl + j) * 3;
  o[0] = m1;
  o[1] = E1;
  o[2] = T1;
}

// ---------------------------------------------------------------------------
// bound_grid_free_kernel<L>: the full level grid with free switches (the
// default platform) when nl divides 32.  As in the binary case, without a tie
// every level's new value is m1 + c_l (a1 always stays, every other level
// moves from it at no cost), so the state is (m1, E1, T1) and a step is
// m1 += min_l c_l, E1 += e_a, T1 += tau_a (a = the argmin) -- valid while
// RN(m1 + c_second) != RN(m1 + c_min) (monotone RN: then no other level ties
// the minimum).  Levels at or above l*(x) (capacity >= x: q = 0) cost the
// constants P_l dt + lam dt, increasing in l, so only cf_l* and cf_l*+1 can
// be the minimum or runner-up among them; the levels below l* are stretched
// (rare: ~4 % of the mix traces' samples exceed even the r_min capacity) and
// their (tau, e) are computed in the lane.  l* per (trace, step) comes from
// the warp's staged samples.  A tie anywhere in a chunk sends the warp back to
// the chunk's start: the careful pass rebuilds every level's state at the
// tie step (V_l = m1 + c_l, E_l = E1 + e_l, T_l = T1 + tau_l -- the oracle's
// own sums, as no level tied before) and finishes with the oracle's
// per-level recurrence.  Bit-identical to the oracle DP.
// ---------------------------------------------------------------------------
// shared loads by 32-bit window address (a generic pointer into a __shared__
// array indexed at run time makes the compiler re-derive the window base --
// an S2UR of the CTA id -- at every use)
__device__ __forceinline__ double lds_f64a(uint32_t a) {
  double v;
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ float lds_f32a(uint32_t a) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds_u8a(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}

template <int L, int P>
__global__ void __launch_bounds__(32)
bound_grid_free_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
                       const double* __restrict__ lambdas, int32_t nl, int32_t lstep, DevPlatform plat,
                       double bw_max, double p_lo, double p_span, const __grid_constant__ BoundThr thr,
                       double* __restrict__ out) {
  __shared__ float s_x[2][kBinChunk][16];       // [buffer][step][trace slot]
  __shared__ __align__(16) uint8_t s_ls[kBinChunk][16];  // l* of (step, slot)
  __shared__ double s_invB[L], s_P[L], s_Pdt[L];
  // per-level state after a tie (rare): per-thread local memory, so the
  // CTA's shared memory stays small enough for every warp to be resident
  double s_Vl[L], s_El[L], s_Tl[L];
  __shared__ float s_thr[32];
  const int lane = threadIdx.x;
  for (int i = lane; i < L; i += 32) {
    const int l = plat.r_min + i * lstep;
    const double B = (bw_max * (double)l) / (double)plat.r_max;
    s_invB[i] = 1.0 / B;
    s_P[i] = p_lo + (p_span * (double)(l - plat.r_min)) / (double)(plat.r_max - plat.r_min);
    s_Pdt[i] = s_P[i] * plat.dt;
  }
  s_thr[lane] = lane < L ? thr.x[lane] : INFINITY;
  __syncwarp();
  const uint32_t a_x = (uint32_t)__cvta_generic_to_shared(&s_x[0][0][0]);
  const uint32_t a_ls = (uint32_t)__cvta_generic_to_shared(&s_ls[0][0]);
  const uint32_t a_invB = (uint32_t)__cvta_generic_to_shared(&s_invB[0]);
  const uint32_t a_P = (uint32_t)__cvta_generic_to_shared(&s_P[0]);
  const uint32_t a_Pdt = (uint32_t)__cvta_generic_to_shared(&s_Pdt[0]);
  const uint32_t a_thr = (uint32_t)__cvta_generic_to_shared(&s_thr[0]);
  // P lanes per chain (h = lane % P): they split the stretched levels of a
  // slow step (l = h mod P) and merge by shuffles; 32 / P chains per warp
  constexpr int kLgP = P == 1 ? 0 : (P == 2 ? 1 : (P == 4 ? 2 : 3));
  const int h = lane & (P - 1), ch = lane >> kLgP;
  const int lgnl = __ffs(nl) - 1, lgtpw = 5 - kLgP - lgnl, tpw = 1 << lgtpw;
  const int slot = ch >> lgnl, j = ch & (nl - 1);
  const int64_t n0 = (int64_t)blockIdx.x * tpw;
  const int64_t n = n0 + slot;
  const bool active = n < N;
  const double lam = lambdas[j];
  const double dt = plat.dt, cQ = plat.cQ;
  const double lt0 = lam * dt;
  const double Pdt0 = s_Pdt[0], cf0 = Pdt0 + lt0, cf1 = L > 1 ? s_Pdt[1] + lt0 : INFINITY;
  for (int i = lane; i < kBinChunk * 16; i += 32) (&s_ls[0][0])[i] = 0;  // bytes >= tpw stay 0
  __syncwarp();
  // t = 0 runs at r_max (every other level unreachable)
  double m1, E1, T1;
  {
    const double xd = (double)(active ? __ldg(x + n) : 0.0f);
    const double tau = dt + cQ * q_as_double(xd, s_invB[L - 1]);
    const double e = s_P[L - 1] * tau;
    m1 = e + lam * tau;
    E1 = e;
    T1 = tau;
  }
  bool general = false;
  const int r_l = lane & (tpw - 1), k_l = lane >> lgtpw, kstride = 32 >> lgtpw;
  const bool r_ok = n0 + r_l < N;
  const float* xl = x + (r_ok ? n0 + r_l : 0);
  const int64_t ldk = (int64_t)kstride * ld;
  auto stage = [&](int64_t c) {
    const int64_t t0 = 1 + c * kBinChunk;
    const float* src = xl + (t0 + k_l) * ld;
    float* dst = &s_x[c & 1][k_l][r_l];
    int64_t t = t0 + k_l;
    for (int i = 0; i < tpw; ++i) {
      const bool ok = r_ok && t < T;
      cp_async4z(dst, ok ? src : x, ok);
      src += ldk;
      dst += kstride * 16;
      t += kstride;
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  const int64_t nch = (T - 1 + kBinChunk - 1) / kBinChunk;
  if (nch > 0) stage(0);
  for (int64_t c = 0; c < nch; ++c) {
    if (c + 1 < nch) {
      stage(c + 1);
      asm volatile("cp.async.wait_group 1;" ::: "memory");
    } else {
      asm volatile("cp.async.wait_group 0;" ::: "memory");
    }
    __syncwarp();
    const int64_t t0 = 1 + c * kBinChunk;
    const int kn = (int)(T - t0 < kBinChunk ? T - t0 : kBinChunk);
    // l* of every (step, slot) of the chunk, once
    const uint32_t a_xc = a_x + (uint32_t)((c & 1) * kBinChunk * 16 * 4);
    for (int k = k_l; k < kn; k += kstride) {
      const float xf = lds_f32a(a_xc + (uint32_t)(k * 64 + r_l * 4));
      int ls = 0;
      while (ls < L && xf > lds_f32a(a_thr + 4u * ls)) ++ls;  // capacities increase with the level
      s_ls[k][r_l] = (uint8_t)ls;
    }
    __syncwarp();
    // steps where some trace of the warp is stretched at r_min (bit k)
    uint32_t slowm;
    {
      const uint4 w = *reinterpret_cast<const uint4*>(&s_ls[lane][0]);  // bytes >= tpw stay 0
      slowm = __ballot_sync(0xFFFFFFFFu, lane < kn && (w.x | w.y | w.z | w.w) != 0u);
    }
    // (c, e, tau) of level l at step k of this lane's trace
    auto level = [&](int k, int l, int ls, double& cl, double& el, double& tl) {
      if (l < ls) {
        tl = dt + cQ * q_as_double((double)lds_f32a(a_xc + (uint32_t)(k * 64 + slot * 4)), lds_f64a(a_invB + 8u * l));
        el = lds_f64a(a_P + 8u * l) * tl;
        cl = el + lam * tl;
      } else {
        tl = dt; el = lds_f64a(a_Pdt + 8u * l);
        cl = el + lt0;
      }
    };
    bool redo = false;
    if (!general) {
      const double m1s = m1, E1s = E1, T1s = T1;
      bool tie = false;
      for (int k = 0; k < kn;) {
        // a run of steps where no trace of the warp is stretched: every
        // level costs its constant, so the minimum is cf_0 and the runner-up
        // cf_1 -- three adds and the tie test per step
        const uint32_t rest = slowm >> k;  // k < 32
        const int kend = rest ? k + __ffs(rest) - 1 : kn;
#pragma unroll 4
        for (; k < kend; ++k) {
          const double m1n = m1 + cf0;
          tie |= (m1 + cf1) == m1n;
          m1 = m1n;
          E1 = E1 + Pdt0;
          T1 = T1 + dt;
        }
        if (k >= kn) break;
        const int ls = (int)lds_u8a(a_ls + (uint32_t)(k * 16 + slot));
        double cmin = INFINITY, c2 = INFINITY, ea = 0.0, ta = 0.0;
        if (ls < L && h == 0) {  // the lowest unstretched level, and the next one
          ea = lds_f64a(a_Pdt + 8u * ls);
          ta = dt;
          cmin = ea + lt0;
          if (ls + 1 < L) c2 = lds_f64a(a_Pdt + 8u * (ls + 1)) + lt0;
        }
        for (int l = h; l < ls; l += P) {  // stretched levels (rare), this lane's share
          double cl, el, tl;
          level(k, l, ls, cl, el, tl);
          const bool lt = cl < cmin;
          c2 = lt ? cmin : (cl < c2 ? cl : c2);
          cmin = lt ? cl : cmin;
          ea = lt ? el : ea;
          ta = lt ? tl : ta;
        }
#pragma unroll
        for (int sh = 1; sh < P; sh <<= 1) {  // merge the shares (an exact equality of costs is a tie either way)
          const double oc = __shfl_xor_sync(0xFFFFFFFFu, cmin, sh), oc2 = __shfl_xor_sync(0xFFFFFFFFu, c2, sh);
          const double oe = __shfl_xor_sync(0xFFFFFFFFu, ea, sh), ot = __shfl_xor_sync(0xFFFFFFFFu, ta, sh);
          const bool lt = oc < cmin;
          const double lose = lt ? cmin : oc;
          c2 = lose < c2 ? lose : c2;
          c2 = oc2 < c2 ? oc2 : c2;
          cmin = lt ? oc : cmin;
          ea = lt ? oe : ea;
          ta = lt ? ot : ta;
        }
        const double m1n = m1 + cmin;
        tie |= (m1 + c2) == m1n;  // another level's value equals the minimum
        m1 = m1n;
        E1 = E1 + ea;
        T1 = T1 + ta;
        ++k;
      }
      if (__any_sync(0xFFFFFFFFu, tie)) {
        m1 = m1s; E1 = E1s; T1 = T1s;
        redo = true;
      }
    }
    if (general || redo) {
#pragma unroll 1
      for (int k = 0; k < kn; ++k) {
        const int ls = s_ls[k][slot];
        if (!general) {
          double cmin = INFINITY, c2 = INFINITY, ea = 0.0, ta = 0.0;
#pragma unroll
          for (int l = 0; l < L; ++l) {
            double cl, el, tl;
            level(k, l, ls, cl, el, tl);
            const bool lt = cl < cmin;
            c2 = lt ? cmin : (cl < c2 ? cl : c2);
            cmin = lt ? cl : cmin;
            ea = lt ? el : ea;
            ta = lt ? tl : ta;
          }
          const double m1n = m1 + cmin;
          if (__any_sync(0xFFFFFFFFu, (m1 + c2) == m1n)) {
            // a tie: every level's state after this step, the oracle's sums
#pragma unroll 1
            for (int l = 0; l < L; ++l) {
              double cl, el, tl;
              level(k, l, ls, cl, el, tl);
              s_Vl[l] = m1 + cl;
              s_El[l] = E1 + el;
              s_Tl[l] = T1 + tl;
            }
            general = true;
          } else {
            m1 = m1n;
            E1 = E1 + ea;
            T1 = T1 + ta;
          }
        } else {
          // the oracle's recurrence with free switches: best other level o
          // (lowest on ties), stay when V_l <= V_o
          int a1 = 0, a2 = 1;
          if (s_Vl[1] < s_Vl[0]) { a1 = 1; a2 = 0; }
#pragma unroll 1
          for (int l = 2; l < L; ++l) {
            const double v = s_Vl[l];
            if (v < s_Vl[a1]) { a2 = a1; a1 = l; }
            else if (v < s_Vl[a2]) a2 = l;
          }
          const double V1 = s_Vl[a1], E1o = s_El[a1], T1o = s_Tl[a1];
          const double V2 = s_Vl[a2], E2o = s_El[a2], T2o = s_Tl[a2];
#pragma unroll 1
          for (int l = 0; l < L; ++l) {
            double cl, el, tl;
            level(k, l, ls, cl, el, tl);
            const bool oa = l != a1;  // best other level: a1, or a2 for a1 itself
            const double vo = oa ? V1 : V2, eo = oa ? E1o : E2o, to = oa ? T1o : T2o;
            const double v = s_Vl[l];
            const bool stay = v <= vo;
            s_Vl[l] = (stay ? v : vo) + cl;
            s_El[l] = (stay ? s_El[l] : eo) + el;
            s_Tl[l] = (stay ? s_Tl[l] : to) + tl;
          }
        }
      }
    }
    __syncwarp();  // s_x[c & 1] is restaged by chunk c + 2, s_te / s_ls by the next chunk
  }
  if (general) {
    int b = 0;
    for (int l = 1; l < L; ++l)
      if (s_Vl[l] < s_Vl[b]) b = l;
    m1 = s_Vl[b]; E1 = s_El[b]; T1 = s_Tl[b];
  }
  if (!active || h) return;
  double* o = out + (n * nl + j) * 3;
  o[0] = m1;
  o[1] = E1;
  o[2] = T1;
}

#ifndef MAGUS_GRID_P
#define MAGUS_GRID_P 8  // most lanes per (trace, lambda) chain of the free-switch grid DP
#endif
constexpr int kGridP = MAGUS_GRID_P;

int launch_bound(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
                 const double* lambdas_dev, int32_t nl, bool full_grid, const DevPlatform& plat,
                 double bw_max, double p_lo, double p_span, double* out) {
  const int32_t L = full_grid ? plat.r_max - plat.r_min + 1 : 2;
  const int32_t lstep = full_grid ? 1 : plat.r_max - plat.r_min;
  const unsigned blocks = (unsigned)((N * nl + kBoundThreads - 1) / kBoundThreads);
  // (every lambda and switch cost is finite and >= 0, validated by the caller)
  BoundThr thr;
  for (int i = 0; i < 32; ++i) {
    const int l = plat.r_min + i * lstep;
    thr.x[i] = i < L ? stretch_threshold(1.0 / ((bw_max * (double)l) / (double)plat.r_max)) : INFINITY;
  }
  const unsigned warps = (unsigned)((N * nl + 15) / 16);  // 16 chains (2 lanes each) per warp
  if (L == 2 && plat.e_sw == 0.0 && plat.t_sw == 0.0 && nl >= 2 && 32 % nl == 0)
    bound_binary_shared_kernel<<<(unsigned)((N + (32 / nl) - 1) / (32 / nl)), 32, 0, s>>>(
        x, N, T, ld, lambdas_dev, nl, plat, bw_max, p_lo, p_span, thr.x[1], out);
  else if (L == 2 && plat.e_sw == 0.0 && plat.t_sw == 0.0)
    bound_binary_free_kernel<<<(unsigned)((N * nl + 31) / 32), 32, 0, s>>>(x, N, T, ld, lambdas_dev, nl, plat,
                                                                         bw_max, p_lo, p_span, thr.x[0], thr.x[1], out);
  else if (L == 2)  // two levels with switch costs: the branch-free per-step kernel
    bound_binary_kernel<<<blocks, kBoundThreads, 0, s>>>(x, N, T, ld, lambdas_dev, nl, plat, bw_max, p_lo,
                                                         p_span, out);
  else if ((L == 15 || L == 18) && plat.e_sw == 0.0 && plat.t_sw == 0.0 && nl >= 2 && nl <= 16 &&
           32 % nl == 0) {
    // lanes per chain: as many as the warp allows up to kGridP (more lanes
    // split a slow step's stretched levels further; measured best at 8 for
    // the mix traces, 18.3 vs 21.4 ms at 4)
    const int P = std::min(kGridP, 32 / nl);
    const unsigned wb = (unsigned)((N + (32 / P / nl) - 1) / (32 / P / nl));
    auto go = [&](auto kern) {
      kern<<<wb, 32, 0, s>>>(x, N, T, ld, lambdas_dev, nl, lstep, plat, bw_max, p_lo, p_span, thr, out);
    };
    if (L == 15) {
      if (P >= 8) go(bound_grid_free_kernel<15, 8>);
      else if (P == 4) go(bound_grid_free_kernel<15, 4>);
      else go(bound_grid_free_kernel<15, 2>);
    } else {
      if (P >= 8) go(bound_grid_free_kernel<18, 8>);
      else if (P == 4) go(bound_grid_free_kernel<18, 4>);
      else go(bound_grid_free_kernel<18, 2>);
    }
  } else if (L == 15)
    bound_dp_kernel<15><<<warps, 32, 0, s>>>(x, N, T, ld, lambdas_dev, nl, lstep, plat, bw_max, p_lo, p_span, thr,
                                             out);
  else if (L == 18)
    bound_dp_kernel<18><<<warps, 32, 0, s>>>(x, N, T, ld, lambdas_dev, nl, lstep, plat, bw_max, p_lo, p_span, thr,
                                             out);
  else  // other level counts: the generic kernel
    bound_kernel<32><<<blocks, kBoundThreads, 0, s>>>(x, N, T, ld, lambdas_dev, nl, L, plat.r_min, lstep,
                                                      plat, bw_max, p_lo, p_span, out);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
