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

// The full ratio grid with a compile-time level count L (the platforms'
// 15 and 18 ratios): every per-level array is register-resident (fully
// unrolled loops; the chosen predecessor's energy / time are picked by
// selects, not by a dynamic index), in-place update.  Same fp64 operations
// in the same order as bound_kernel.
template <int L>
__global__ void __launch_bounds__(kBoundThreads)
bound_grid_kernel(const float* __restrict__ x, int64_t N, int64_t T, int64_t ld,
                  const double* __restrict__ lambdas, int32_t nl, DevPlatform plat, double bw_max,
                  double p_lo, double p_span, double* __restrict__ out) {
  __shared__ double s_invB[L], s_P[L];
  __shared__ float s_x[32][kBoundThreads];
  for (int i = threadIdx.x; i < L; i += blockDim.x) {
    const int l = plat.r_min + i;
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
  constexpr int imax = L - 1;  // ascending level set ending at r_max

  double V[L], E[L], Tm[L];
#pragma unroll
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
    const double xd = (double)xt;
    if (t == 0) {
      const double tau = plat.dt + plat.cQ * q_as_double(xd, s_invB[imax]);
      const double e = s_P[imax] * tau;
      V[imax] = e + lam * tau;
      E[imax] = e;
      Tm[imax] = tau;
      continue;
    }
    // best and second best previous state (lowest index on ties)
    int a1 = 0;
    double m1 = V[0];
#pragma unroll
    for (int i = 1; i < L; ++i)
      if (V[i] < m1) { m1 = V[i]; a1 = i; }
    int a2 = -1;
    double m2 = INFINITY;
#pragma unroll
    for (int i = 0; i < L; ++i)
      if (i != a1 && (a2 < 0 || V[i] < m2)) { m2 = V[i]; a2 = i; }
    double E1 = 0.0, T1 = 0.0, E2 = 0.0, T2 = 0.0;
#pragma unroll
    for (int i = 0; i < L; ++i) {
      if (i == a1) { E1 = E[i]; T1 = Tm[i]; }
      if (i == a2) { E2 = E[i]; T2 = Tm[i]; }
    }
    const bool sw = t >= 2;
#pragma unroll
    for (int i = 0; i < L; ++i) {
      const bool isa1 = i == a1;
      const double other = isa1 ? m2 : m1;
      const double move = sw ? other + sw_c : other;
      double v, e0, t0;
      if (V[i] <= move) {
        v = V[i]; e0 = E[i]; t0 = Tm[i];
      } else {
        const double Eo = isa1 ? E2 : E1, To = isa1 ? T2 : T1;
        v = move;
        e0 = sw ? Eo + plat.e_sw : Eo;
        t0 = sw ? To + plat.t_sw : To;
      }
      const double tau = plat.dt + plat.cQ * q_as_double(xd, s_invB[i]);
      const double e = s_P[i] * tau;
      V[i] = v + (e + lam * tau);
      E[i] = e0 + e;
      Tm[i] = t0 + tau;
    }
  }
  if (!active) return;
  int b = 0;
  double vb = V[0], eb = E[0], tb = Tm[0];
#pragma unroll
  for (int i = 1; i < L; ++i)
    if (V[i] < vb) { b = i; vb = V[i]; eb = E[i]; tb = Tm[i]; }
  double* o = out + ((int64_t)n * nl + j) * 3;
  o[0] = vb;
  o[1] = eb;
  o[2] = tb;
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

int launch_bound(cudaStream_t s, const float* x, int64_t N, int64_t T, int64_t ld,
                 const double* lambdas_dev, int32_t nl, bool full_grid, const DevPlatform& plat,
                 double bw_max, double p_lo, double p_span, double* out) {
  const int32_t L = full_grid ? plat.r_max - plat.r_min + 1 : 2;
  const int32_t lstep = full_grid ? 1 : plat.r_max - plat.r_min;
  const unsigned blocks = (unsigned)((N * nl + kBoundThreads - 1) / kBoundThreads);
  if (L == 2)
    bound_binary_kernel<<<blocks, kBoundThreads, 0, s>>>(x, N, T, ld, lambdas_dev, nl, plat, bw_max, p_lo,
                                                         p_span, out);
  else if (L == 15)
    bound_grid_kernel<15><<<blocks, kBoundThreads, 0, s>>>(x, N, T, ld, lambdas_dev, nl, plat, bw_max, p_lo,
                                                           p_span, out);
  else if (L == 18)
    bound_grid_kernel<18><<<blocks, kBoundThreads, 0, s>>>(x, N, T, ld, lambdas_dev, nl, plat, bw_max, p_lo,
                                                           p_span, out);
  else
    bound_kernel<32><<<blocks, kBoundThreads, 0, s>>>(x, N, T, ld, lambdas_dev, nl, L, plat.r_min, lstep,
                                                      plat, bw_max, p_lo, p_span, out);
  return cudaGetLastError() == cudaSuccess ? 1 : -1;
}

}  // namespace magus
