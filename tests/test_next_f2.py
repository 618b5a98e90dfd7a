"""NEXT row f2: offline-optimal schedules under model M (a lower bound on what
any uncore policy -- MAGUS included -- can reach), by DP over the levels.

The DP is pinned by brute force over every schedule on tiny traces (the
same objective written out as a plain sum), by the property that MAGUS never
beats it, and by the parametric behaviour in lambda; the CUDA kernel must
reproduce the oracle's DP bit for bit."""
from __future__ import annotations

import itertools
import math

import numpy as np
import pytest

import gen
import oracle

R_MIN, R_MAX = 8, 22


def _brute(x, lam, plat_kw, levels):
    """min over every schedule of sum_t (P_l tau + lam tau) + switch costs,
    accumulated in time order exactly like the definition."""
    p = dict(dict(r_min=8, r_max=22, dt=0.2, bw_max=32000.0, beta=1.0, p_other=218.0, p_unc_min=0.0,
                  p_unc_max=82.0, e_sw=0.0, t_sw=0.0), **plat_kw)
    cQ = (p["dt"] * p["beta"]) / 16777216.0

    def q(xv, l):
        r = float(np.float32(xv)) * (1.0 / ((p["bw_max"] * l) / p["r_max"]))
        if r > 1.0:
            s = min(r - 1.0, 32768.0)
            return int(s * 16777216.0)
        return 0

    def P(l):
        return (p["p_other"] + p["p_unc_min"]) + ((p["p_unc_max"] - p["p_unc_min"]) * (l - p["r_min"])) / (p["r_max"] - p["r_min"])

    T = len(x)
    best = None
    for sched in itertools.product(levels, repeat=T - 1):   # dec[0..T-2]; dec[T-1] only affects nothing
        lv = [p["r_max"]] + list(sched)                       # level of interval t = dec[t-1]
        cost = 0.0
        for t in range(T):
            tau = p["dt"] + cQ * float(q(x[t], lv[t]))
            e = P(lv[t]) * tau
            if t >= 2 and lv[t] != lv[t - 1]:
                cost = cost + (p["e_sw"] + lam * p["t_sw"])
            cost = cost + (e + lam * tau)
        best = cost if best is None else min(best, cost)
    return best


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("lam,plat_kw", [(0.0, {}), (300.0, {}), (1e4, {}),
                                         (50.0, dict(e_sw=3.0, t_sw=0.01)), (0.0, dict(e_sw=500.0))])
def test_dp_equals_brute_force_binary(seed, lam, plat_kw):
    rng = np.random.default_rng(seed)
    x = rng.choice([300.0, 9000.0, 12500.0, 18000.0, 26000.0, 40000.0], size=11).astype(np.float32)
    got = oracle.offline_bound(x, lam, oracle.platform(**plat_kw))
    assert got[0] == _brute(x, lam, plat_kw, [R_MIN, R_MAX])


@pytest.mark.parametrize("seed", range(2))
def test_dp_equals_brute_force_full_grid(seed):
    rng = np.random.default_rng(10 + seed)
    x = rng.choice([300.0, 9000.0, 12500.0, 26000.0], size=5).astype(np.float32)
    kw = dict(r_min=8, r_max=11, bw_max=20000.0, e_sw=1.0, t_sw=0.001)
    got = oracle.offline_bound(x, 100.0, oracle.platform(**kw), full_grid=True)
    assert got[0] == _brute(x, 100.0, kw, [8, 9, 10, 11])


def test_magus_never_beats_the_offline_optimum():
    """north_star: an exhaustive lower bound MAGUS can never beat -- here at
    scale through the DP (lambda = 0: least energy of any schedule)."""
    x = gen.gen_traces(gen.SEEDS[2], 24, 2000)
    r = oracle.replay(x, oracle.policy())
    for n in range(24):
        e_opt = oracle.offline_bound(x[:, n], 0.0)[1]
        e_full = oracle.offline_bound(x[:, n], 0.0, full_grid=True)[1]
        assert e_opt <= r.summary[0, n]["energy"] * (1 + 1e-12)
        assert e_full <= e_opt * (1 + 1e-12)            # more levels can only help


def test_lambda_trades_energy_for_time():
    x = gen.gen_traces(gen.SEEDS[1], 6, 1500)
    for n in range(6):
        rows = [oracle.offline_bound(x[:, n], lam) for lam in (0.0, 10.0, 100.0, 1e3, 1e5)]
        e = [r[1] for r in rows]
        t = [r[2] for r in rows]
        assert all(t[i + 1] <= t[i] * (1 + 1e-12) for i in range(4))
        assert all(e[i + 1] >= e[i] * (1 - 1e-12) for i in range(4))
        base = oracle.replay(x[:, n:n + 1], oracle.policy()).base["time"][0]
        assert math.isclose(t[-1], base, rel_tol=1e-12)  # huge lambda: all intervals at max


# ------------------------------- GPU parity --------------------------------

@pytest.mark.gpu
@pytest.mark.parametrize("full_grid,r_max", [(False, 22), (True, 22), (True, 25), (True, 12), (False, 25)])
def test_gpu_offline_bound_bit_exact(full_grid, r_max):
    """Binary and full-grid DPs (15 and 18 ratios: the register-resident
    kernels; 5 ratios: the generic one) vs the oracle DP, bit for bit."""
    torch = pytest.importorskip("torch")
    magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")
    N, T = 150, 1777
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    lams = [0.0, 25.0, 400.0, 1e6]
    plat = magus.platform_preset()
    plat.e_switch_j, plat.t_switch_s = 2.0, 0.004
    plat.ratio_max = r_max
    plat_o = oracle.platform(e_sw=2.0, t_sw=0.004, r_max=r_max)
    with magus.Context(device=0, platform=plat) as ctx:
        out = ctx.offline_bound(torch.from_numpy(x).cuda(), lams, full_grid=full_grid)
        torch.cuda.synchronize()
        got = out.cpu().numpy()
    for n in range(0, N, 7):
        for j, lam in enumerate(lams):
            ref = oracle.offline_bound(x[:, n], lam, plat_o, full_grid=full_grid)
            assert np.array_equal(got[n, j], ref), (n, lam)


@pytest.mark.gpu
@pytest.mark.parametrize("full_grid", [False, True])
@pytest.mark.parametrize("case", ["free_switch", "flat_power_ties", "tiny_switch", "adversarial", "short"])
@pytest.mark.parametrize("nl", [3, 4, 8])
def test_gpu_offline_bound_modes_bit_exact(full_grid, case, nl):
    """The throughput kernel's two bookkeeping modes: free
    switches (the paper's default: scalar path sums), equal power at every
    level (exact ties everywhere: per-level histories and the lowest-index
    rule), a tiny switch cost (mode changes mid-chunk), adversarial traces,
    and T = 1, 2, 33, 34 -- all bit for bit against the oracle DP."""
    torch = pytest.importorskip("torch")
    magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")
    kw = {"free_switch": {}, "flat_power_ties": dict(p_unc_min=41.0, p_unc_max=41.0),
          "tiny_switch": dict(e_sw=1e-9, p_unc_min=41.0, p_unc_max=41.0000001),
          "adversarial": dict(e_sw=0.5), "short": {}}[case]
    plat = magus.platform_preset()
    plat.e_switch_j = kw.get("e_sw", 0.0)
    plat.p_unc_min_w = kw.get("p_unc_min", plat.p_unc_min_w)
    plat.p_unc_max_w = kw.get("p_unc_max", plat.p_unc_max_w)
    plat_o = oracle.platform(**kw)
    # 4 / 8 lambdas: a warp holds whole traces (the binary kernel's shared
    # per-(trace, step) model-M terms; the free-switch grid kernel with 8 /
    # 4 lanes per chain); 3: traces straddle warps (the generic kernels)
    lams = {3: [0.0, 25.0, 400.0], 4: [0.0, 25.0, 400.0, 1e6],
            8: [0.0, 10.0, 25.0, 40.0, 160.0, 400.0, 2560.0, 1e6]}[nl]
    Ts = [1, 2, 33, 34] if case == "short" else [1999]
    kind = gen.KIND_ADVERSARIAL if case == "adversarial" else gen.KIND_MIX
    with magus.Context(device=0, platform=plat) as ctx:
        for T in Ts:
            N = 70
            x = gen.gen_traces(gen.SEEDS[2], N, T, kind=kind)
            out = ctx.offline_bound(torch.from_numpy(x).cuda(), lams, full_grid=full_grid)
            torch.cuda.synchronize()
            got = out.cpu().numpy()
            for n in range(0, N, 3):
                for j, lam in enumerate(lams):
                    ref = oracle.offline_bound(x[:, n], lam, plat_o, full_grid=full_grid)
                    assert np.array_equal(got[n, j], ref), (case, T, n, lam)
