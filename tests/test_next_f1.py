"""NEXT row f1: Sec. 6.3 burst Jaccard and Sec. 6.4 Pareto front, in batch.

CPU tests pin the oracle (hand-derived counts, set identities, brute force);
GPU tests compare both CUDA kernels with it bit for bit.
P@41094-P@41603 (Sec. 6.3: bursts = throughput above a predefined threshold,
Jaccard of the binary sequences of the MAGUS and max-uncore runs);
P@43882-P@44696 (Sec. 6.4 / Fig. 7: energy/runtime Pareto fronts)."""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

R_MIN, R_MAX = 8, 22
B_MIN = 32000.0 * 8 / 22    # 11636.36 MB/s: capacity at the min ratio (model M 4.1)


def _plat(theta):
    return oracle.platform(burst=theta)


# ------------------------------- CPU pins ---------------------------------

def test_jaccard_hand_example():
    """Burst of width 1 (20000 MB/s) at t0 = 20 on a 1000 MB/s base, then a
    second one at t = 35.  MAGUS (golden burst_w1): min from round 29 on, so
    interval 36 (= dec[35]) ... the second burst at t = 35 runs at level
    dec[34] = min: its delivered throughput is capped at B_min = 11636 MB/s.
    With theta = 12000: B = {20, 35}, A = {20}: Jaccard 1/2.
    With theta = 10000: the cap does not hide it: A = B, Jaccard 1."""
    x = np.full(40, 1000.0, np.float32)
    x[20] = x[35] = 20000.0
    for theta, want in ((12000.0, (1, 2, 1, 2)), (10000.0, (2, 2, 2, 2)), (25000.0, (0, 0, 0, 0))):
        r = oracle.replay(x, oracle.policy(), _plat(theta), want_dec=True)
        s = r.summary[0, 0]
        assert (s["n_burst_magus"], s["n_burst_base"], s["n_burst_inter"], s["n_burst_union"]) == want


def test_jaccard_set_identities_and_bounds():
    x = gen.gen_traces(gen.SEEDS[2], 64, 3000)
    for theta in (500.0, 5000.0, 11000.0, 11637.0, 15000.0, 30000.0, 40000.0):
        r = oracle.replay(x, oracle.policy(), _plat(theta))
        s = r.summary[0]
        # A (MAGUS) is a subset of B (baseline): capacities B_l <= B_max
        assert (s["n_burst_inter"] == s["n_burst_magus"]).all()
        assert (s["n_burst_union"] == s["n_burst_base"]).all()
        if theta < B_MIN:   # no level hides a burst
            assert (s["n_burst_magus"] == s["n_burst_base"]).all()
        if theta >= 32000.0:
            assert (s["n_burst_base"] == 0).all()
        # the base count is config independent and equals a direct count
        assert np.array_equal(s["n_burst_base"], (x.astype(np.float64) > theta).sum(axis=0))
        w, f = oracle.totals(s, r.base, x.shape[0], _plat(theta))
        assert w[15] == s["n_burst_base"].sum() and w[16] == s["n_burst_magus"].sum()
        assert 0.0 <= f[6] <= 1.0


def test_jaccard_counts_match_decisions():
    """|A| recomputed from the oracle's decision sequence: interval t runs at
    dec[t-1] (reading R6), so a burst at t is kept unless dec[t-1] = min and
    B_min <= theta."""
    x = gen.gen_traces(gen.SEEDS[1], 16, 2000)
    theta = 12000.0
    r = oracle.replay(x, oracle.policy(), _plat(theta), want_dec=True)
    lvl = np.concatenate([np.full((16, 1), R_MAX), r.dec[0][:, :-1]], axis=1).T  # [T, N]
    burst = x.astype(np.float64) > theta
    kept = burst & (lvl == R_MAX)
    assert np.array_equal(kept.sum(axis=0), r.summary[0]["n_burst_magus"])


def test_pareto_front_definition():
    e = np.array([5.0, 4.0, 4.0, 6.0, 3.0, 3.0])
    t = np.array([1.0, 2.0, 2.0, 0.5, 5.0, 6.0])
    on = oracle.pareto_front(e, t)
    # 5 is dominated by 4 (same energy, longer time); duplicates (1, 2) both stay
    assert on.tolist() == [True, True, True, True, True, False]
    rng = np.random.default_rng(0)
    for _ in range(50):   # brute force: on front <=> no point weakly better in both, strictly in one
        e, t = rng.integers(0, 6, 12).astype(float), rng.integers(0, 6, 12).astype(float)
        on = oracle.pareto_front(e, t)
        for i in range(12):
            dom = any(e[j] <= e[i] and t[j] <= t[i] and (e[j] < e[i] or t[j] < t[i]) for j in range(12))
            assert on[i] == (not dom)


def test_pareto_host_matches_oracle():
    magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")
    x = gen.gen_traces(gen.SEEDS[3], 40, 1500)
    pols = magus.grid_fleet64()
    po = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                               tau_dec=p.tau_dec, t_hi=p.t_hi) for p in pols])
    r = oracle.replay(x, po)
    words, fl = [], []
    for c in range(len(pols)):
        w, f = oracle.totals(r.summary[c], r.base, 1500)
        words.append(w)
        fl.append(f)
    fl = np.array(fl)
    got = magus.pareto_front_host(np.array(words))
    assert np.array_equal(got, oracle.pareto_front(fl[:, 0], fl[:, 1]))
    assert got.any()


# ------------------------------- GPU parity --------------------------------

@pytest.mark.gpu
@pytest.mark.parametrize("theta", [10000.0, 12000.0, 20000.0])
def test_gpu_bursts_bit_exact(theta):
    torch = pytest.importorskip("torch")
    magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")
    N, T = 260, 3001
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    plat = magus.platform_preset()
    plat.burst_mbs = theta
    pols = [magus.make_policy(), magus.make_policy(W=4, t_hi=0.2), magus.make_policy(W=10, t_hi=0.5),
            magus.make_policy(W=7, H=13, tau_inc=90, tau_dec=-90)]
    po = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                               tau_dec=p.tau_dec, t_hi=p.t_hi) for p in pols])
    ref = oracle.replay(x, po, _plat(theta))
    xd = torch.zeros((T, 260), dtype=torch.float32, device="cuda:0")
    xd[:, :N] = torch.from_numpy(x).cuda()
    with magus.Context(device=0, platform=plat) as ctx:
        for kernel, segs, bundle in ((magus.KERNEL_REFERENCE, 0, 0), (magus.KERNEL_STREAM, 0, 0),
                                     (magus.KERNEL_STREAM, 9, 4), (magus.KERNEL_STREAM, 3, 2)):
            ctx.set_option(magus.OPT_KERNEL, kernel)
            ctx.set_option(magus.OPT_SEGMENTS, segs)
            ctx.set_option(magus.OPT_BUNDLE, bundle)
            r = ctx.replay(xd, pols, n_traces=N)
            torch.cuda.synchronize()
            got = r.summary_numpy()
            for f in ("n_burst_base", "n_burst_magus", "energy_j", "n_changes", "digest"):
                of = {"energy_j": "energy"}.get(f, f)
                assert np.array_equal(got[f], ref.summary[of]), (f, kernel, segs, bundle)
            tot = r.totals_numpy()
            for c in range(len(pols)):
                w, fo = oracle.totals(ref.summary[c], ref.base, T, _plat(theta))
                assert np.array_equal(tot[c], w)
                d = ctx.totals_derive(tot[c])
                assert d["jaccard"] == fo[6] and d["energy_j"] == fo[0]
            # the front from the oracle's own fleet energies/times (never the library's)
            on = ctx.pareto_front(r.totals)
            fos = [oracle.totals(ref.summary[c], ref.base, T, _plat(theta))[1] for c in range(len(pols))]
            assert np.array_equal(on, oracle.pareto_front([fo[0] for fo in fos], [fo[1] for fo in fos]))
