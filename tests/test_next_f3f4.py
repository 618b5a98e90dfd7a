"""NEXT rows f3 (closed-loop replay) and f4 (gradual step rule).

f3: the monitor observes the delivered throughput min(x_t, B(l_t)) (model M
capacity at the ratio that governed interval t) -- Fig. 5's shortfall at min
uncore (P@37360, P@38709).  f4: +-step ratio per event instead of the jump to
max/min (the contrast the paper draws with UPS's gradual stepping, P@35554,
P@30719).  Hand-derived worked examples live in tests/golden/
(closed_loop_shortfall.txt, open_loop_same_trace.txt, gradual_step_down.txt).
"""
from __future__ import annotations

import itertools
import math
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle

R_MIN, R_MAX = 8, 22
B_MIN = 32000.0 * 8 / 22


def _all_traces(alphabet, T):
    return np.ascontiguousarray(np.array(list(itertools.product(alphabet, repeat=T)), np.float32).T)


# ------------------------------- CPU pins: f4 ------------------------------

@pytest.mark.parametrize("step", [R_MAX - R_MIN, 20, 100])
def test_gradual_with_full_step_is_the_paper_rule(step):
    """A step >= r_max - r_min reaches the bound in one event: identical to the
    jump rule, decisions and model-M results bit for bit."""
    x = gen.gen_traces(gen.SEEDS[2], 64, 3000)
    a = oracle.replay(x, oracle.policy(), want_dec=True)
    b = oracle.replay(x, oracle.policy(variant=2, step=step), want_dec=True)
    assert np.array_equal(a.dec, b.dec) and np.array_equal(a.summary, b.summary)


@pytest.mark.parametrize("step", [1, 2, 5])
def test_gradual_literal_equals_walk_and_invariants(step):
    pol = oracle.policy(W=4, H=5, t_hi=0.4, variant=2, step=step)
    x = _all_traces([0.0, 30000.0], 12)
    a = oracle.replay(x, pol, want_dec=True)
    b = oracle.replay(x, pol, want_dec=True, closed_form=True)
    assert np.array_equal(a.dec, b.dec) and np.array_equal(a.summary, b.summary)
    x = gen.gen_traces(gen.SEEDS[3], 48, 4000)
    pol = oracle.policy(variant=2, step=step)
    a = oracle.replay(x, pol, want_dec=True)
    b = oracle.replay(x, pol, want_dec=True, closed_form=True)
    assert np.array_equal(a.dec, b.dec) and np.array_equal(a.summary, b.summary)
    d = a.dec[0]
    assert d.min() >= R_MIN and d.max() <= R_MAX
    jumps = np.diff(d, axis=1)
    hi_next = a.hi[0][:, 1:] == 1
    assert (np.abs(jumps[~hi_next]) <= step).all()           # +-step unless hi
    assert (d[a.hi[0] == 1] == R_MAX).all()                   # hi => max


def test_multilevel_energy_exact_rational():
    """Model M's general form: energy = sum over levels of P_l * time_l, with
    P_l linear between the Fig. 2 ends; checked against exact rationals."""
    plat = oracle.platform(r_min=8, r_max=16, bw_max=16384.0, beta=0.5, p_other=100.0,
                           p_unc_min=0.0, p_unc_max=64.0)
    x = np.array([1000.0, 9000.0, 20000.0, 500.0, 30000.0, 12000.0], np.float32)
    dec = np.array([12, 9, 16, 8, 10, 13], np.int32)
    s, _ = oracle.account(x, dec, plat)
    dt, beta = Fraction(0.2), Fraction(1, 2)
    e = Fraction(0)
    levels = [16] + list(dec[:-1])
    for xt, lvl in zip(x, levels):
        B = Fraction(16384) * lvl / 16
        sig = max(Fraction(0), Fraction(float(xt)) / B - 1)
        q = math.floor(sig * 2 ** 24)
        P = 100 + Fraction(64) * (lvl - 8) / 8
        e += P * (dt + dt * beta * Fraction(q, 2 ** 24))
    assert math.isclose(s["energy"], float(e), rel_tol=1e-14)


# ------------------------------- CPU pins: f3 ------------------------------

def test_closed_loop_equals_open_loop_below_the_min_capacity():
    """If every sample is below B(r_min) nothing is ever capped."""
    x = np.minimum(gen.gen_traces(gen.SEEDS[1], 64, 3000), np.float32(11000.0))
    a = oracle.replay(x, oracle.policy(), want_dec=True)
    b = oracle.replay(x, oracle.policy(variant=1), want_dec=True)
    assert np.array_equal(a.dec, b.dec) and np.array_equal(a.summary, b.summary)


def test_closed_loop_sees_less_and_invariants():
    x = gen.gen_traces(gen.SEEDS[2], 96, 4000)
    a = oracle.replay(x, oracle.policy(), want_dec=True)
    b = oracle.replay(x, oracle.policy(variant=1), want_dec=True)
    d = b.dec[0]
    assert np.isin(d, [R_MIN, R_MAX]).all() and (d[b.hi[0] == 1] == R_MAX).all()
    assert not np.array_equal(a.dec, b.dec)   # the cap changes some decisions
    # delivered throughput is never above demand, so a burst seen by the
    # closed loop is seen by the open loop: its increase events can only drop
    assert (b.summary[0]["slowdown"] >= 0).all()
    with pytest.raises(ValueError):
        oracle.replay(x[:, :2], oracle.policy(variant=1), closed_form=True)


def test_closed_loop_literal_brute_force_recurrence():
    """Exhaustive 3-level traces: the literal Mdfs closed loop against a
    direct recurrence written from the definition (y_t from dec[t-1])."""
    W, H, thi = 3, 4, 0.5
    x = _all_traces([1000.0, 11000.0, 24000.0], 9)
    r = oracle.replay(x, oracle.policy(W=W, H=H, t_hi=thi, tau_inc=200, tau_dec=-500, variant=1), want_dec=True)
    B = {R_MIN: 32000.0 * R_MIN / R_MAX, R_MAX: 32000.0 * R_MAX / R_MAX}
    for n in range(x.shape[1]):
        dec, y, ev = [], [], []
        lvl = R_MAX
        for t in range(x.shape[0]):
            y.append(min(float(x[t, n]), B[lvl]))   # observed under the level in effect
            if t >= W:
                s = sum(ev[max(0, t - H):t])
                hi = s / H >= thi
                d = (y[t] - y[t - W + 1]) / W
                p = 1 if d > 200 else (-1 if d < -500 else 0)
                if hi:
                    lvl = R_MAX
                elif p:
                    lvl = R_MAX if p > 0 else R_MIN
                ev.append(int(p != 0))
            else:
                ev.append(0)
            dec.append(lvl)
        assert r.dec[0, n].tolist() == dec


# ------------------------------- GPU parity --------------------------------

@pytest.mark.gpu
@pytest.mark.parametrize("variant,step", [(0, 0), (1, 0), (2, 1), (2, 3), (3, 2)])
def test_gpu_variants_levels_and_summaries(variant, step):
    torch = pytest.importorskip("torch")
    magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")
    N, T = 190, 2777
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    pols = [magus.make_policy(variant=variant, step=step), magus.make_policy(W=4, t_hi=0.2, variant=variant, step=step),
            magus.make_policy(W=40, H=50, tau_inc=120, tau_dec=-90, t_hi=0.3, variant=variant, step=step)]
    po = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc, tau_dec=p.tau_dec,
                               t_hi=p.t_hi, variant=p.variant, step=p.step) for p in pols])
    plat_o = oracle.platform(burst=12000.0)
    ref = oracle.replay(x, po, plat_o, want_dec=True)
    plat = magus.platform_preset()
    plat.burst_mbs = 12000.0
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    with magus.Context(device=0, platform=plat) as ctx:
        levels, res = ctx.replay_levels(xd, pols)
        torch.cuda.synchronize()
        lv = levels.cpu().numpy().transpose(0, 2, 1)          # [C, N, T]
        assert np.array_equal(lv, ref.dec.astype(np.uint8))
        got = res.summary_numpy()
        for gf, of in [("n_events", "n_events"), ("n_hi_rounds", "n_hi_rounds"), ("n_msr_writes", "n_msr_writes"),
                       ("n_changes", "n_changes"), ("n_min_dec", "n_min_dec"), ("n_min_int", "n_min_int"),
                       ("q_min", "q_min"), ("q_max", "q_max"), ("digest", "digest"), ("time_s", "time"),
                       ("energy_j", "energy"), ("slowdown", "slowdown"), ("viol", "viol"),
                       ("n_burst_base", "n_burst_base"), ("n_burst_magus", "n_burst_magus")]:
            assert np.array_equal(got[gf], ref.summary[of]), gf
        tot = res.totals_numpy()
        for c in range(len(pols)):
            w, _ = oracle.totals(ref.summary[c], ref.base, T, plat_o)
            assert np.array_equal(tot[c], w)
        if variant == 0:   # the paper's rule through magus_replay too (stream kernel)
            r2 = ctx.replay(xd, pols[:2])
            torch.cuda.synchronize()
            assert np.array_equal(r2.summary_numpy(), got[:2])
