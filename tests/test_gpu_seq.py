"""The sequential-variant kernel (kernels_seq.cu, OPT_KERNEL = 3) vs the CPU
oracle and vs the literal per-sample kernel, element by element.

It runs NEXT f3 (closed loop: Alg. 1 observes min(x_t, B(l_t)), P@37360 /
P@38709), f4 (gradual +-step rule, P@35554) and their combination, plus the
paper's rule whenever per-interval levels are requested.  Bar: levels,
decision words, counters, q sums and digests bit-exact; model-M time/energy
bit-exact (same fp64 order, no FMA contraction); totals words bit-exact.
Shapes cover several 16-step cp.async chunks and 32-step decision words with
ragged tails, traces not a multiple of the warp, T < W, NaN samples, a
platform with another ratio range, and configs of different variants in one
launch (each thread follows its own config).
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")

FIELDS = [("n_events", "n_events"), ("n_hi_rounds", "n_hi_rounds"), ("n_msr_writes", "n_msr_writes"),
          ("n_changes", "n_changes"), ("n_min_dec", "n_min_dec"), ("n_min_int", "n_min_int"),
          ("q_min", "q_min"), ("q_max", "q_max"), ("digest", "digest"), ("time_s", "time"),
          ("energy_j", "energy"), ("slowdown", "slowdown"), ("viol", "viol"),
          ("n_burst_base", "n_burst_base"), ("n_burst_magus", "n_burst_magus")]


def _opol(pols):
    return oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc, tau_dec=p.tau_dec,
                                 t_hi=p.t_hi, variant=p.variant, step=p.step) for p in pols])


def _platforms(kind, burst):
    if kind == "a100":
        po = oracle.platform(burst=burst)
        pm = magus.platform_preset(magus.PLATFORM_INTEL_A100)
    else:   # another ratio range (Max1550's 8-25, P@29831) and a tighter capacity
        po = oracle.platform(r_min=8, r_max=25, bw_max=20000.0, beta=0.5, burst=burst)
        pm = magus.platform_preset(magus.PLATFORM_INTEL_A100)
        pm.ratio_min, pm.ratio_max, pm.bw_max_mbs, pm.beta = 8, 25, 20000.0, 0.5
    pm.burst_mbs = burst
    return po, pm


def _levels(ctx, x, pols, kernel):
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    ctx.set_option(magus.OPT_KERNEL, kernel)
    try:
        lv, res = ctx.replay_levels(xd, pols)
        torch.cuda.synchronize()
    finally:
        ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_AUTO)
    return lv.cpu().numpy().transpose(0, 2, 1), res      # [C, N, T]


def _check(lv, res, ref, po, T, C):
    assert np.array_equal(lv, ref.dec.astype(np.uint8)), "levels differ"
    got = res.summary_numpy()
    for gf, of in FIELDS:
        a, b = got[gf], ref.summary[of]
        bad = np.argwhere(a != b)
        assert bad.size == 0, f"{gf}: first mismatch at {bad[0]} gpu={a[tuple(bad[0])]} oracle={b[tuple(bad[0])]}"
    tot = res.totals_numpy()
    for c in range(C):
        w, _ = oracle.totals(ref.summary[c], ref.base, T, po)
        assert np.array_equal(tot[c], w), f"totals of config {c}"


MIXED = [  # (variant, step) of each config in ONE launch
    [(1, 0)], [(2, 1)], [(2, 3)], [(3, 2)], [(0, 0)],
    [(1, 0), (0, 0), (2, 2), (3, 1)],
]


@pytest.mark.parametrize("kernel", [3, 1])
@pytest.mark.parametrize("mix", range(len(MIXED)))
@pytest.mark.parametrize("N,T", [(190, 2777), (33, 17), (1, 1)])
def test_seq_kernel_vs_oracle(kernel, mix, N, T):
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    pols = []
    for v, s in MIXED[mix]:
        pols.append(magus.make_policy(variant=v, step=s))
        pols.append(magus.make_policy(W=4, H=7, t_hi=0.2, variant=v, step=s))
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, kernel)
    _check(lv, res, ref, po, T, len(pols))


@pytest.mark.parametrize("variant,step,W,H", [(1, 0, 64, 64), (1, 0, 2, 1), (3, 1, 100, 33), (2, 4, 200, 50),
                                              (0, 0, 70, 40)])
def test_seq_kernel_window_history_extremes(variant, step, W, H):
    N, T = 70, 3001
    x = gen.gen_traces(gen.SEEDS[2], N, T)
    pols = [magus.make_policy(W=W, H=H, tau_inc=40.0, tau_dec=-60.0, t_hi=0.25, variant=variant, step=step)]
    po, pm = _platforms("max1550", 9000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, 3)
    _check(lv, res, ref, po, T, 1)


def test_seq_kernel_nan_and_short_traces():
    """NaN samples (reading R9: both Alg. 1 tests false, never a burst) and
    T < W (no MDFS round at all)."""
    N, T = 64, 700
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    rng = np.random.default_rng(5)
    x[rng.integers(0, T, 300), rng.integers(0, N, 300)] = np.nan
    pols = [magus.make_policy(variant=1), magus.make_policy(variant=3, step=2), magus.make_policy(W=800, variant=2, step=1)]
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, 3)
    _check(lv, res, ref, po, T, len(pols))


def test_seq_kernel_decision_words_through_replay():
    """magus_replay with closed-loop gradual configs runs the sequential
    kernel (auto choice) and writes the same decision words as the oracle."""
    N, T = 100, 4099
    x = gen.gen_traces(gen.SEEDS[4], N, T)
    pols = [magus.make_policy(variant=1), magus.make_policy(W=6, variant=3, step=14)]
    ref = oracle.replay(x, _opol(pols), want_dec=True)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    with magus.Context(device=0) as ctx:
        r = ctx.replay(xd, pols, want_decisions=True)
        torch.cuda.synchronize()
        assert ctx.stats()["last_kernel"] == 3
    words = oracle.decision_words(ref.dec, 8)
    assert np.array_equal(r.decisions_numpy().transpose(0, 2, 1), words)
    got = r.summary_numpy()
    for gf, of in FIELDS[:13]:
        assert np.array_equal(got[gf], ref.summary[of]), gf


def test_seq_kernel_rejects_unsupported_closed_window():
    """A closed-loop jump config with W > 65 runs on neither the sequential
    nor the speculative kernel: forcing it fails loudly, auto falls back to
    the per-sample kernel."""
    N, T = 40, 500
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    pols = [magus.make_policy(W=66, variant=1)]
    ref = oracle.replay(x, _opol(pols), want_dec=True)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    with magus.Context(device=0) as ctx:
        for k in (3, 5):
            ctx.set_option(magus.OPT_KERNEL, k)
            with pytest.raises(Exception):
                ctx.replay_levels(xd, pols)
        ctx.set_option(magus.OPT_KERNEL, 0)
        lv, res = ctx.replay_levels(xd, pols)
        torch.cuda.synchronize()
        assert ctx.stats()["last_kernel"] == 1
    assert np.array_equal(lv.cpu().numpy().transpose(0, 2, 1), ref.dec.astype(np.uint8))
