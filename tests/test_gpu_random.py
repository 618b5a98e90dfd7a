"""Randomised parity: seeded random shapes, policies, kernels and options in
ONE context, every result bit for bit against the CPU oracle.

Each case draws N, T, a padded row stride, a trace kind, 1-6 policies (W,
H, L, tau_inc, tau_dec, t_hi anywhere in their valid ranges, biased to the
paper's values), a kernel (auto, stream, the per-sample reference with the
printed divisions, or the walk kernels through replay_levels), a segment
count, the bundle size and the 128/512-trace CTA option.  Cases share the
context on purpose: the kernel paths reuse its scratch one after another
(the stale-status hazard of ADVICE round 1 lived exactly there)."""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

FIELDS = ("n_events", "n_hi_rounds", "n_msr_writes", "n_changes", "n_min_dec", "n_min_int", "q_min", "q_max",
          "digest", "time_s", "energy_j")
ORACLE_NAME = {"time_s": "time", "energy_j": "energy"}


def _random_policy(rng):
    W = int(rng.choice([2, 3, 4, 6, 10, 10, 10, 16, 17, 33]))
    H = int(rng.choice([1, 5, 10, 10, 10, 13, 32]))
    L = float(W) if rng.random() < 0.7 else float(rng.uniform(0.5, 40.0))
    tau_inc = float(rng.choice([0.0, 100.0, 200.0, 300.0, rng.uniform(0, 3000)]))
    tau_dec = float(rng.choice([-250.0, -500.0, -1000.0, -rng.uniform(0, 6000)]))
    t_hi = float(rng.choice([0.1, 0.2, 0.3, 0.4, 0.5, 1.0, 1.2, rng.uniform(0.05, 1.0)]))
    return dict(W=W, H=H, L=L, tau_inc=tau_inc, tau_dec=tau_dec, t_hi=t_hi)


@pytest.fixture(scope="module")
def ctx():
    import paper_conf_sc_zhengspl25_b200 as magus
    with magus.Context(device=0) as c:
        yield c


@pytest.mark.parametrize("case", range(64))
def test_random_case_bit_exact(ctx, case):
    import torch

    import paper_conf_sc_zhengspl25_b200 as magus
    rng = np.random.default_rng(0x5EED0000 + case)
    N = int(rng.choice([1, 7, 31, 128, 129, 511, 512, 513, int(rng.integers(1, 900))]))
    T = int(rng.choice([1, 9, 33, 64, 1000, int(rng.integers(1, 4000))]))
    ld = (N + 3) // 4 * 4 + 4 * int(rng.integers(0, 3))
    kind = gen.KIND_ADVERSARIAL if rng.random() < 0.3 else gen.KIND_MIX
    x = gen.gen_traces(gen.SEEDS[2] + case, N, T, kind=kind, ld=ld)
    rows = [_random_policy(rng) for _ in range(int(rng.integers(1, 7)))]
    if rng.random() < 0.4:  # a bundle: configs that differ only in t_hi
        base = rows[0]
        rows = [dict(base, t_hi=t) for t in (0.2, 0.3, 0.4, 0.5)] + rows[1:]
    pols = [magus.make_policy(W=r["W"], H=r["H"], L=r["L"], tau_inc=r["tau_inc"], tau_dec=r["tau_dec"],
                              t_hi=r["t_hi"]) for r in rows]
    ref = oracle.replay(x, oracle.policies(rows), n_traces=N, want_dec=True)
    xd = torch.from_numpy(x).cuda()
    kernel = int(rng.choice([magus.KERNEL_AUTO, magus.KERNEL_STREAM, magus.KERNEL_STREAM, magus.KERNEL_REFERENCE,
                             magus.KERNEL_WALK]))
    stream_ok = all(2 <= r["W"] <= 33 and 1 <= r["H"] <= 32 for r in rows)
    if kernel == magus.KERNEL_STREAM and not stream_ok:
        kernel = magus.KERNEL_AUTO
    ctx.set_option(magus.OPT_KERNEL, kernel)
    ctx.set_option(magus.OPT_SEGMENTS, int(rng.choice([0, 0, 1, 2, 5, int(rng.integers(1, 40))])))
    ctx.set_option(magus.OPT_BUNDLE, int(rng.choice([0, 1, 2, 4])))
    ctx.set_option(magus.OPT_NARROW, int(rng.integers(0, 2)))
    try:
        if kernel == magus.KERNEL_WALK:
            lv, r = ctx.replay_levels(xd, pols, n_traces=N)
            torch.cuda.synchronize()
            assert np.array_equal(lv.cpu().numpy().transpose(0, 2, 1), ref.dec.astype(np.uint8)), "levels"
        else:
            r = ctx.replay(xd, pols, n_traces=N, want_decisions=True)
            torch.cuda.synchronize()
            words = oracle.decision_words(ref.dec, 8)
            assert np.array_equal(r.decisions_numpy().transpose(0, 2, 1), words), "decisions"
        got = r.summary_numpy()
        for f in FIELDS:
            assert np.array_equal(got[f], ref.summary[ORACLE_NAME.get(f, f)]), (f, kernel)
        tot = r.totals_numpy()
        for c in range(len(rows)):
            assert np.array_equal(tot[c], oracle.totals(ref.summary[c], ref.base, T)[0]), ("totals", c)
    finally:
        for opt in (magus.OPT_KERNEL, magus.OPT_SEGMENTS, magus.OPT_BUNDLE, magus.OPT_NARROW):
            ctx.set_option(opt, 0)
