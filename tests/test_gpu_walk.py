"""The time-segmented open-loop kernel (kernels_walk.cu, OPT_KERNEL = 4) vs
the CPU oracle, element by element.

It runs NEXT f4 (gradual +-step rule, P@35554) and the paper's jump rule
(Alg. 3 l.18-25) with per-interval level output.  Each segment's effect on
the carried level is a composed clamp-shift map, so the
bar is the same as for the unsegmented kernels: levels, decision words,
counters, q sums and digests bit-exact, model-M time / energy bit-exact
(same fp64 order, no FMA contraction), totals words bit-exact -- for every
segment count, including one segment per 32-step word, segment boundaries
inside the warm-up and inside the Alg. 2 history, ragged tails, NaN samples,
T < W, another ratio range, bursts, and mixed variants in one launch.
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")

from test_gpu_seq import FIELDS, _check, _opol, _platforms  # noqa: E402


def _levels(ctx, x, pols, segments=0, kernel=4, walk1=0):
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    ctx.set_option(magus.OPT_KERNEL, kernel)
    ctx.set_option(magus.OPT_SEGMENTS, segments)
    ctx.set_option(magus.OPT_WALK1, walk1)
    try:
        lv, res = ctx.replay_levels(xd, pols)
        torch.cuda.synchronize()
        assert ctx.stats()["last_kernel"] == kernel
    finally:
        ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_AUTO)
        ctx.set_option(magus.OPT_SEGMENTS, 0)
        ctx.set_option(magus.OPT_WALK1, 0)
    return lv.cpu().numpy().transpose(0, 2, 1), res      # [C, N, T]


MIXED = [  # (variant, step) of each config in ONE launch
    [(2, 1)], [(2, 3)], [(0, 0)], [(2, 14)], [(0, 0), (2, 2), (2, 5)],
]


@pytest.mark.parametrize("walk1", [0, 1])
@pytest.mark.parametrize("mix", range(len(MIXED)))
@pytest.mark.parametrize("segments", [0, 1, 3, 11, 87])
def test_walk_kernel_vs_oracle(mix, segments, walk1):
    N, T = 190, 2777            # 87 segments of 32 steps: every word its own segment
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    pols = []
    for v, s in MIXED[mix]:
        pols.append(magus.make_policy(variant=v, step=s))
        pols.append(magus.make_policy(W=4, H=7, t_hi=0.2, variant=v, step=s))
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, segments, walk1=walk1)
    _check(lv, res, ref, po, T, len(pols))


@pytest.mark.parametrize("walk1", [0, 1])
@pytest.mark.parametrize("segments", [0, 11, 87])
def test_walk_kernel_carry_dependent_segments(segments, walk1):
    """No override (t_hi = 2: s/H >= 2 never holds) and +-1 steps over a
    14-ratio range: a segment's map rarely becomes constant, so the one-pass
    kernel replays long carry-dependent prefixes (often whole segments) after
    the look-back, through chains of non-constant predecessor maps."""
    N, T = 160, 2777
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    pols = [magus.make_policy(variant=2, step=1, t_hi=2.0), magus.make_policy(W=4, H=7, t_hi=2.0, variant=2, step=2)]
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, segments, walk1=walk1)
    _check(lv, res, ref, po, T, len(pols))


@pytest.mark.parametrize("walk1", [0, 1])
@pytest.mark.parametrize("N,T,segments", [(33, 17, 0), (1, 1, 0), (1, 10000, 0), (1, 10000, 300), (129, 64, 2)])
def test_walk_kernel_shapes(N, T, segments, walk1):
    x = gen.gen_traces(gen.SEEDS[2], N, T)
    pols = [magus.make_policy(variant=2, step=1), magus.make_policy(variant=0)]
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, segments, walk1=walk1)
    _check(lv, res, ref, po, T, len(pols))


@pytest.mark.parametrize("variant,step,W,H", [(2, 1, 2, 1), (2, 4, 200, 50), (0, 0, 70, 64), (2, 2, 33, 64)])
@pytest.mark.parametrize("segments", [0, 9])
def test_walk_kernel_window_history_extremes(variant, step, W, H, segments):
    """Segment boundaries fall inside the warm-up (W = 200 > a 96-step
    segment) and inside the 64-round Alg. 2 history."""
    N, T = 70, 3001
    x = gen.gen_traces(gen.SEEDS[2], N, T)
    pols = [magus.make_policy(W=W, H=H, tau_inc=40.0, tau_dec=-60.0, t_hi=0.25, variant=variant, step=step)]
    po, pm = _platforms("max1550", 9000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, segments)
    _check(lv, res, ref, po, T, 1)


def test_walk_kernel_nan_and_short_traces():
    """NaN samples (reading R9) and T < W (no MDFS round at all)."""
    N, T = 64, 700
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    rng = np.random.default_rng(5)
    x[rng.integers(0, T, 300), rng.integers(0, N, 300)] = np.nan
    pols = [magus.make_policy(variant=2, step=2), magus.make_policy(W=800, variant=2, step=1),
            magus.make_policy(variant=0)]
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        for segs in (0, 5):
            lv, res = _levels(ctx, x, pols, segs)
            _check(lv, res, ref, po, T, len(pols))


def test_walk_kernel_adversarial_oscillation():
    """Config-5-shaped adversarial traces (exact Alg. 1 ties, square waves,
    F5 burst widths) drive the frequent-transition override constantly."""
    N, T = 96, 4000
    x = gen.gen_traces(gen.SEEDS[5], N, T, kind=gen.KIND_ADVERSARIAL)
    pols = [magus.make_policy(variant=2, step=1), magus.make_policy(variant=2, step=3, t_hi=0.6)]
    po, pm = _platforms("a100", 0.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, 13)
    _check(lv, res, ref, po, T, len(pols))


def test_walk_kernel_auto_choice_and_decision_words():
    """magus_replay with gradual (open-loop) configs runs the walk kernel by
    default and writes the oracle's decision words (bit = dec is r_min)."""
    N, T = 100, 4099
    x = gen.gen_traces(gen.SEEDS[4], N, T)
    pols = [magus.make_policy(variant=2, step=1), magus.make_policy(W=6, variant=2, step=14)]
    ref = oracle.replay(x, _opol(pols), want_dec=True)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    with magus.Context(device=0) as ctx:
        r = ctx.replay(xd, pols, want_decisions=True)
        torch.cuda.synchronize()
        assert ctx.stats()["last_kernel"] == 4
        assert ctx.stats()["last_segments"] > 1
    words = oracle.decision_words(ref.dec, 8)
    assert np.array_equal(r.decisions_numpy().transpose(0, 2, 1), words)
    got = r.summary_numpy()
    for gf, of in FIELDS[:13]:
        assert np.array_equal(got[gf], ref.summary[of]), gf


def test_walk_kernel_rejects_closed_loop():
    """The closed loop (f3) has no exact time segmentation: forcing the walk
    kernel on it fails loudly; auto runs the sequential kernel."""
    N, T = 40, 500
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    pols = [magus.make_policy(variant=2, step=1), magus.make_policy(variant=1)]
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    with magus.Context(device=0) as ctx:
        ctx.set_option(magus.OPT_KERNEL, 4)
        with pytest.raises(Exception):
            ctx.replay_levels(xd, pols)
        ctx.set_option(magus.OPT_KERNEL, 0)
        ctx.replay_levels(xd, pols)
        torch.cuda.synchronize()
        assert ctx.stats()["last_kernel"] == 3


@pytest.mark.parametrize("W", [4, 6, 10, 16])
@pytest.mark.parametrize("segments", [1, 11, 87])
def test_walk_kernel_compile_time_window(W, segments):
    """Every config of the launch shares W in {4, 6, 10, 16}: pass 1 takes
    the Alg. 1 lags from its register window (segment starts reload it, the
    warm-up and the ragged tail take the row-load path)."""
    N, T = 150, 2777
    x = gen.gen_traces(gen.SEEDS[4], N, T)
    pols = [magus.make_policy(W=W, variant=2, step=2), magus.make_policy(W=W, H=7, t_hi=0.3, variant=2, step=1),
            magus.make_policy(W=W, variant=0)]
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, segments)
    _check(lv, res, ref, po, T, len(pols))
