"""The speculatively time-segmented closed loop (kernels_spec.cu,
OPT_KERNEL = 5) vs the CPU oracle, element by element.

NEXT f3 with the paper's jump rule: Alg. 1 observes the delivered
throughput min(x_t, B(l_t)) (P@37360 / P@38709).  Each segment replays
OPT_SPEC_WARM rounds before it from a guessed state; a segment whose
guessed state differs from the true one is replayed again from the true
state.  Results must be bit-identical whatever the warm-up: tiny warm-ups
(every speculation wrong), long ones, segment boundaries inside the
warm-up, many segments, adversarial traces, NaN samples, W / H extremes,
another ratio range and bursts.
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


def _levels(ctx, x, pols, segments=0, warm=0):
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_SPEC)
    ctx.set_option(magus.OPT_SEGMENTS, segments)
    ctx.set_option(magus.OPT_SPEC_WARM, warm)
    try:
        lv, res = ctx.replay_levels(xd, pols)
        torch.cuda.synchronize()
        assert ctx.stats()["last_kernel"] == magus.KERNEL_SPEC
    finally:
        ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_AUTO)
        ctx.set_option(magus.OPT_SEGMENTS, 0)
        ctx.set_option(magus.OPT_SPEC_WARM, 0)
    return lv.cpu().numpy().transpose(0, 2, 1), res


@pytest.mark.parametrize("segments,warm", [(0, 0), (1, 0), (7, 1), (7, 40), (87, 3), (87, 5000), (20, 64)])
@pytest.mark.parametrize("kind", [magus.GEN_MIX, magus.GEN_ADVERSARIAL])
def test_spec_kernel_vs_oracle(segments, warm, kind):
    N, T = 190, 2777
    x = gen.gen_traces(gen.SEEDS[1], N, T, kind=kind)
    pols = [magus.make_policy(variant=1), magus.make_policy(W=4, H=7, t_hi=0.2, variant=1),
            magus.make_policy(tau_inc=100.0, tau_dec=-250.0, t_hi=0.5, variant=1)]
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        lv, res = _levels(ctx, x, pols, segments, warm)
    _check(lv, res, ref, po, T, len(pols))


@pytest.mark.parametrize("W,H", [(2, 1), (65, 64), (33, 64), (10, 33)])
def test_spec_kernel_window_history_extremes(W, H):
    N, T = 70, 3001
    x = gen.gen_traces(gen.SEEDS[2], N, T)
    pols = [magus.make_policy(W=W, H=H, tau_inc=40.0, tau_dec=-60.0, t_hi=0.25, variant=1)]
    po, pm = _platforms("max1550", 9000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        for segs, warm in ((9, 0), (30, 2)):
            lv, res = _levels(ctx, x, pols, segs, warm)
            _check(lv, res, ref, po, T, 1)


def test_spec_kernel_nan_and_short_traces():
    N, T = 64, 700
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    rng = np.random.default_rng(5)
    x[rng.integers(0, T, 300), rng.integers(0, N, 300)] = np.nan
    pols = [magus.make_policy(variant=1), magus.make_policy(W=65, variant=1)]
    po, pm = _platforms("a100", 12000.0)
    ref = oracle.replay(x, _opol(pols), po, want_dec=True)
    with magus.Context(device=0, platform=pm) as ctx:
        for segs, warm in ((0, 0), (5, 1)):
            lv, res = _levels(ctx, x, pols, segs, warm)
            _check(lv, res, ref, po, T, len(pols))
        lv, res = _levels(ctx, x[:20], pols, 0, 0)          # T < W for the second config
    ref = oracle.replay(np.ascontiguousarray(x[:20]), _opol(pols), po, want_dec=True)
    _check(lv, res, ref, po, 20, len(pols))


def test_spec_kernel_decision_words_through_replay():
    """magus_replay on the speculative kernel (time-segmented) writes the
    oracle's decision words and summaries."""
    N, T = 100, 20000
    x = gen.gen_traces(gen.SEEDS[4], N, T)
    pols = [magus.make_policy(variant=1), magus.make_policy(W=6, variant=1)]
    ref = oracle.replay(x, _opol(pols), want_dec=True)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    with magus.Context(device=0) as ctx:
        ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_SPEC)
        r = ctx.replay(xd, pols, want_decisions=True)
        torch.cuda.synchronize()
        assert ctx.stats()["last_kernel"] == magus.KERNEL_SPEC
        assert ctx.stats()["last_segments"] > 1
    words = oracle.decision_words(ref.dec, 8)
    assert np.array_equal(r.decisions_numpy().transpose(0, 2, 1), words)
    got = r.summary_numpy()
    for gf, of in FIELDS[:13]:
        assert np.array_equal(got[gf], ref.summary[of]), gf
