"""Edge cases of the boundary on the GPU: validation before any launch
(outputs untouched), the maximum interval count T = 2^24, degenerate traces,
and the auto kernel choice for the paper's rule outside the stream kernel's
template range (W > 33 or H > 32 -> the walk kernels)."""
from __future__ import annotations

import math

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")

from test_gpu_parity import FIELDS, to_oracle_policies  # noqa: E402


@pytest.fixture(scope="module")
def ctx():
    with magus.Context(device=0) as c:
        yield c


BAD_POLICIES = [dict(W=1), dict(H=0), dict(H=65), dict(L=0.0), dict(L=-1.0), dict(L=math.inf),
                dict(tau_inc=math.nan), dict(tau_dec=math.inf), dict(t_hi=0.0), dict(t_hi=math.nan)]


@pytest.mark.parametrize("bad", BAD_POLICIES)
def test_invalid_policy_rejected_before_launch(ctx, bad):
    x = ctx.gen_traces(gen.SEEDS[1], 64, 500)
    out = ctx.replay(x, [magus.make_policy()], want_decisions=True)
    torch.cuda.synchronize()
    before = [t.clone() for t in (out.summary, out.base, out.decisions, out.totals)]
    with pytest.raises(magus.MagusError) as e:
        ctx.replay(x, [magus.make_policy(), magus.make_policy(**bad)], out=None)
    assert e.value.status == magus.ERR_INVALID_ARG
    torch.cuda.synchronize()
    for a, b in zip(before, (out.summary, out.base, out.decisions, out.totals)):
        assert torch.equal(a, b)


def test_invalid_shapes_rejected(ctx):
    x = ctx.gen_traces(gen.SEEDS[1], 64, 100)
    pol = [magus.make_policy()]
    with pytest.raises(magus.MagusError):
        ctx.replay(x, pol, n_traces=0)
    with pytest.raises(magus.MagusError):
        ctx.replay(x[:0], pol)
    with pytest.raises(magus.MagusError):
        ctx.replay(x, pol, n_traces=65)          # ld < n_traces
    big = torch.empty(((1 << 24) + 1, 4), dtype=torch.float32, device="cuda:0")
    with pytest.raises(magus.MagusError):          # T > 2^24 (model M's exact integer sums)
        ctx.replay(big, pol)
    del big


def test_maximum_interval_count(ctx):
    """T = 2^24 intervals (the limit that keeps every q sum below 2^63) on
    the stream kernel; the oracle checks two traces in full."""
    N, T = 32, 1 << 24
    xd = ctx.gen_traces(gen.SEEDS[3], N, T)
    pols = [magus.policy_preset(magus.POLICY_PAPER_DEFAULT)]
    r = ctx.replay(xd, pols, want_decisions=False)
    torch.cuda.synchronize()
    assert ctx.stats()["last_kernel"] == magus.KERNEL_STREAM
    got = r.summary_numpy()
    for n in (0, 31):
        xs = xd[:, n:n + 1].cpu().numpy()
        ref = oracle.replay(np.ascontiguousarray(xs), to_oracle_policies(pols))
        for gf, of in FIELDS:
            assert got[gf][0, n] == ref.summary[of][0, 0], (gf, n)
    del xd


def test_degenerate_traces(ctx):
    """Constant, all-zero, all-NaN and huge-valued traces (F1: no events,
    energy = base energy bitwise) next to ordinary ones."""
    T = 3000
    x = gen.gen_traces(gen.SEEDS[2], 8, T)
    x[:, 0] = 5000.0
    x[:, 1] = 0.0
    x[:, 2] = np.nan
    x[:, 3] = 3.0e38
    x[:, 4] = -7.0
    pols = [magus.make_policy(), magus.make_policy(W=4, H=3, t_hi=0.34)]
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    for kernel in (magus.KERNEL_STREAM, magus.KERNEL_REFERENCE, magus.KERNEL_WALK):
        ctx.set_option(magus.OPT_KERNEL, kernel)
        try:
            r = ctx.replay(xd, pols, want_decisions=True)
            torch.cuda.synchronize()
        finally:
            ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_AUTO)
        got = r.summary_numpy()
        for gf, of in FIELDS:
            assert np.array_equal(got[gf], ref.summary[of]), (kernel, gf)
        base = r.base_numpy()
        for n in (0, 1, 4):                       # constant traces: F1
            assert got["n_events"][0, n] == 0 and got["energy_j"][0, n] == base["energy_j"][n]


@pytest.mark.parametrize("W,H", [(40, 10), (10, 48), (64, 64)])
def test_paper_rule_outside_stream_templates_runs_on_walk(ctx, W, H):
    N, T = 300, 5000
    x = gen.gen_traces(gen.SEEDS[4], N, T)
    pols = [magus.make_policy(W=W, H=H, tau_inc=100.0, tau_dec=-250.0, t_hi=0.2)]
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    r = ctx.replay(xd, pols, want_decisions=True)
    torch.cuda.synchronize()
    assert ctx.stats()["last_kernel"] == magus.KERNEL_WALK
    got = r.summary_numpy()
    for gf, of in FIELDS:
        assert np.array_equal(got[gf], ref.summary[of]), gf
    words = oracle.decision_words(ref.dec, 8)
    assert np.array_equal(r.decisions_numpy().transpose(0, 2, 1), words)
