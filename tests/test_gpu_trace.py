"""MAGUS_OPT_TRACE (diagnostics): the per-CTA timeline is complete and
ordered, and tracing leaves every result bit-identical."""
from __future__ import annotations

import numpy as np
import pytest

import gen

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("narrow", [0, 1])
def test_trace_timeline_and_results_unchanged(narrow):
    import torch

    import paper_conf_sc_zhengspl25_b200 as m
    N, T = 1000, 20_000
    x = torch.from_numpy(gen.gen_traces(gen.SEEDS[2], N, T)).cuda()
    pol = [m.policy_preset(m.POLICY_PAPER_DEFAULT)]
    with m.Context(device=0) as ctx:
        ctx.set_option(m.OPT_KERNEL, m.KERNEL_STREAM)
        ctx.set_option(m.OPT_SEGMENTS, 5)
        ctx.set_option(m.OPT_NARROW, narrow)
        a = ctx.replay(x, pol, want_decisions=True)
        ctx.set_option(m.OPT_TRACE, 1)
        b = ctx.replay(x, pol, want_decisions=True)
        tr = ctx.trace()
        ctx.set_option(m.OPT_TRACE, 0)
        c = ctx.replay(x, pol, want_decisions=True)   # the timeline address is cleared again
        torch.cuda.synchronize()
        grid = ctx.stats()["last_grid"]
    for r in (b, c):
        assert np.array_equal(a.summary_numpy(), r.summary_numpy())
        assert np.array_equal(a.decisions_numpy(), r.decisions_numpy())
        assert np.array_equal(a.totals_numpy(), r.totals_numpy())
    tr_per_cta = 128 if narrow else 512       # traces per CTA
    ngroups = (N + tr_per_cta - 1) // tr_per_cta
    assert len(tr) == grid == ngroups * 5
    t = tr[:, :4].astype(np.int64)
    assert (t > 0).all() and (np.diff(t, axis=1) >= 0).all()
    assert sorted(zip(tr[:, 5].tolist(), tr[:, 6].tolist())) == [(s, g) for s in range(5) for g in range(ngroups)]
    assert tr[:, 7].sum() == ngroups          # one finaliser per trace group
