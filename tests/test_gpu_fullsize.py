"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times, on sampled outputs the oracle computes one by one (each trace's
results depend only on its own samples; the totals are checked through
their exact integer words on the sampled subset by partition invariance).

  config 3  4,096 x 100,000 x SWEEP256 (4 W-group launches, bundles of 4)
  config 4  one GPU's shard at 8 GPUs: 8,192 x 1,000,000 x FLEET64, one shot
  config 5  16,384 adversarial x 1,000,000 x paper_default
  config 2  f4 gradual through the walk kernels (143 segments), and through
            the one-pass walk kernel (MAGUS_OPT_WALK1)
  config 2  f3 closed loop through the sequential kernel (transition codes)

Config 2 (paper's rule) is in test_gpu_parity.py; config 4 through the
time-chunked path is sampled by bench.py (parity_sample_ok) and by
test_gpu_resume.py at smaller T.
"""
from __future__ import annotations

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


def _sample(N, k, seed):
    rng = np.random.default_rng(seed)
    return np.unique(np.r_[0, 127, 128, N - 1, rng.integers(0, N, k)])


def _check_sample(ctx, xd, pols, sample, r):
    got = r.summary_numpy()
    xs = xd[:, torch.as_tensor(sample, device=xd.device)].cpu().numpy()
    ref = oracle.replay(np.ascontiguousarray(xs), to_oracle_policies(pols))
    assert ref.summary["n_events"].sum() > 0 and ref.summary["n_changes"].sum() > 0  # non-trivial data
    for i, n in enumerate(sample):
        for gf, of in FIELDS:
            a, b = got[gf][:, n], ref.summary[of][:, i]
            bad = np.flatnonzero(a != b)
            assert bad.size == 0, f"{gf}: trace {n}, config {bad[0]}: gpu={a[bad[0]]} oracle={b[bad[0]]}"


def test_full_config3_sweep256_sampled(ctx):
    N, T = 4096, 100_000
    xd = ctx.gen_traces(gen.SEEDS[3], N, T)
    pols = magus.grid_sweep256()
    r = ctx.replay(xd, pols, want_decisions=False)
    torch.cuda.synchronize()
    assert ctx.stats()["last_kernel"] == magus.KERNEL_STREAM
    _check_sample(ctx, xd, pols, _sample(N, 2, 3), r)
    del xd


def test_full_config4_shard_fleet64_sampled(ctx):
    N, T = 8192, 1_000_000            # 65,536 / 8 GPUs; 32.8 GB of traces
    xd = ctx.gen_traces(gen.SEEDS[4], N, T, id0=3 * N)   # rank 3's block of global ids
    pols = magus.grid_fleet64()
    r = ctx.replay(xd, pols, want_decisions=False)
    torch.cuda.synchronize()
    _check_sample(ctx, xd, pols, np.array([0, 4097, N - 1]), r)
    del xd, r
    torch.cuda.empty_cache()


def test_full_config5_adversarial_sampled(ctx):
    N, T = 16384, 1_000_000           # 65.5 GB of traces
    xd = ctx.gen_traces(gen.SEEDS[5], N, T, kind=magus.GEN_ADVERSARIAL)
    pols = [magus.policy_preset(magus.POLICY_PAPER_DEFAULT)]
    r = ctx.replay(xd, pols, want_decisions=False)
    torch.cuda.synchronize()
    _check_sample(ctx, xd, pols, _sample(N, 10, 5), r)
    del xd, r
    torch.cuda.empty_cache()


def test_full_config2_gradual_walk_sampled(ctx):
    N, T = 4096, 100_000
    xd = ctx.gen_traces(gen.SEEDS[2], N, T)
    pols = [magus.make_policy(variant=2, step=2), magus.make_policy(variant=2, step=1)]
    r = ctx.replay(xd, pols, want_decisions=True)
    torch.cuda.synchronize()
    assert ctx.stats()["last_kernel"] == magus.KERNEL_WALK
    assert ctx.stats()["last_segments"] > 50
    sample = _sample(N, 12, 2)
    _check_sample(ctx, xd, pols, sample, r)
    xs = xd[:, torch.as_tensor(sample, device=xd.device)].cpu().numpy()
    ref = oracle.replay(np.ascontiguousarray(xs), to_oracle_policies(pols), want_dec=True)
    dec = r.decisions_numpy()
    for i, n in enumerate(sample):
        for c in range(len(pols)):
            assert np.array_equal(dec[c, :, n], oracle.decision_words(ref.dec[c, i], 8)), (n, c)


def test_full_config2_gradual_sweep_in_config_batches(ctx):
    """Eight gradual configs at 4096 x 100,000: their pass-1 masks (1.2 GB)
    exceed the walk kernels' 1 GB budget, so the configs run in two batches
    of map + replay launches; sampled traces vs the oracle."""
    N, T = 4096, 100_000
    xd = ctx.gen_traces(gen.SEEDS[2], N, T)
    pols = [magus.make_policy(variant=2, step=st, tau_inc=ti, t_hi=th)
            for st in (1, 3) for ti in (200.0, 300.0) for th in (0.3, 0.5)]
    r = ctx.replay(xd, pols, want_decisions=False)
    torch.cuda.synchronize()
    assert ctx.stats()["last_kernel"] == magus.KERNEL_WALK
    _check_sample(ctx, xd, pols, np.array([0, 1, 2047, N - 1]), r)


def test_full_config2_gradual_one_pass_walk_sampled(ctx):
    """The one-pass walk kernel (decoupled look-back, carry-dependent prefixes
    replayed) at the bench's size and segmentation."""
    N, T = 4096, 100_000
    xd = ctx.gen_traces(gen.SEEDS[2], N, T)
    pols = [magus.make_policy(variant=2, step=2)]
    ctx.set_option(magus.OPT_WALK1, 1)
    try:
        r = ctx.replay(xd, pols, want_decisions=True)
        torch.cuda.synchronize()
    finally:
        ctx.set_option(magus.OPT_WALK1, 0)
    assert ctx.stats()["last_kernel"] == magus.KERNEL_WALK
    sample = _sample(N, 12, 5)
    _check_sample(ctx, xd, pols, sample, r)
    xs = xd[:, torch.as_tensor(sample, device=xd.device)].cpu().numpy()
    ref = oracle.replay(np.ascontiguousarray(xs), to_oracle_policies(pols), want_dec=True)
    dec = r.decisions_numpy()
    for i, n in enumerate(sample):
        assert np.array_equal(dec[0, :, n], oracle.decision_words(ref.dec[0, i], 8)), n


def test_full_config2_closed_loop_sampled(ctx):
    """f3 at the bench's size: seq_kernel, one chain per trace over 100,000
    rounds, decisions and every summary field bit-exact on a sample."""
    N, T = 4096, 100_000
    xd = ctx.gen_traces(gen.SEEDS[3], N, T)
    pols = [magus.make_policy(variant=1)]
    r = ctx.replay(xd, pols, want_decisions=True)
    torch.cuda.synchronize()
    assert ctx.stats()["last_kernel"] == magus.KERNEL_SEQUENTIAL
    sample = _sample(N, 12, 6)
    _check_sample(ctx, xd, pols, sample, r)
    xs = xd[:, torch.as_tensor(sample, device=xd.device)].cpu().numpy()
    ref = oracle.replay(np.ascontiguousarray(xs), to_oracle_policies(pols), want_dec=True)
    dec = r.decisions_numpy()
    for i, n in enumerate(sample):
        assert np.array_equal(dec[0, :, n], oracle.decision_words(ref.dec[0, i], 8)), n
