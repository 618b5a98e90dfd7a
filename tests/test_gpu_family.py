"""The configuration-family kernel (kernels_family.cu) vs the CPU oracle, bit
for bit (needs a B200).

A (W, H) group of <= 16 bundles of 4 configs (t_hi variants) with <= 8
distinct inverted tau_inc / tau_dec thresholds -- a sweep grid (P@43882,
Sec. 6.4) -- runs in one CTA per (32 traces, segment): the Alg. 1 compares
once per sample for every config, the stretch sums from per-word prefix sums.
Cases: SWEEP256 / FLEET64 (the paper-shaped grids), random families (any W in
[2, 33], H = 10 and runtime H, 1-16 bundles, 1-8 thresholds, padded
bundles), adversarial traces (NaN, 3e38, negative, above the capacity at
r_max: the q_max prefix path), ragged N and T, 1-40 segments, decisions,
time-chunked replay; and family on == family off (the per-bundle stream
kernel) on every output word.
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle
from test_gpu_parity import R_MIN, assert_parity, to_oracle_policies

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")


@pytest.fixture(scope="module")
def ctx():
    c = magus.Context(device=0)
    yield c
    c.close()


def _run(ctx, x, pols, family=True, segments=0, decisions=True):
    T, N = x.shape
    ld = (N + 3) // 4 * 4
    buf = torch.zeros((T, ld), dtype=torch.float32, device="cuda:0")
    buf[:, :N] = torch.from_numpy(x).cuda()
    ctx.set_option(magus.OPT_FAMILY, 0 if family else 1)
    ctx.set_option(magus.OPT_SEGMENTS, segments)
    try:
        r = ctx.replay(buf, pols, n_traces=N, want_decisions=decisions)
        torch.cuda.synchronize()
        return r
    finally:
        ctx.set_option(magus.OPT_FAMILY, 0)
        ctx.set_option(magus.OPT_SEGMENTS, 0)


def _check(ctx, x, pols, segments=0, decisions=True):
    T, N = x.shape
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=decisions)
    r = _run(ctx, x, pols, True, segments, decisions)
    assert_parity(r, ref, pols, T, check_dec=False)
    if decisions:
        words = oracle.decision_words(ref.dec, R_MIN)
        assert np.array_equal(r.decisions_numpy().transpose(0, 2, 1), words), "decision words"
    return r


def _random_family(rng):
    """A family-eligible policy list: one (W, H, L), ni x nd threshold pairs
    (<= 16 bundles), 1-4 t_hi each (short bundles are padded)."""
    W = int(rng.choice([2, 3, 4, 6, 10, 16, 17, 31, 32, 33]))
    H = int(rng.choice([10, 10, 1, 5, 13, 32]))
    L = float(W) if rng.random() < 0.7 else float(rng.uniform(0.5, 40.0))
    ni, nd = int(rng.integers(1, 9)), int(rng.integers(1, 9))
    incs = sorted(set(float(v) for v in rng.choice([0.0, 50.0, 100.0, 200.0, 300.0, 400.0, 1000.0, 2500.0], ni)))
    decs = sorted(set(float(v) for v in rng.choice([-100.0, -250.0, -500.0, -750.0, -1000.0, -3000.0], nd)))
    pairs = [(a, b) for a in incs for b in decs]
    rng.shuffle(pairs)
    pairs = pairs[:16]
    rows = []
    for a, b in pairs:
        nth = int(rng.integers(1, 5))
        for t in sorted(rng.choice([0.1, 0.2, 0.3, 0.4, 0.5, 0.7, 1.0], nth, replace=False)):
            rows.append(dict(W=W, H=H, L=L, tau_inc=a, tau_dec=b, t_hi=float(t)))
    order = rng.permutation(len(rows))  # configs in any order
    return [magus.make_policy(**rows[i]) for i in order]


def test_sweep256_family_small(ctx):
    N, T = 100, 3001
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    _check(ctx, x, magus.grid_sweep256(), decisions=True)


@pytest.mark.parametrize("segments", [1, 3, 40])
def test_fleet64_family_segments(ctx, segments):
    N, T = 77, 4000
    x = gen.gen_traces(gen.SEEDS[2] + segments, N, T, kind=gen.KIND_ADVERSARIAL)
    _check(ctx, x, magus.grid_fleet64(), segments=segments)


@pytest.mark.parametrize("case", range(24))
def test_random_family_bit_exact(ctx, case):
    rng = np.random.default_rng(0xFA0000 + case)
    pols = _random_family(rng)
    N = int(rng.choice([1, 31, 32, 33, 95, 200]))
    T = int(rng.choice([1, 31, 33, 700, 2049]))
    kind = gen.KIND_ADVERSARIAL if rng.random() < 0.4 else gen.KIND_MIX
    x = gen.gen_traces(gen.SEEDS[5] + case, N, T, kind=kind)
    _check(ctx, x, pols, segments=int(rng.choice([0, 1, 2, 7])))


def test_family_equals_bundle_kernel(ctx):
    """Every output word identical to the per-bundle stream kernel's at a size
    spanning many trace groups and segments."""
    N, T = 1000, 20000
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    pols = magus.grid_sweep256()
    a = _run(ctx, x, pols, True, 0, True)
    a = (a.summary_numpy().copy(), a.base_numpy().copy(), a.decisions_numpy().copy(), a.totals_numpy().copy())
    b = _run(ctx, x, pols, False, 0, True)
    assert np.array_equal(a[0], b.summary_numpy())
    assert np.array_equal(a[1], b.base_numpy())
    assert np.array_equal(a[2], b.decisions_numpy())
    assert np.array_equal(a[3], b.totals_numpy())


def test_family_resume_chunks(ctx):
    """Time-chunked replay (config 4's mode) on the family kernel."""
    from test_gpu_resume import check_chunked
    N, T = 70, 3000
    x = gen.gen_traces(gen.SEEDS[4], N, T, kind=gen.KIND_ADVERSARIAL)
    check_chunked(ctx, x, magus.grid_fleet64(), [0, 64, 1024, 1056, 2496, 3000], segments=2)


def test_family_launch_is_used(ctx):
    """SWEEP256 runs as 4 family launches (one per W), FLEET64 as one."""
    N, T = 64, 500
    xd = ctx.gen_traces(gen.SEEDS[1], N, T)
    for pols, nl, grid in ((magus.grid_sweep256(), 4, 4 * 2), (magus.grid_fleet64(), 1, 2)):
        ctx.set_option(magus.OPT_SEGMENTS, 1)
        before = ctx.stats()["launches_total"]
        ctx.replay(xd, pols, want_summary=False, want_base=False)
        torch.cuda.synchronize()
        st = ctx.stats()
        ctx.set_option(magus.OPT_SEGMENTS, 0)
        assert st["launches_total"] - before == nl
        assert st["last_family"] == nl
        assert st["last_grid"] == grid  # 2 groups of 32 traces x 1 segment per launch
    ctx.set_option(magus.OPT_FAMILY, 1)
    try:
        ctx.replay(xd, magus.grid_fleet64(), want_summary=False, want_base=False)
        torch.cuda.synchronize()
        assert ctx.stats()["last_family"] == 0
    finally:
        ctx.set_option(magus.OPT_FAMILY, 0)
