"""CUDA path vs the CPU oracle, element by element (needs a B200).

Everything goes through the C-ABI (libmagus.so) via the thin binding.  The
bar: decisions, counters, digests and q sums bit-exact; per-(trace, config)
time/energy bit-exact (model M fixes the fp64 operation order and both sides
compile without FMA contraction); fleet totals: integer words bit-exact, fp64
derivation bit-exact, and within 1e-12 of the exactly rounded sum of the
per-trace energies.
"""
from __future__ import annotations

import math

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")

R_MIN = 8
FIELDS = [("n_events", "n_events"), ("n_hi_rounds", "n_hi_rounds"), ("n_msr_writes", "n_msr_writes"),
          ("n_changes", "n_changes"), ("n_min_dec", "n_min_dec"), ("n_min_int", "n_min_int"),
          ("q_min", "q_min"), ("q_max", "q_max"), ("digest", "digest"), ("time_s", "time"),
          ("energy_j", "energy"), ("slowdown", "slowdown"), ("viol", "viol")]


@pytest.fixture(scope="module")
def ctx():
    c = magus.Context(device=0)
    yield c
    c.close()


def to_oracle_policies(pols):
    return oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                 tau_dec=p.tau_dec, t_hi=p.t_hi, variant=p.variant, step=p.step) for p in pols])


def run_gpu(ctx, x_np, pols, kernel, segments=0, ld=None, decisions=True):
    T, N = x_np.shape
    ld = (N + 3) // 4 * 4 if ld is None else ld      # TMA needs a 16-B row pitch
    xd = torch.zeros((T, ld), dtype=torch.float32, device="cuda:0")
    xd[:, :N] = torch.from_numpy(x_np).cuda()
    ctx.set_option(magus.OPT_KERNEL, kernel)
    ctx.set_option(magus.OPT_SEGMENTS, segments)
    try:
        r = ctx.replay(xd, pols, n_traces=N, want_decisions=decisions)
        torch.cuda.synchronize()
    finally:
        ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_AUTO)
        ctx.set_option(magus.OPT_SEGMENTS, 0)
    return r


def assert_parity(r, ref, pols, T, check_dec=True):
    got = r.summary_numpy()
    for gf, of in FIELDS:
        a, b = got[gf], ref.summary[of]
        bad = np.argwhere(a != b)
        assert bad.size == 0, f"{gf}: first mismatch at {bad[0]} gpu={a[tuple(bad[0])]} oracle={b[tuple(bad[0])]}"
    gb = r.base_numpy()
    assert np.array_equal(gb["q_base"], ref.base["q_base"])
    assert np.array_equal(gb["time_s"], ref.base["time"]) and np.array_equal(gb["energy_j"], ref.base["energy"])
    if check_dec and r.decisions is not None:
        words = oracle.decision_words(ref.dec, R_MIN)                 # [C, N, nw]
        got_w = r.decisions_numpy().transpose(0, 2, 1)               # [C, N, nw]
        assert np.array_equal(got_w, words), "decision bits differ"
    tot = r.totals_numpy()
    for c in range(len(pols)):
        w, f = oracle.totals(ref.summary[c], ref.base, T)
        assert np.array_equal(tot[c], w), f"totals words differ for config {c}"


POLS_SMALL = None


def small_policies():
    P = [magus.policy_preset(magus.POLICY_PAPER_DEFAULT), magus.policy_preset(magus.POLICY_PAPER_PARETO),
         magus.make_policy(W=2, H=1, tau_inc=50, tau_dec=-50, t_hi=1.0),
         magus.make_policy(W=4, H=10, tau_inc=100, tau_dec=-250, t_hi=0.2),
         magus.make_policy(W=6, H=10, tau_inc=400, tau_dec=-1000, t_hi=0.5),
         magus.make_policy(W=16, H=10, tau_inc=300, tau_dec=-750, t_hi=0.3),
         magus.make_policy(W=33, H=32, tau_inc=37, tau_dec=-61, t_hi=0.25),
         magus.make_policy(W=7, H=5, L=3.5, tau_inc=123.25, tau_dec=-77.5, t_hi=0.6),
         magus.make_policy(W=12, H=17, tau_inc=150, tau_dec=-300, t_hi=1.5)]
    return P


@pytest.mark.parametrize("kernel", [magus.KERNEL_REFERENCE, magus.KERNEL_STREAM])
@pytest.mark.parametrize("kind", [gen.KIND_MIX, gen.KIND_ADVERSARIAL])
def test_parity_small(ctx, kernel, kind):
    N, T = 300, 3001                       # ragged in both tiles (128 traces, 32 steps)
    x = gen.gen_traces(gen.SEEDS[1] + kind, N, T, kind=kind)
    pols = small_policies()
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    r = run_gpu(ctx, x, pols, kernel)
    assert_parity(r, ref, pols, T)


@pytest.mark.parametrize("segments", [1, 2, 3, 7, 29, 94])
def test_segmentation_is_exact(ctx, segments):
    N, T = 256, 3000
    x = gen.gen_traces(gen.SEEDS[2], N, T)
    pols = small_policies()[:6]
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    r = run_gpu(ctx, x, pols, magus.KERNEL_STREAM, segments=segments)
    assert_parity(r, ref, pols, T)


def test_prefix_fixup_long_quiet_segments(ctx):
    """Traces that stay at min for many segments force the carry fix-up to
    flip whole segments (no action inside) and to patch their decision bits."""
    N, T = 130, 4000
    t = np.arange(T)[:, None]
    x = np.where(t < 300, 20000.0, 900.0) * np.ones((1, N))
    x[2000:2003, ::3] = 30000.0                       # a late burst on some traces
    x = x.astype(np.float32)
    pols = [magus.make_policy(), magus.make_policy(W=4, H=10, t_hi=0.5)]
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    for segments in (0, 5, 40, 125):
        r = run_gpu(ctx, x, pols, magus.KERNEL_STREAM, segments=segments)
        assert_parity(r, ref, pols, T)


@pytest.mark.parametrize("kernel", [magus.KERNEL_REFERENCE, magus.KERNEL_STREAM])
@pytest.mark.parametrize("N,T,ld", [(1, 1, 4), (1, 9, 4), (1, 10, 4), (5, 11, 8), (3, 31, 4), (33, 32, 36),
                                    (129, 33, 132), (1, 10000, 4), (64, 65, 64)])
def test_edge_shapes(ctx, kernel, N, T, ld):
    x = gen.gen_traces(gen.SEEDS[3], N, T, kind=gen.KIND_ADVERSARIAL)
    pols = small_policies()
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    r = run_gpu(ctx, x, pols, kernel, ld=ld)
    assert_parity(r, ref, pols, T)


def test_special_values(ctx):
    """NaN -> hold; exact Alg. 1 ties; huge stretch (cap 2^15); negatives."""
    N, T = 64, 700
    rng = np.random.default_rng(5)
    x = rng.choice([0.0, 1000.0, 3000.0, 6000.0, 6001.0, 1001.0, 3001.0, 24000.0, 5e9, 3e38, -5000.0],
                   size=(T, N)).astype(np.float32)
    x[rng.random((T, N)) < 0.02] = np.nan
    pols = small_policies()
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    for kernel in (magus.KERNEL_REFERENCE, magus.KERNEL_STREAM):
        r = run_gpu(ctx, x, pols, kernel, segments=5 if kernel == magus.KERNEL_STREAM else 0)
        assert_parity(r, ref, pols, T)


def test_threshold_inversion_boundaries(ctx):
    """Deltas at and +-1 ulp around tau * L for awkward L (non-power-of-two)."""
    T = 64
    pols = [magus.make_policy(W=2, H=3, L=L, tau_inc=ti, tau_dec=td, t_hi=0.7)
            for L, ti, td in [(3.0, 0.1, -0.7), (10.0, 200.0, -500.0), (7.0, 1 / 3, -2 / 3), (0.3, 17.0, -19.0)]]
    cols = []
    for p in pols:
        for thr in (p.tau_inc * p.deriv_len, p.tau_dec * p.deriv_len):
            f = np.float32(thr)
            for v in (np.nextafter(f, np.float32(-np.inf)), f, np.nextafter(f, np.float32(np.inf))):
                col = np.zeros(T, np.float32)
                col[1::2] = v                               # lag-1 deltas of +-v
                cols.append(col)
    x = np.stack(cols, axis=1)
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    for kernel in (magus.KERNEL_REFERENCE, magus.KERNEL_STREAM):
        assert_parity(run_gpu(ctx, x, pols, kernel), ref, pols, T)


def test_sweep256_small_and_best(ctx):
    N, T = 160, 2000
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    pols = magus.grid_sweep256()
    ref = oracle.replay(x, to_oracle_policies(pols))
    r = run_gpu(ctx, x, pols, magus.KERNEL_AUTO, decisions=False)
    assert_parity(r, ref, pols, T, check_dec=False)
    best, row, feasible = ctx.sweep_best(r.totals)
    viol = [oracle.totals(ref.summary[c], ref.base, T)[0][1] for c in range(256)]
    energy = [oracle.totals(ref.summary[c], ref.base, T)[1][0] for c in range(256)]
    ob, ofeas = oracle.sweep_best(viol, energy)
    assert (best, feasible) == (ob, ofeas)
    assert row["energy_j"] == energy[ob]
    e_parts = math.fsum(ref.summary[ob]["energy"].tolist())
    assert math.isclose(row["energy_j"], e_parts, rel_tol=1e-12)


def test_device_generator_matches_host(ctx):
    for kind in (gen.KIND_MIX, gen.KIND_ADVERSARIAL):
        d = ctx.gen_traces(gen.SEEDS[4], 300, 777, kind=kind, id0=1000, ld=304)
        torch.cuda.synchronize()
        h = gen.gen_traces(gen.SEEDS[4], 300, 777, kind=kind, id0=1000, ld=304)
        assert np.array_equal(d.cpu().numpy(), h)


def test_replay_host_e2e_matches_device(ctx):
    N, T = 200, 2500
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    pols = small_policies()[:3]
    s, b, d, t = ctx.replay_host(x, pols, want_decisions=True)
    r = run_gpu(ctx, x, pols, magus.KERNEL_AUTO)
    assert np.array_equal(s, r.summary_numpy()) and np.array_equal(b, r.base_numpy())
    assert np.array_equal(d, r.decisions_numpy()) and np.array_equal(t, r.totals_numpy())


def test_fake_sharded_totals_equal_single(ctx):
    """Partition + merge without NCCL: G shards on one GPU, integer totals
    summed on the host == one replay over all traces (bitwise)."""
    N, T = 512, 3000
    xd = ctx.gen_traces(gen.SEEDS[4], N, T)
    pols = magus.grid_fleet64()[:16]
    full = ctx.replay(xd, pols, want_summary=False, want_base=False).totals_numpy()
    for G in (2, 4, 8):
        acc = np.zeros_like(full)
        per = N // G
        for g in range(G):
            sub = xd[:, g * per:(g + 1) * per]          # column block, same ld
            t = ctx.replay(sub, pols, n_traces=per, want_summary=False, want_base=False).totals_numpy()
            acc[:, 0] += t[:, 0]
            acc[:, 1:15] += t[:, 1:15]
        acc[:, 15] = full[:, 15]
        assert np.array_equal(acc, full)


def test_full_config2_sampled_parity(ctx):
    """BASELINE config 2 at full size (4096 x 100,000, paper default) in the
    launch configuration bench.py times; the oracle checks a sample of traces
    one by one (each trace's result depends only on its own samples)."""
    N, T = 4096, 100_000
    xd = ctx.gen_traces(gen.SEEDS[2], N, T)
    pol = [magus.policy_preset(magus.POLICY_PAPER_DEFAULT)]
    r = ctx.replay(xd, pol, want_decisions=True)
    torch.cuda.synchronize()
    got = r.summary_numpy()
    dec = r.decisions_numpy()
    sample = np.r_[0, 1, 127, 128, 2047, 4095, np.random.default_rng(0).integers(0, N, 26)]
    xs = xd[:, torch.as_tensor(sample, device="cuda:0")].cpu().numpy()
    ref = oracle.replay(np.ascontiguousarray(xs), oracle.policy(), want_dec=True)
    for i, n in enumerate(sample):
        for gf, of in FIELDS:
            assert got[gf][0, n] == ref.summary[of][0, i], (gf, n)
        words = oracle.decision_words(ref.dec[0, i], R_MIN)
        assert np.array_equal(dec[0, :, n], words)
    # the reference kernel agrees on every trace
    ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_REFERENCE)
    try:
        r2 = ctx.replay(xd, pol, want_decisions=False)
        torch.cuda.synchronize()
    finally:
        ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_AUTO)
    assert np.array_equal(r2.summary_numpy(), got)
    assert np.array_equal(r2.totals_numpy(), r.totals_numpy())


@pytest.mark.parametrize("bundle", [0, 1, 2, 4])
def test_bundles_share_alg1_alg2_work_exactly(ctx, bundle):
    """Configs differing only in t_hi share Delta, events and the window count
    (one thread, NB configs); padding and any NB give identical results."""
    N, T = 200, 2600
    x = gen.gen_traces(gen.SEEDS[3], N, T)
    pols = [magus.make_policy(W=10, tau_inc=ti, tau_dec=td, t_hi=th)
            for (ti, td) in [(200, -500), (100, -250)] for th in (0.2, 0.3, 0.4, 0.5, 0.7)]
    pols += [magus.make_policy(W=6, tau_inc=300, tau_dec=-750, t_hi=th) for th in (0.1, 0.4, 1.5)]
    pols += [magus.make_policy(W=7, H=13, L=3.0, tau_inc=90, tau_dec=-90, t_hi=th) for th in (0.25, 0.5)]
    ref = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    ctx.set_option(magus.OPT_BUNDLE, bundle)
    try:
        for segments in (0, 7):
            r = run_gpu(ctx, x, pols, magus.KERNEL_STREAM, segments=segments)
            assert_parity(r, ref, pols, T)
    finally:
        ctx.set_option(magus.OPT_BUNDLE, 0)
