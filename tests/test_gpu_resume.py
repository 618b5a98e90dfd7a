"""Time-chunked replay (magus_replay_resume) vs the CPU oracle (needs a B200).

SURVEY §8(b) names the resumable call and §8(d)/(e) need it for config 4
(262 GB of traces on one GPU).  Its exactness rests on the closed form of
Alg. 3: p_t and the Alg. 2 history depend only on
x[t-W-H+1..t], and dec[t_start-1] is the only carried decision state.

The bar: after every chunk the summaries, base and totals equal the ORACLE's
replay of the prefix [0, t_end) bit for bit, and the concatenated decision
words of all chunks equal the oracle's decisions of the whole trace.
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle
from test_gpu_parity import R_MIN, assert_parity, small_policies, to_oracle_policies

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")


@pytest.fixture(scope="module")
def ctx():
    c = magus.Context(device=0)
    yield c
    c.close()


def stream_policies():
    # stream-kernel configs only (W <= 33, H <= 32); bundles of NB > 1 included
    P = [p for p in small_policies() if p.history <= 32 and p.window <= 33]
    fleet = magus.grid_fleet64()
    return P + [fleet[i] for i in (0, 16, 32, 48, 37, 38)]


def run_chunks(ctx, x, pols, bounds, segments=0):
    """Replays x [T, N] in chunks [bounds[i], bounds[i+1]); yields per chunk
    (t_end, result)."""
    T, N = x.shape
    ld = (N + 3) // 4 * 4
    halo = magus.resume_halo(pols)
    state = ctx.resume_state(N, pols)
    ctx.set_option(magus.OPT_SEGMENTS, segments)
    try:
        for t_start, t_end in zip(bounds[:-1], bounds[1:]):
            t_base = max(0, t_start - halo)
            buf = torch.zeros((t_end - t_base, ld), dtype=torch.float32, device="cuda:0")
            buf[:, :N] = torch.from_numpy(x[t_base:t_end]).cuda()
            r = ctx.replay_resume(buf, pols, state, t_base=t_base, t_start=t_start, n_traces=N,
                                  want_decisions=True)
            torch.cuda.synchronize()
            yield t_start, t_end, r
    finally:
        ctx.set_option(magus.OPT_SEGMENTS, 0)


def check_chunked(ctx, x, pols, bounds, segments=0):
    T, N = x.shape
    full = oracle.replay(x, to_oracle_policies(pols), want_dec=True)
    full_words = oracle.decision_words(full.dec, R_MIN)          # [C, N, nw]
    for t_start, t_end, r in run_chunks(ctx, x, pols, bounds, segments):
        ref = oracle.replay(np.ascontiguousarray(x[:t_end]), to_oracle_policies(pols))
        assert_parity(r, ref, pols, t_end, check_dec=False)
        got = r.decisions_numpy().transpose(0, 2, 1)            # [C, N, words of the chunk]
        w0, w1 = t_start // 32, (t_end + 31) // 32
        assert np.array_equal(got, full_words[:, :, w0:w1]), f"decision words of chunk [{t_start}, {t_end})"


@pytest.mark.parametrize("kind", [gen.KIND_MIX, gen.KIND_ADVERSARIAL])
def test_resume_chunks_match_oracle(ctx, kind):
    N, T = 300, 4001                                   # ragged tiles
    x = gen.gen_traces(gen.SEEDS[1] + 7 + kind, N, T, kind=kind)
    check_chunked(ctx, x, stream_policies(), [0, 64, 1024, 1056, 2720, 4001])


@pytest.mark.parametrize("segments", [1, 3, 17])
def test_resume_carry_through_quiet_chunks(ctx, segments):
    """A held min (the F5 echo of a 2-sample burst) must cross chunk borders
    and whole action-free segments: every look-back falls through to the
    resume carry."""
    N, T = 130, 6000
    t = np.arange(T)[:, None]
    x = np.full((T, N), 900.0)
    x[1000:1002, ::2] = 30000.0                        # echo -> min from t = 1009, held
    x[4500:4502, 1::4] = 30000.0                        # a late one on other traces
    x[3000:3100, 5::7] = np.where(t[3000:3100] % 2 == 0, 20000.0, 900.0)  # oscillation -> hi
    x = x.astype(np.float32)
    pols = [magus.make_policy(), magus.make_policy(W=4, H=10, t_hi=0.5),
            magus.make_policy(W=10, H=10, tau_inc=300, t_hi=0.4)]
    check_chunked(ctx, x, pols, [0, 1024, 1056, 3008, 4512, 6000], segments=segments)


def test_resume_equals_one_shot(ctx):
    """Chunked == one-shot replay (summary bytes, totals, decisions)."""
    N, T = 1000, 9000
    x = gen.gen_traces(gen.SEEDS[2] + 11, N, T)
    pols = stream_policies()
    ld = (N + 3) // 4 * 4
    xd = torch.zeros((T, ld), dtype=torch.float32, device="cuda:0")
    xd[:, :N] = torch.from_numpy(x).cuda()
    one = ctx.replay(xd, pols, n_traces=N, want_decisions=True)
    words = []
    last = None
    for _, _, r in run_chunks(ctx, x, pols, [0, 2048, 2080, 7040, 9000]):
        words.append(r.decisions_numpy())
        last = r
    torch.cuda.synchronize()
    assert np.array_equal(last.summary.cpu().numpy(), one.summary.cpu().numpy())
    assert np.array_equal(last.base.cpu().numpy(), one.base.cpu().numpy())
    assert np.array_equal(last.totals.cpu().numpy(), one.totals.cpu().numpy())
    assert np.array_equal(np.concatenate(words, axis=1), one.decisions_numpy())


def test_resume_validation(ctx):
    pols = [magus.make_policy()]
    N = 8
    state = ctx.resume_state(N, pols)
    buf = torch.zeros((64, 8), dtype=torch.float32, device="cuda:0")
    with pytest.raises(magus.MagusError):       # t_start not a multiple of 32
        ctx.replay_resume(buf, pols, state, t_base=0, t_start=5)
    with pytest.raises(magus.MagusError):       # halo missing (W + H - 1 = 19 rows -> 32)
        ctx.replay_resume(buf, pols, state, t_base=64, t_start=64)
    with pytest.raises(magus.MagusError):       # t_start outside the buffer
        ctx.replay_resume(buf, pols, state, t_base=0, t_start=64)
    gradual = [magus.make_policy(variant=magus.VARIANT_GRADUAL, step=1)]
    with pytest.raises(magus.MagusError):       # per-sample variants do not chunk
        ctx.replay_resume(buf, gradual, ctx.resume_state(N, gradual), t_base=0, t_start=0)


@pytest.mark.parametrize("kind", [gen.KIND_MIX, gen.KIND_ADVERSARIAL])
def test_gen_resume_matches_one_shot(ctx, kind):
    """Chunked device generation == the host generator (and so == one shot)."""
    N, T = 300, 2000
    host = gen.gen_traces(gen.SEEDS[4] + kind, N, T, kind=kind, id0=77)
    state = ctx.gen_state(N)
    buf = torch.zeros((700, 304), dtype=torch.float32, device="cuda:0")
    got = []
    for t0, t1 in [(0, 5), (5, 700), (700, 1333), (1333, 2000)]:
        ctx.gen_traces_resume(gen.SEEDS[4] + kind, N, t0, t1 - t0, state, buf, kind=kind, id0=77)
        got.append(buf[: t1 - t0, :N].cpu().numpy().copy())
    assert np.array_equal(np.concatenate(got), host)
