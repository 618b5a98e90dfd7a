"""magus_sweep_best_async: the device derivation/choice must equal the host
one bit for bit, including 128-bit q sums (correctly rounded u128 -> double)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")


def _random_totals(rng, C, big):
    w = np.zeros((C, magus.TOT_WORDS), np.uint64)
    w[:, 0] = rng.integers(1, 1 << 20, C)
    w[:, 1] = rng.integers(0, 3, C)                       # some configs feasible, some not
    for k in range(2, 8):
        w[:, k] = rng.integers(0, 1 << 40, C)
    w[:, 14] = w[:, 0] * np.uint64(100000)
    w[:, 7] = np.minimum(w[:, 7], w[:, 14])
    for k in range(8, 14):                                # q limb sums: up to 2^64 - 1
        w[:, k] = rng.integers(0, (1 << 63) if big else (1 << 40), C, dtype=np.uint64) * np.uint64(2 if big else 1)
    w[:, 15] = rng.integers(0, 1 << 30, C)
    w[:, 16] = np.minimum(w[:, 15], rng.integers(0, 1 << 30, C).astype(np.uint64))
    return w


@pytest.mark.parametrize("big", [False, True])
@pytest.mark.parametrize("seed", range(3))
def test_device_choice_equals_host(big, seed):
    rng = np.random.default_rng(seed)
    with magus.Context(device=0) as ctx:
        for C in (1, 7, 64, 256):
            w = _random_totals(rng, C, big)
            if seed == 2:
                w[:, 1] = 1                                   # none feasible
            td = torch.from_numpy(w.view(np.int64).copy()).cuda()
            out = ctx.sweep_best_async(td)
            torch.cuda.synchronize()
            best, row, feasible = ctx.sweep_result(out)
            hb, hrow, hfeas = magus.sweep_best_host(w)
            assert (best, feasible) == (hb, hfeas)
            for k, v in hrow.items():
                assert row[k] == v or (np.isnan(row[k]) and np.isnan(v)), k
            for c in range(C):
                d = magus.derive_host(w[c])
                assert d["energy_j"] == ctx.totals_derive(w[c])["energy_j"]


def test_async_step_matches_sync_step():
    import gen
    with magus.Context(device=0) as ctx:
        x = ctx.gen_traces(gen.SEEDS[3], 256, 3000)
        pols = magus.grid_fleet64()
        r = ctx.replay(x, pols, want_summary=False, want_base=False)
        out = ctx.sweep_best_async(r.totals)
        torch.cuda.synchronize()
        assert ctx.sweep_result(out) == ctx.sweep_best(r.totals)


@pytest.mark.parametrize("config", [2, 3])
def test_bench_steps_in_flight_agree(config):
    """bench.py with two steps in flight (two contexts on two streams)
    reports the same choice as strictly serial steps, and every launch of
    both contexts is counted."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    lines = []
    for inflight in (1, 2):
        r = subprocess.run([sys.executable, "bench.py", "--config", str(config), "--n-traces", "1024", "--n-steps",
                            "131072", "--steps", "6", "--warmup", "3", "--no-cpu-baseline", "--no-e2e",
                            "--inflight", str(inflight)], cwd=root, capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-2000:]
        lines.append(json.loads(r.stdout.strip().splitlines()[-1]))
    a, b = lines
    # (inputs above 4 x L2: no flush between steps, so steps may overlap)
    assert a["run"]["steps_in_flight"] == 1 and b["run"]["steps_in_flight"] == 2
    assert a["best_config"] == b["best_config"] and a["feasible"] == b["feasible"]
    assert a["gpu_launches"] == b["gpu_launches"]
