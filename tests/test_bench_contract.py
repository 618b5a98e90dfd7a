"""bench.py's contract on the CPU: the reference arm (the oracle on the host
cores) prints one JSON line with the keys the driver reads, and the
thread-partitioned oracle used by the CPU baseline equals the plain
single-threaded oracle trace for trace."""
from __future__ import annotations

import json
import os
import subprocess
import sys

import numpy as np

import gen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


_RUN_AND_LIST_SO = """
import runpy, sys
sys.argv = ["bench.py", "--impl", "reference", "--steps", "1", "--warmup", "1", "--cpu-threads", "2",
            "--ref-budget", "8"]
try:
    runpy.run_path("bench.py", run_name="__main__")
except SystemExit:
    pass
maps = open("/proc/self/maps").read()
print("LOADED:" + ",".join(sorted({ln.split()[-1].rsplit("/", 1)[-1] for ln in maps.splitlines()
                                  if ln.rstrip().endswith(".so")})))
"""


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, "-c", _RUN_AND_LIST_SO], cwd=ROOT, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0, r.stderr
    lines = [ln for ln in r.stdout.splitlines() if ln.strip() and not ln.startswith("LOADED:")]
    loaded = [ln for ln in r.stdout.splitlines() if ln.startswith("LOADED:")][0]
    # the reference arm runs the oracle only: the product library is never loaded
    assert "libmagus.so" not in loaded.split(":", 1)[1].split(","), loaded
    assert "liboracle.so" in loaded, loaded
    assert len(lines) == 1
    d = json.loads(lines[0])
    # our arm's config object, field for field
    assert d["config"] == bench.workload_config(2, 1, "traces")
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 2
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["config"]["workload"].startswith("cfg2")


def test_partitioned_oracle_equals_single_thread():
    x = gen.gen_traces(gen.SEEDS[2], 37, 3000)
    pols = bench.oracle_grid("sweep256")[:5]
    ref = oracle.replay(x, pols).summary
    pool = bench.OraclePool(4)
    try:
        got = pool.replay(x, pols)
    finally:
        pool.close()
    assert got.shape == ref.shape
    for f in ref.dtype.names:
        assert np.array_equal(got[f], ref[f]), f


def test_committed_bench_lines_carry_the_contract_keys():
    """Every bench line kept under profiles/ has the keys the driver and the
    judge read (roofline with its fraction, clocks, launches, baselines)."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r0*_bench_*.json")))
    assert files
    for f in files:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
                  "dtype", "data", "config"):
            assert k in d, (f, k)
        assert d["value"] > 0, f
        if d.get("impl") == "reference":
            assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
            continue
        assert "workload" in d["config"], f
        r = d["roofline"]
        assert r["bound"] in ("hbm", "alu") and r["peak"] > 0 and r["achieved"] > 0, f
        assert abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-9, f
        assert d["gpu_launches"] > 0 and "clocks" in d, f


def test_oracle_grids_match_the_product_grids():
    """The reference arm uses the oracle's own restatement of SWEEP256 /
    FLEET64; it must equal the library's presets."""
    import oracle
    for grid in ("sweep256", "fleet64"):
        o = bench.oracle_grid(grid)
        p = bench.oracle_policies(bench.policies_for(grid))
        assert o.tobytes() == p.tobytes(), grid
    g = oracle.grid_sweep256()
    assert (g[165]["W"], g[165]["tau_inc"], g[165]["tau_dec"], g[165]["t_hi"]) == (10, 200.0, -500.0, 0.4)
    assert (g[166]["tau_inc"]) == 300.0
    f = oracle.grid_fleet64()
    assert len(f) == 64 and f[37]["tau_inc"] == 200.0 and f[38]["tau_inc"] == 300.0


def test_workload_config_scaling_labels():
    """Configs 1-3 are quoted on one B200 (weak: traces per GPU); configs 4
    and 5 are fixed fleets sharded over the GPUs (strong)."""
    for g in (1, 2, 4, 8):
        c5 = bench.workload_config(5, g, "traces")
        assert c5["n_traces_total"] == 16384 and c5["scaling"] == "strong"
        assert c5["n_traces_per_gpu"] == 16384 // g
        assert c5["workload"].startswith("cfg5: 16,384 traces")
        c4 = bench.workload_config(4, g, "traces")
        assert c4["n_traces_total"] == 65536 and c4["scaling"] == "strong"
        c2 = bench.workload_config(2, g, "traces")
        assert c2["n_traces_total"] == 4096 * g and c2["scaling"] == "weak"
        c3 = bench.workload_config(3, g, "configs")
        assert c3["n_traces_total"] == 4096 and c3["n_traces_per_gpu"] == 4096 and c3["scaling"] == "strong"
