"""CPU ORACLE for the MAGUS replay -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package (``paper_conf_sc_zhengspl25_b200``) never does.

A ctypes wrapper over ``oracle/liboracle.so`` (built from magus_oracle.cpp by
``__graft_entry__.build()`` with ``g++ -O2 -ffp-contract=off``).  All types
here are defined independently of ``include/magus.h``.

Pinned by ``tests/test_oracle_*.py`` against closed forms, brute force,
invariants and the hand-derived golden fixtures in ``tests/golden/``.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")

POLICY_DT = np.dtype([("W", "<i4"), ("H", "<i4"), ("L", "<f8"), ("tau_inc", "<f8"),
                      ("tau_dec", "<f8"), ("t_hi", "<f8"), ("variant", "<i4"), ("step", "<i4")],
                     align=True)
PLATFORM_DT = np.dtype([("r_min", "<i4"), ("r_max", "<i4"), ("dt", "<f8"), ("bw_max", "<f8"),
                        ("beta", "<f8"), ("p_other", "<f8"), ("p_unc_min", "<f8"),
                        ("p_unc_max", "<f8"), ("e_sw", "<f8"), ("t_sw", "<f8"),
                        ("bound", "<f8"), ("burst", "<f8")], align=True)
SUMMARY_DT = np.dtype([("n_events", "<i8"), ("n_hi_rounds", "<i8"), ("n_msr_writes", "<i8"),
                       ("n_changes", "<i8"), ("n_min_dec", "<i8"), ("n_min_int", "<i8"),
                       ("q_min", "<u8"), ("q_max", "<u8"), ("digest", "<u8"), ("time", "<f8"),
                       ("energy", "<f8"), ("slowdown", "<f8"), ("viol", "<i4"),
                       ("reserved", "<i4"), ("n_burst_base", "<i8"), ("n_burst_magus", "<i8"),
                       ("n_burst_inter", "<i8"), ("n_burst_union", "<i8")], align=True)
BASE_DT = np.dtype([("q_base", "<u8"), ("time", "<f8"), ("energy", "<f8"),
                    ("reserved", "<u8")], align=True)

_lib = None


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build()")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i64, i32, f64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
    lib.oracle_alg1.restype = ctypes.c_int
    lib.oracle_alg1.argtypes = [vp, i32, f64, f64, f64]
    lib.oracle_alg2.restype = ctypes.c_int
    lib.oracle_alg2.argtypes = [vp, i32, f64]
    for fn in (lib.oracle_replay, lib.oracle_replay_closed_form):
        fn.restype = ctypes.c_int
        fn.argtypes = [vp, i64, i64, i64, vp, i32, vp, vp, vp, vp, vp]
    lib.oracle_model_account.restype = ctypes.c_int
    lib.oracle_model_account.argtypes = [vp, i64, vp, vp, vp, vp]
    lib.oracle_totals.restype = ctypes.c_int
    lib.oracle_totals.argtypes = [vp, vp, i64, i64, vp, vp, vp]
    lib.oracle_energy_sum.restype = ctypes.c_double
    lib.oracle_energy_sum.argtypes = [vp, i64]
    lib.oracle_offline_bound.restype = ctypes.c_int
    lib.oracle_offline_bound.argtypes = [vp, i64, vp, f64, i32, vp]
    lib.oracle_sweep_best.restype = ctypes.c_int
    lib.oracle_sweep_best.argtypes = [vp, vp, i32, vp]
    for n in ("summary", "policy", "platform"):
        getattr(lib, f"oracle_sizeof_{n}").restype = ctypes.c_int32
    assert lib.oracle_sizeof_summary() == SUMMARY_DT.itemsize
    assert lib.oracle_sizeof_policy() == POLICY_DT.itemsize
    assert lib.oracle_sizeof_platform() == PLATFORM_DT.itemsize
    _lib = lib
    return lib


# ---------------------------------------------------------------------------
# Paper parameters (restated here, independently of the product presets).
# ---------------------------------------------------------------------------

def policy(W=10, H=10, L=None, tau_inc=200.0, tau_dec=-500.0, t_hi=0.4, variant=0, step=None) -> np.ndarray:
    """One config.  Defaults: P@25197 (200 / "500" read as -500 / 0.4), H = 10
    (P@24182), W = 10 and L = W (readings R4/R5).  variant: 0 the
    paper's MAGUS; 1 closed loop (NEXT f3); 2 gradual +-step rule (NEXT f4)."""
    p = np.zeros(1, dtype=POLICY_DT)
    p["W"], p["H"] = W, H
    p["L"] = float(W if L is None else L)
    p["tau_inc"], p["tau_dec"], p["t_hi"] = tau_inc, tau_dec, t_hi
    p["variant"] = variant
    p["step"] = (1 if variant & 2 else 0) if step is None else step
    return p


def policies(rows) -> np.ndarray:
    out = np.zeros(len(rows), dtype=POLICY_DT)
    for i, r in enumerate(rows):
        out[i] = policy(**r)[0]
    return out


def grid_sweep256() -> np.ndarray:
    """SWEEP256 (reading R16 of DESIGN.md 3): tau_inc in
    {100, 200, 300, 400} x tau_dec in {-250, -500, -750, -1000} x t_hi in
    {0.2, 0.3, 0.4, 0.5} x W in {4, 6, 10, 16}, L = W, H = 10; index =
    iInc + 4 (iDec + 4 (iHi + 4 iW)).  paper_default (P@25197) is index 165,
    paper_pareto (P@44170) 166.  Restated here, independently of the product."""
    rows = []
    for W in (4, 6, 10, 16):
        for t_hi in (0.2, 0.3, 0.4, 0.5):
            for tau_dec in (-250.0, -500.0, -750.0, -1000.0):
                for tau_inc in (100.0, 200.0, 300.0, 400.0):
                    rows.append(dict(W=W, H=10, L=float(W), tau_inc=tau_inc, tau_dec=tau_dec, t_hi=t_hi))
    return policies(rows)


def grid_fleet64() -> np.ndarray:
    """FLEET64: the tau_inc x tau_dec x t_hi lines of
    SWEEP256 at W = L = H = 10; index = iInc + 4 (iDec + 4 iHi); default 37."""
    g = grid_sweep256()
    return np.ascontiguousarray(g[g["W"] == 10])


def platform(r_min=8, r_max=22, dt=0.2, bw_max=32000.0, beta=1.0, p_other=218.0,
             p_unc_min=0.0, p_unc_max=82.0, e_sw=0.0, t_sw=0.0, bound=0.05, burst=0.0) -> np.ndarray:
    """Intel+A100 (uncore 0.8-2.2 GHz, P@29320); 82 W uncore range (Fig. 2,
    P@12253); 0.2 s (P@44789); 5 % bound (P@1715).  bw_max/beta/p_other are
    model-M assumptions."""
    p = np.zeros(1, dtype=PLATFORM_DT)
    for k, v in dict(r_min=r_min, r_max=r_max, dt=dt, bw_max=bw_max, beta=beta, p_other=p_other,
                     p_unc_min=p_unc_min, p_unc_max=p_unc_max, e_sw=e_sw, t_sw=t_sw,
                     bound=bound, burst=burst).items():
        p[k] = v
    return p


@dataclass
class OracleResult:
    summary: np.ndarray          # [C, N] SUMMARY_DT
    base: np.ndarray             # [N] BASE_DT
    dec: np.ndarray | None       # [C, N, T] int32 uncore ratio per round
    hi: np.ndarray | None        # [C, N, T] int32 high_freq_status per round


def _as_traces(x) -> tuple[np.ndarray, int, int, int]:
    x = np.ascontiguousarray(x, dtype=np.float32)
    if x.ndim == 1:
        x = x.reshape(-1, 1)
    T, ld = x.shape
    return x, T, ld, ld


def replay(x, pols, plat=None, n_traces=None, want_dec=False, closed_form=False) -> OracleResult:
    """x: time-major float32 [T, ld] (or 1-D for one trace)."""
    lib = _load()
    x, T, ld, _ = _as_traces(x)
    N = ld if n_traces is None else n_traces
    pols = np.ascontiguousarray(pols, dtype=POLICY_DT).reshape(-1)
    plat = platform() if plat is None else np.ascontiguousarray(plat, dtype=PLATFORM_DT)
    C = len(pols)
    summ = np.zeros((C, N), dtype=SUMMARY_DT)
    base = np.zeros(N, dtype=BASE_DT)
    dec = np.zeros((C, N, T), dtype=np.int32) if want_dec else None
    hi = np.zeros((C, N, T), dtype=np.int32) if want_dec else None
    fn = lib.oracle_replay_closed_form if closed_form else lib.oracle_replay
    rc = fn(x.ctypes.data, N, T, ld, pols.ctypes.data, C, plat.ctypes.data, summ.ctypes.data,
            base.ctypes.data, dec.ctypes.data if want_dec else None,
            hi.ctypes.data if want_dec else None)
    if rc != 0:
        raise ValueError("oracle_replay rejected its arguments")
    return OracleResult(summ, base, dec, hi)


def alg1(ls, L, tau_inc, tau_dec) -> int:
    a = np.ascontiguousarray(ls, dtype=np.float64)
    return int(_load().oracle_alg1(a.ctypes.data, len(a), L, tau_inc, tau_dec))


def alg2(ls, t_hi) -> bool:
    a = np.ascontiguousarray(ls, dtype=np.int32)
    return bool(_load().oracle_alg2(a.ctypes.data, len(a), t_hi))


def account(x, dec, plat=None):
    """Model M for an arbitrary decision sequence dec[0..T-1] (ratios)."""
    x = np.ascontiguousarray(x, dtype=np.float32).reshape(-1)
    dec = np.ascontiguousarray(dec, dtype=np.int32).reshape(-1)
    plat = platform() if plat is None else np.ascontiguousarray(plat, dtype=PLATFORM_DT)
    s = np.zeros(1, dtype=SUMMARY_DT)
    b = np.zeros(1, dtype=BASE_DT)
    rc = _load().oracle_model_account(x.ctypes.data, len(x), dec.ctypes.data, plat.ctypes.data,
                                      s.ctypes.data, b.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_model_account rejected its arguments")
    return s[0], b[0]


def totals(summary_row: np.ndarray, base: np.ndarray, T: int, plat=None):
    """(int words[18], derived[7]) for one config's [N] summaries; derived =
    energy, time, base_energy, base_time, saving, slowdown, jaccard."""
    plat = platform() if plat is None else np.ascontiguousarray(plat, dtype=PLATFORM_DT)
    s = np.ascontiguousarray(summary_row, dtype=SUMMARY_DT)
    b = np.ascontiguousarray(base, dtype=BASE_DT)
    w = np.zeros(18, dtype=np.uint64)
    f = np.zeros(7, dtype=np.float64)
    rc = _load().oracle_totals(s.ctypes.data, b.ctypes.data, len(s), T, plat.ctypes.data,
                               w.ctypes.data, f.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_totals rejected its arguments")
    return w, f


def offline_bound(x, lam: float, plat=None, full_grid: bool = False) -> np.ndarray:
    """NEXT f2 DP for one trace: {cost, energy, time} of the schedule that
    minimises energy + lam * time under model M (magus_oracle.cpp)."""
    x = np.ascontiguousarray(x, dtype=np.float32).reshape(-1)
    plat = platform() if plat is None else np.ascontiguousarray(plat, dtype=PLATFORM_DT)
    out = np.zeros(3, np.float64)
    rc = _load().oracle_offline_bound(x.ctypes.data, len(x), plat.ctypes.data, float(lam), int(full_grid),
                                      out.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_offline_bound rejected its arguments")
    return out


def pareto_front(energy, time) -> np.ndarray:
    """Sec. 6.4 (Fig. 7): configs not dominated in (energy, runtime); plain O(C^2)."""
    e, t = np.asarray(energy, np.float64), np.asarray(time, np.float64)
    on = np.ones(len(e), bool)
    for i in range(len(e)):
        for j in range(len(e)):
            if e[j] <= e[i] and t[j] <= t[i] and (e[j] < e[i] or t[j] < t[i]):
                on[i] = False
                break
    return on


def energy_sum(summary_row: np.ndarray) -> float:
    s = np.ascontiguousarray(summary_row, dtype=SUMMARY_DT)
    return float(_load().oracle_energy_sum(s.ctypes.data, len(s)))


def sweep_best(viol, energy) -> tuple[int, bool]:
    v = np.ascontiguousarray(viol, dtype=np.uint64)
    e = np.ascontiguousarray(energy, dtype=np.float64)
    b = np.zeros(1, dtype=np.int32)
    rc = _load().oracle_sweep_best(v.ctypes.data, e.ctypes.data, len(v), b.ctypes.data)
    return int(b[0]), rc == 0


def decision_words(dec: np.ndarray, r_min: int) -> np.ndarray:
    """Pack oracle decisions [..., T] into the library's 32-step words
    [..., ceil(T/32)] (bit t%32 = dec[t] == r_min).  Plain bit packing."""
    T = dec.shape[-1]
    nw = (T + 31) // 32
    bits = (dec == r_min).astype(np.uint64)
    pad = nw * 32 - T
    if pad:
        bits = np.concatenate([bits, np.zeros(bits.shape[:-1] + (pad,), np.uint64)], axis=-1)
    bits = bits.reshape(bits.shape[:-1] + (nw, 32))
    weights = (np.uint64(1) << np.arange(32, dtype=np.uint64))
    return (bits * weights).sum(axis=-1).astype(np.uint32)
