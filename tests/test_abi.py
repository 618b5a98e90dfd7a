"""C-ABI surface checks that need no GPU: the library loads, exports every
function include/magus.h declares, and its host-only calls behave."""
import ctypes
import functools
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "magus.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(magus_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    import paper_conf_sc_zhengspl25_b200 as m
    names = _declared()
    assert "magus_replay" in names and "magus_sweep_best" in names and "magus_init" in names
    lib = ctypes.CDLL(m.LIB_PATH)
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    assert set(m.EXPORTED) == set(names)
    assert m.abi_version() == 1


def test_presets_cite_the_paper_values():
    import paper_conf_sc_zhengspl25_b200 as m
    d = m.policy_preset(m.POLICY_PAPER_DEFAULT)
    assert (d.window, d.history, d.deriv_len, d.tau_inc, d.tau_dec, d.t_hi) == (10, 10, 10.0, 200.0, -500.0, 0.4)
    assert m.policy_preset(m.POLICY_PAPER_PARETO).tau_inc == 300.0
    a = m.platform_preset(m.PLATFORM_INTEL_A100)
    assert (a.ratio_min, a.ratio_max, a.dt_s, a.p_unc_max_w, a.slowdown_bound) == (8, 22, 0.2, 82.0, 0.05)
    assert m.platform_preset(m.PLATFORM_INTEL_MAX1550).ratio_max == 25
    with pytest.raises(m.MagusError):
        m.policy_preset(7)


def test_grids_index_convention():
    import paper_conf_sc_zhengspl25_b200 as m
    g = m.grid_sweep256()
    d = g[165]
    assert (d.window, d.tau_inc, d.tau_dec, d.t_hi) == (10, 200.0, -500.0, 0.4)
    assert g[166].tau_inc == 300.0
    seen = {(p.window, p.tau_inc, p.tau_dec, p.t_hi) for p in g}
    assert len(seen) == 256 and all(p.deriv_len == p.window and p.history == 10 for p in g)
    f = m.grid_fleet64()
    assert (f[37].tau_inc, f[37].tau_dec, f[37].t_hi) == (200.0, -500.0, 0.4) and f[38].tau_inc == 300.0


def test_init_without_gpu_fails_cleanly():
    import paper_conf_sc_zhengspl25_b200 as m
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    h = ctypes.c_void_p()
    p = m.platform_preset()
    st = m._lib.magus_init(ctypes.byref(h), 0, None, ctypes.byref(p))
    assert st == m.ERR_CUDA and not h.value


def test_null_context_is_rejected():
    import paper_conf_sc_zhengspl25_b200 as m
    assert m._lib.magus_replay(None, None, 1, 1, 1, None, 1, None, None, None, None) == m.ERR_NOT_INITIALIZED
    assert m._lib.magus_last_error(None) == b"NULL context"
    assert m._lib.magus_status_string(m.ERR_NO_FEASIBLE) == b"no feasible config"


@functools.lru_cache(maxsize=2)
def _sass(tool: str, lib: str, mtime: float) -> str:
    import subprocess
    return subprocess.run([tool, "-sass", lib], capture_output=True, text=True, check=True).stdout


def _consumer_loop_local_ops(sass: str):
    """Local-memory (spill) instructions inside the consumer's word loop: the
    largest backward branch whose target sits just before an mbarrier wait."""
    ins = []
    for line in sass.split("\n"):
        mm = re.search(r"/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
        if mm:
            ins.append((int(mm.group(1), 16), mm.group(2).strip()))
    waits = [a for a, t in ins if "TRYWAIT" in t]
    loops = []
    for a, t in ins:
        mm = re.search(r"BRA (0x[0-9a-f]+)", t)
        if mm and int(mm.group(1), 16) < a:
            tgt = int(mm.group(1), 16)
            if any(tgt <= x <= tgt + 0x200 for x in waits):
                loops.append((tgt, a))
    assert loops, "consumer loop not found"
    lo, hi = max(loops, key=lambda x: x[1] - x[0])
    return hi - lo, [hex(a) for a, t in ins if lo <= a <= hi and ("STL" in t or "LDL" in t)]


@pytest.mark.parametrize("inst,budget", [("ILi10ELi10ELi1ELb0ELi512E", 0), ("ILi10ELi10ELi4ELb0ELi128E", 2),
                                         ("ILi4ELi10ELi4ELb0ELi128E", 2)])
def test_hot_kernels_do_not_spill_in_the_word_loop(inst, budget):
    """The paper-default kernel (W = H = 10, one config per thread, 512-trace
    CTAs) keeps its
    whole word loop in registers; the 4-config bundle kernels of SWEEP256 may
    reload at most two loop-invariant words per 32-step word (~1000
    instructions).  A few bytes spilled around the loop are harmless."""
    import shutil
    log = open(os.path.join(ROOT, "paper_conf_sc_zhengspl25_b200", "build", "ptxas.log")).read()
    blocks = [b for b in re.split(r"Compiling entry function", log) if "stream_kernel" + inst in b]
    assert blocks, f"stream_kernel{inst} missing from the build"
    sp = re.search(r"(\d+) bytes spill stores", blocks[0])
    assert sp and int(sp.group(1)) <= 16
    tool = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(tool) and not shutil.which("cuobjdump"):
        pytest.skip("cuobjdump unavailable")
    lib = os.path.join(ROOT, "paper_conf_sc_zhengspl25_b200", "libmagus.so")
    out = _sass(tool, lib, os.path.getmtime(lib))
    fn = [p for p in out.split("Function : ") if "stream_kernel" + inst in p.split("\n")[0]]
    assert fn
    size, local = _consumer_loop_local_ops(fn[0])
    assert size > 100 and len(local) <= budget, (size, local)


def test_binding_structs_match_header_sizes():
    import paper_conf_sc_zhengspl25_b200 as m
    assert ctypes.sizeof(m.Policy) == 48 and ctypes.sizeof(m.Platform) == 88
    assert m.SUMMARY_DT.itemsize == 120 and m.BASE_DT.itemsize == 32
    assert np.dtype(np.uint64).itemsize * m.TOT_WORDS == 144


def _nextafter(x, d):
    return float(np.nextafter(np.float64(x), np.float64(d)))


def test_threshold_inversion_equals_literal_division():
    """delta > delta_inc <=> RN(delta/L) > tau_inc (Alg. 1 l.3-4), checked at
    delta_inc and its neighbours, for awkward L and tau (Python's float
    division is IEEE round-to-nearest, like the paper's C++)."""
    import paper_conf_sc_zhengspl25_b200 as m
    rng = np.random.default_rng(3)
    cases = [(10.0, 200.0, -500.0), (3.0, 0.1, -0.7), (7.0, 1 / 3, -2 / 3), (0.3, 17.0, -19.0),
             (1e-300, 1e300, -1e300), (1e300, 1e-300, -1e-300), (5.0, 0.0, 0.0), (2.0, -3.0, 4.0)]
    cases += [(float(rng.uniform(0.01, 100)), float(rng.uniform(-1e4, 1e4)), float(rng.uniform(-1e4, 1e4)))
              for _ in range(300)]
    for L, ti, td in cases:
        c = m.policy_inspect(m.make_policy(W=10, L=L, tau_inc=ti, tau_dec=td))
        for base in (c["delta_inc"], c["delta_dec"], ti * L, td * L, 0.0, -0.0):
            for d in (_nextafter(_nextafter(base, -np.inf), -np.inf), _nextafter(base, -np.inf), base,
                      _nextafter(base, np.inf), _nextafter(_nextafter(base, np.inf), np.inf)):
                assert (d > c["delta_inc"]) == (d / L > ti), (L, ti, d)
                assert (d < c["delta_dec"]) == (d / L < td), (L, td, d)
        for d in (np.inf, -np.inf):
            assert (d > c["delta_inc"]) == (d / L > ti) and (d < c["delta_dec"]) == (d / L < td)


def test_k_hi_matches_alg2():
    import paper_conf_sc_zhengspl25_b200 as m
    for H in (1, 3, 7, 10, 32, 64):
        for t_hi in (0.1, 0.2, 0.3, 0.4, 0.5, 1 / 3, 0.99, 1.0, 1.01, 5.0):
            k = m.policy_inspect(m.make_policy(H=H, t_hi=t_hi))["k_hi"]
            want = next((s for s in range(H + 1) if s / H >= t_hi), H + 1)
            assert k == want


def test_stretch_threshold_equals_literal_predicate():
    import paper_conf_sc_zhengspl25_b200 as m
    for bw in (32000.0, 16384.0, 12345.678, 1e-3, 3e38):
        p = m.platform_preset()
        p.bw_max_mbs = bw
        c = m.platform_inspect(p)
        for thr, inv in ((c["x_stretch_min"], c["inv_cap_min"]), (c["x_stretch_max"], c["inv_cap_max"])):
            f = np.float32(thr)
            for x in (np.nextafter(f, np.float32(-np.inf)), f, np.nextafter(f, np.float32(np.inf))):
                assert (x > f) == (float(x) * inv > 1.0)


def test_resume_host_queries():
    """magus_resume_halo = the rows before t_start that fix p_t and the Alg. 2
    history (W + H - 1, rounded up to whole 32-step words); the state holds
    12 u64 accumulators and one u32 carry per (config, trace)."""
    import paper_conf_sc_zhengspl25_b200 as m
    assert m.resume_halo([m.make_policy()]) == 32                      # 10 + 10 - 1 = 19
    assert m.resume_halo([m.make_policy(W=16, H=10), m.make_policy(W=4, H=10)]) == 32  # 25
    assert m.resume_halo([m.make_policy(W=33, H=32)]) == 64            # 64
    assert m.resume_halo([m.make_policy(W=2, H=1)]) == 32              # 2 -> one word
    nb = ctypes.c_size_t()
    assert m._lib.magus_resume_state_bytes(1000, 3, ctypes.byref(nb)) == 0
    assert nb.value == 3 * 1000 * (12 * 8 + 4)
    assert m._lib.magus_resume_state_bytes(0, 3, ctypes.byref(nb)) != 0
    with pytest.raises(m.MagusError):
        m.resume_halo([m.make_policy(W=1)])
