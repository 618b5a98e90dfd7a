"""Python binding of libmagus (include/magus.h): argument marshalling only.

Every step of the replay runs in the CUDA kernels of ``libmagus.so``; this
module converts torch tensors to raw pointers and structs, and fails loudly if
the library is missing (there is no CPU fallback).  PyTorch is used for device
memory, streams and process groups only.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmagus.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing; run `python __graft_entry__.py` (no CPU fallback)")
_lib = ctypes.CDLL(LIB_PATH)

# ---- constants (mirror include/magus.h) ----
OK, ERR_INVALID_ARG, ERR_NOT_INITIALIZED, ERR_CUDA, ERR_NCCL, ERR_OOM, ERR_UNSUPPORTED, ERR_NO_FEASIBLE = range(8)
POLICY_PAPER_DEFAULT, POLICY_PAPER_PARETO = 0, 1
PLATFORM_INTEL_A100, PLATFORM_INTEL_MAX1550 = 0, 1
GEN_MIX, GEN_ADVERSARIAL = 0, 1
OPT_KERNEL, OPT_SEGMENTS, OPT_TIMING, OPT_WAVES, OPT_BUNDLE, OPT_SPEC_WARM, OPT_TRACE, OPT_NARROW = 0, 1, 2, 3, 4, 5, 6, 7
OPT_FAMILY = 8
OPT_WALK1 = 9
KERNEL_AUTO, KERNEL_REFERENCE, KERNEL_STREAM, KERNEL_SEQUENTIAL, KERNEL_WALK, KERNEL_SPEC = 0, 1, 2, 3, 4, 5
TOT_WORDS = 18
TOT_NAMES = ["n_traces", "n_viol", "events", "hi_rounds", "msr_writes", "changes", "min_dec",
             "min_int", "qmin_lo", "qmin_hi", "qmax_lo", "qmax_hi", "qbase_lo", "qbase_hi",
             "n_steps", "burst_base", "burst_magus", "reserved"]


class Policy(ctypes.Structure):
    _fields_ = [("window", ctypes.c_int32), ("history", ctypes.c_int32), ("deriv_len", ctypes.c_double),
                ("tau_inc", ctypes.c_double), ("tau_dec", ctypes.c_double), ("t_hi", ctypes.c_double),
                ("variant", ctypes.c_int32), ("step", ctypes.c_int32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class Platform(ctypes.Structure):
    _fields_ = [("ratio_min", ctypes.c_int32), ("ratio_max", ctypes.c_int32), ("dt_s", ctypes.c_double),
                ("bw_max_mbs", ctypes.c_double), ("beta", ctypes.c_double), ("p_other_w", ctypes.c_double),
                ("p_unc_min_w", ctypes.c_double), ("p_unc_max_w", ctypes.c_double),
                ("e_switch_j", ctypes.c_double), ("t_switch_s", ctypes.c_double),
                ("slowdown_bound", ctypes.c_double), ("burst_mbs", ctypes.c_double)]


class Derived(ctypes.Structure):
    _fields_ = [("energy_j", ctypes.c_double), ("time_s", ctypes.c_double), ("base_energy_j", ctypes.c_double),
                ("base_time_s", ctypes.c_double), ("saving", ctypes.c_double), ("slowdown", ctypes.c_double),
                ("n_viol", ctypes.c_int64), ("n_traces", ctypes.c_int64), ("jaccard", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class Choice(ctypes.Structure):
    _fields_ = [("best", ctypes.c_int32), ("feasible", ctypes.c_int32), ("row", Derived)]


class PolicyConsts(ctypes.Structure):
    _fields_ = [("delta_inc", ctypes.c_double), ("delta_dec", ctypes.c_double), ("k_hi", ctypes.c_int32),
                ("reserved", ctypes.c_int32)]


class PlatformConsts(ctypes.Structure):
    _fields_ = [("x_stretch_min", ctypes.c_float), ("x_stretch_max", ctypes.c_float),
                ("inv_cap_min", ctypes.c_double), ("inv_cap_max", ctypes.c_double),
                ("p_min_w", ctypes.c_double), ("p_max_w", ctypes.c_double)]


class Stats(ctypes.Structure):
    _fields_ = [("launches_total", ctypes.c_int64), ("main_launches", ctypes.c_int64),
                ("main_ms_total", ctypes.c_double), ("last_segments", ctypes.c_int64),
                ("last_kernel", ctypes.c_int64), ("last_grid", ctypes.c_int64),
                ("last_reruns", ctypes.c_int64), ("last_family", ctypes.c_int64)]


SUMMARY_DT = np.dtype([("n_events", "<i8"), ("n_hi_rounds", "<i8"), ("n_msr_writes", "<i8"),
                       ("n_changes", "<i8"), ("n_min_dec", "<i8"), ("n_min_int", "<i8"), ("q_min", "<u8"),
                       ("q_max", "<u8"), ("digest", "<u8"), ("time_s", "<f8"), ("energy_j", "<f8"),
                       ("slowdown", "<f8"), ("viol", "<i4"), ("reserved", "<i4"), ("n_burst_base", "<i8"),
                       ("n_burst_magus", "<i8")])
BASE_DT = np.dtype([("q_base", "<u8"), ("time_s", "<f8"), ("energy_j", "<f8"), ("reserved", "<u8")])
assert SUMMARY_DT.itemsize == 120 and BASE_DT.itemsize == 32

_vp, _i32, _i64, _u64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
_lib.magus_init.argtypes = [ctypes.POINTER(_vp), ctypes.c_int, _vp, ctypes.POINTER(Platform)]
_lib.magus_destroy.argtypes = [_vp]
_lib.magus_set_stream.argtypes = [_vp, _vp]
_lib.magus_status_string.restype = ctypes.c_char_p
_lib.magus_status_string.argtypes = [ctypes.c_int]
_lib.magus_last_error.restype = ctypes.c_char_p
_lib.magus_last_error.argtypes = [_vp]
_lib.magus_abi_version.restype = _i32
_lib.magus_policy_preset.argtypes = [_i32, ctypes.POINTER(Policy)]
_lib.magus_platform_preset.argtypes = [_i32, ctypes.POINTER(Platform)]
_lib.magus_grid_sweep256.argtypes = [ctypes.POINTER(Policy)]
_lib.magus_grid_fleet64.argtypes = [ctypes.POINTER(Policy)]
_lib.magus_replay.argtypes = [_vp, _vp, _i64, _i64, _i64, ctypes.POINTER(Policy), _i32, _vp, _vp, _vp, _vp]
_lib.magus_replay_host.argtypes = [_vp, _vp, _i64, _i64, _i64, ctypes.POINTER(Policy), _i32, _vp, _vp, _vp, _vp]
_lib.magus_replay_resume.argtypes = [_vp, _vp, _i64, _i64, _i64, _i64, _i64, ctypes.POINTER(Policy), _i32, _vp,
                                     _vp, _vp, _vp, _vp]
_lib.magus_resume_state_bytes.argtypes = [_i64, _i32, ctypes.POINTER(ctypes.c_size_t)]
_lib.magus_resume_halo.argtypes = [ctypes.POINTER(Policy), _i32, ctypes.POINTER(_i64)]
_lib.magus_replay_levels.argtypes = [_vp, _vp, _i64, _i64, _i64, ctypes.POINTER(Policy), _i32, _vp, _vp, _vp]
_lib.magus_offline_bound.argtypes = [_vp, _vp, _i64, _i64, _i64, _vp, _i32, _i32, _vp]
_lib.magus_sweep_best_async.argtypes = [_vp, _vp, _i32, _vp]
_lib.magus_totals_derive.argtypes = [_vp, _vp, ctypes.POINTER(Derived)]
_lib.magus_sweep_best.argtypes = [_vp, _vp, _i32, ctypes.POINTER(_i32), ctypes.POINTER(Derived)]
_lib.magus_gen_traces.argtypes = [_vp, _u64, _i64, _i64, _i64, _i64, _i32, _vp]
_lib.magus_gen_traces_resume.argtypes = [_vp, _u64, _i64, _i64, _i64, _i64, _i64, _i32, _vp, _vp]
_lib.magus_gen_state_bytes.argtypes = [_i64, ctypes.POINTER(ctypes.c_size_t)]
_lib.magus_set_option.argtypes = [_vp, _i32, _i64]
_lib.magus_policy_inspect.argtypes = [ctypes.POINTER(Policy), ctypes.POINTER(PolicyConsts)]
_lib.magus_platform_inspect.argtypes = [ctypes.POINTER(Platform), ctypes.POINTER(PlatformConsts)]
_lib.magus_get_stats.argtypes = [_vp, ctypes.POINTER(Stats)]
_lib.magus_derive_host.argtypes = [ctypes.POINTER(Platform), _vp, ctypes.POINTER(Derived)]
_lib.magus_pareto_front.argtypes = [_vp, _vp, _i32, _vp, ctypes.POINTER(_i32)]
_lib.magus_pareto_front_host.argtypes = [ctypes.POINTER(Platform), _vp, _i32, _vp, ctypes.POINTER(_i32)]
_lib.magus_sweep_best_host.argtypes = [ctypes.POINTER(Platform), _vp, _i32, ctypes.POINTER(_i32),
                                       ctypes.POINTER(Derived)]
_lib.magus_reset_stats.argtypes = [_vp]
_lib.magus_get_trace.argtypes = [_vp, _vp, _i64, ctypes.POINTER(_i64)]
_lib.magus_comm_unique_id.argtypes = [_vp]
_lib.magus_comm_init.argtypes = [_vp, _vp, _i32, _i32]
_lib.magus_allreduce_totals.argtypes = [_vp, _vp, _i32]
for _f in ("magus_init", "magus_destroy", "magus_set_stream", "magus_policy_preset", "magus_platform_preset",
           "magus_grid_sweep256", "magus_grid_fleet64", "magus_replay", "magus_replay_host",
           "magus_totals_derive", "magus_sweep_best", "magus_gen_traces", "magus_set_option",
           "magus_get_stats", "magus_reset_stats", "magus_policy_inspect", "magus_platform_inspect", "magus_derive_host",
           "magus_sweep_best_host", "magus_pareto_front", "magus_pareto_front_host",
           "magus_replay_levels", "magus_offline_bound", "magus_sweep_best_async",
           "magus_comm_unique_id", "magus_comm_init", "magus_allreduce_totals", "magus_get_trace"):
    getattr(_lib, _f).restype = ctypes.c_int

EXPORTED = ["magus_init", "magus_destroy", "magus_set_stream", "magus_status_string", "magus_last_error",
            "magus_abi_version", "magus_policy_preset", "magus_platform_preset", "magus_grid_sweep256",
            "magus_grid_fleet64", "magus_replay", "magus_replay_host", "magus_totals_derive",
            "magus_sweep_best", "magus_gen_traces", "magus_set_option", "magus_get_stats",
            "magus_reset_stats", "magus_policy_inspect", "magus_platform_inspect", "magus_derive_host",
            "magus_sweep_best_host", "magus_pareto_front", "magus_pareto_front_host",
            "magus_replay_levels", "magus_offline_bound", "magus_sweep_best_async",
            "magus_replay_resume", "magus_resume_state_bytes", "magus_resume_halo",
            "magus_gen_traces_resume", "magus_gen_state_bytes",
            "magus_comm_unique_id", "magus_comm_init", "magus_allreduce_totals", "magus_get_trace"]
COMM_ID_BYTES = 128
VARIANT_CLOSED_LOOP, VARIANT_GRADUAL = 1, 2


class MagusError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        msg = _lib.magus_status_string(status).decode()
        super().__init__(f"{msg}: {detail}" if detail else msg)


def comm_unique_id() -> bytes:
    """The optional native NCCL path: rank 0 creates the id (128 bytes) and
    ships it to every rank by its own means (e.g. a torch.distributed
    broadcast or a file)."""
    buf = ctypes.create_string_buffer(COMM_ID_BYTES)
    st = _lib.magus_comm_unique_id(ctypes.cast(buf, _vp))
    if st:
        raise MagusError(st, "comm_unique_id")
    return buf.raw


def abi_version() -> int:
    return int(_lib.magus_abi_version())


def policy_preset(pid: int = POLICY_PAPER_DEFAULT) -> Policy:
    p = Policy()
    st = _lib.magus_policy_preset(pid, ctypes.byref(p))
    if st:
        raise MagusError(st)
    return p


def platform_preset(pid: int = PLATFORM_INTEL_A100) -> Platform:
    p = Platform()
    st = _lib.magus_platform_preset(pid, ctypes.byref(p))
    if st:
        raise MagusError(st)
    return p


def grid_sweep256() -> list[Policy]:
    arr = (Policy * 256)()
    _lib.magus_grid_sweep256(arr)
    return list(arr)


def grid_fleet64() -> list[Policy]:
    arr = (Policy * 64)()
    _lib.magus_grid_fleet64(arr)
    return list(arr)


def resume_halo(policies) -> int:
    """Rows before t_start a resume chunk must carry (multiple of 32)."""
    arr, C = _policy_array(policies)
    r = _i64()
    st = _lib.magus_resume_halo(arr, C, ctypes.byref(r))
    if st:
        raise MagusError(st, "resume_halo")
    return r.value


def policy_inspect(p: Policy) -> dict:
    o = PolicyConsts()
    st = _lib.magus_policy_inspect(ctypes.byref(p), ctypes.byref(o))
    if st:
        raise MagusError(st, "policy_inspect")
    return {"delta_inc": o.delta_inc, "delta_dec": o.delta_dec, "k_hi": o.k_hi}


def platform_inspect(p: Platform) -> dict:
    o = PlatformConsts()
    st = _lib.magus_platform_inspect(ctypes.byref(p), ctypes.byref(o))
    if st:
        raise MagusError(st, "platform_inspect")
    return {k: getattr(o, k) for k, _ in o._fields_}


def derive_host(totals_row, platform: Platform | None = None) -> dict:
    """Fleet fp64 quantities of one config from its integer totals (no GPU)."""
    plat = platform if platform is not None else platform_preset()
    w = np.ascontiguousarray(np.asarray(totals_row).view(np.uint64).reshape(TOT_WORDS))
    d = Derived()
    st = _lib.magus_derive_host(ctypes.byref(plat), _vp(w.ctypes.data), ctypes.byref(d))
    if st:
        raise MagusError(st, "derive_host")
    return d.as_dict()


def sweep_best_host(totals, platform: Platform | None = None) -> tuple[int, dict, bool]:
    """(best, derived row, feasible) from host totals [C, TOT_WORDS=18] (no GPU)."""
    plat = platform if platform is not None else platform_preset()
    w = np.ascontiguousarray(np.asarray(totals).view(np.uint64).reshape(-1, TOT_WORDS))
    best, d = _i32(), Derived()
    st = _lib.magus_sweep_best_host(ctypes.byref(plat), _vp(w.ctypes.data), len(w), ctypes.byref(best),
                                    ctypes.byref(d))
    if st not in (OK, ERR_NO_FEASIBLE):
        raise MagusError(st, "sweep_best_host")
    return int(best.value), d.as_dict(), st == OK


def pareto_front_host(totals, platform: Platform | None = None) -> np.ndarray:
    """Sec. 6.4 energy/runtime Pareto front over configs (host totals [C, W])."""
    plat = platform if platform is not None else platform_preset()
    w = np.ascontiguousarray(np.asarray(totals).view(np.uint64).reshape(-1, TOT_WORDS))
    on = np.zeros(len(w), np.int32)
    nf = _i32()
    st = _lib.magus_pareto_front_host(ctypes.byref(plat), _vp(w.ctypes.data), len(w), _vp(on.ctypes.data),
                                      ctypes.byref(nf))
    if st:
        raise MagusError(st, "pareto_front_host")
    return on.astype(bool)


def make_policy(W=10, H=10, L=None, tau_inc=200.0, tau_dec=-500.0, t_hi=0.4, variant=0, step=None) -> Policy:
    step = (1 if variant & VARIANT_GRADUAL else 0) if step is None else step
    return Policy(W, H, float(W if L is None else L), tau_inc, tau_dec, t_hi, variant, step)


def _policy_array(policies) -> tuple[ctypes.Array, int]:
    pols = list(policies)
    arr = (Policy * len(pols))(*pols)
    return arr, len(pols)


@dataclass
class ReplayResult:
    summary: object | None      # torch.uint8 [C, N, SUMMARY_DT.itemsize=120] (use summary_numpy())
    base: object | None         # torch.uint8 [N, 32]
    decisions: object | None    # torch.int32 view of uint32 [C, ceil(T/32), N]
    totals: object | None       # torch.int64 view of uint64 [C, TOT_WORDS=18]
    n_traces: int
    n_configs: int

    def summary_numpy(self) -> np.ndarray:
        return self.summary.cpu().numpy().view(SUMMARY_DT).reshape(self.n_configs, self.n_traces)

    def base_numpy(self) -> np.ndarray:
        return self.base.cpu().numpy().view(BASE_DT).reshape(self.n_traces)

    def totals_numpy(self) -> np.ndarray:
        return self.totals.cpu().numpy().view(np.uint64).reshape(self.n_configs, TOT_WORDS)

    def decisions_numpy(self) -> np.ndarray:
        return self.decisions.cpu().numpy().view(np.uint32)


def _check_out(out: ReplayResult, N: int, C: int, nw: int, dev, want_summary: bool, want_base: bool,
               want_decisions: bool, want_totals: bool) -> None:
    """Caller-supplied output buffers must match this call exactly: the kernels
    write [C, N, ...] / [C, nw, N] / [C, TOT_WORDS] without bounds checks."""
    torch = __import__("torch")
    spec = (("summary", want_summary, (C, N, SUMMARY_DT.itemsize), torch.uint8),
            ("base", want_base, (N, 32), torch.uint8),
            ("decisions", want_decisions, (C, nw, N), torch.int32),
            ("totals", want_totals, (C, TOT_WORDS), torch.int64))
    for name, want, shape, dt in spec:
        t = getattr(out, name)
        if t is None:
            if want:
                raise ValueError(f"replay(out=...): {name} requested but out.{name} is None")
            continue
        if tuple(t.shape) != shape or t.dtype != dt or t.device != dev or not t.is_contiguous():
            raise ValueError(f"replay(out=...): out.{name} is {tuple(t.shape)} {t.dtype} on {t.device}, "
                             f"this call needs {shape} {dt} on {dev} (contiguous)")
    if out.n_traces != N or out.n_configs != C:
        raise ValueError(f"replay(out=...): result is for N={out.n_traces}, C={out.n_configs}; call has N={N}, C={C}")


class Context:
    """A libmagus context bound to one CUDA device and a torch stream."""

    def __init__(self, device: int = 0, platform: Platform | None = None, stream=None):
        import torch
        self._torch = torch
        self.device = device
        self.platform = platform if platform is not None else platform_preset()
        self._stream = stream if stream is not None else torch.cuda.current_stream(device)
        h = _vp()
        st = _lib.magus_init(ctypes.byref(h), device, _vp(self._stream.cuda_stream), ctypes.byref(self.platform))
        if st:
            raise MagusError(st, "magus_init")
        self._h = h

    # -- plumbing --
    def close(self):
        if getattr(self, "_h", None):
            _lib.magus_destroy(self._h)
            self._h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, st: int, what: str):
        if st and st != ERR_NO_FEASIBLE:
            raise MagusError(st, f"{what}: {_lib.magus_last_error(self._h).decode()}")

    def set_stream(self, stream):
        self._stream = stream
        self._check(_lib.magus_set_stream(self._h, _vp(stream.cuda_stream)), "set_stream")

    def set_option(self, key: int, value: int):
        self._check(_lib.magus_set_option(self._h, key, int(value)), "set_option")

    def stats(self) -> dict:
        s = Stats()
        self._check(_lib.magus_get_stats(self._h, ctypes.byref(s)), "get_stats")
        return {k: getattr(s, k) for k, _ in s._fields_}

    def reset_stats(self):
        self._check(_lib.magus_reset_stats(self._h), "reset_stats")

    def trace(self) -> np.ndarray:
        """Per-CTA timeline of the last traced stream replay (OPT_TRACE):
        uint64 [CTAs, 8] = start, scan end, look-back end, end (ns), SM,
        segment, trace group, finalised-the-group flag."""
        cap = self.stats()["last_grid"]
        out = np.zeros((max(cap, 1), 8), np.uint64)
        n = _i64()
        self._check(_lib.magus_get_trace(self._h, _vp(out.ctypes.data), cap, ctypes.byref(n)), "get_trace")
        return out[:n.value]

    # -- the API --
    def gen_traces(self, seed: int, n_traces: int, n_steps: int, kind: int = GEN_MIX, id0: int = 0,
                   ld: int | None = None, out=None):
        torch = self._torch
        ld = n_traces if ld is None else ld
        if out is None:
            out = torch.zeros((n_steps, ld), dtype=torch.float32, device=f"cuda:{self.device}")
        st = _lib.magus_gen_traces(self._h, seed & 0xFFFFFFFFFFFFFFFF, id0, n_traces, n_steps, ld, kind,
                                   _vp(out.data_ptr()))
        self._check(st, "gen_traces")
        return out

    def gen_state(self, n_traces: int):
        """Device phase-machine state for gen_traces_resume."""
        nb = ctypes.c_size_t()
        if _lib.magus_gen_state_bytes(n_traces, ctypes.byref(nb)):
            raise MagusError(1, "gen_state_bytes")
        return self._torch.empty(((nb.value + 7) // 8,), dtype=self._torch.int64, device=f"cuda:{self.device}")

    def gen_traces_resume(self, seed: int, n_traces: int, t0: int, n_rows: int, state, out, kind: int = GEN_MIX,
                          id0: int = 0):
        """Intervals [t0, t0 + n_rows) of the traces into out rows 0.. (out: [>= n_rows, ld])."""
        st = _lib.magus_gen_traces_resume(self._h, seed & 0xFFFFFFFFFFFFFFFF, id0, n_traces, t0, n_rows,
                                          out.stride(0), kind, _vp(state.data_ptr()), _vp(out.data_ptr()))
        self._check(st, "gen_traces_resume")
        return out

    def replay(self, traces, policies, n_traces: int | None = None, want_summary: bool = True,
               want_base: bool = True, want_decisions: bool = False, want_totals: bool = True,
               out: ReplayResult | None = None) -> ReplayResult:
        """traces: CUDA float32 tensor [T, ld], time-major (row stride ld)."""
        torch = self._torch
        assert traces.is_cuda and traces.dtype == torch.float32 and traces.dim() == 2
        assert traces.stride(1) == 1
        T, ld = traces.shape[0], traces.stride(0)
        N = traces.shape[1] if n_traces is None else n_traces
        arr, C = _policy_array(policies)
        dev = traces.device
        if out is None:
            nw = (T + 31) // 32
            out = ReplayResult(
                summary=torch.empty((C, N, SUMMARY_DT.itemsize), dtype=torch.uint8, device=dev)
                if want_summary else None,
                base=torch.empty((N, 32), dtype=torch.uint8, device=dev) if want_base else None,
                decisions=torch.empty((C, nw, N), dtype=torch.int32, device=dev) if want_decisions else None,
                totals=torch.empty((C, TOT_WORDS), dtype=torch.int64, device=dev) if want_totals else None,
                n_traces=N, n_configs=C)
        else:
            _check_out(out, N, C, (T + 31) // 32, dev, want_summary, want_base, want_decisions, want_totals)
        p = lambda t: _vp(t.data_ptr()) if t is not None else None  # noqa: E731
        st = _lib.magus_replay(self._h, _vp(traces.data_ptr()), N, T, ld, arr, C, p(out.summary), p(out.base),
                               p(out.decisions), p(out.totals))
        self._check(st, "replay")
        return out

    def resume_state(self, n_traces: int, policies):
        """Zeroed device resume state (t = 0) for replay_resume."""
        _, C = _policy_array(policies)
        nb = ctypes.c_size_t()
        st = _lib.magus_resume_state_bytes(n_traces, C, ctypes.byref(nb))
        self._check(st, "resume_state_bytes")
        return self._torch.zeros(((nb.value + 7) // 8,), dtype=self._torch.int64, device=f"cuda:{self.device}")

    def replay_resume(self, traces, policies, state, t_base: int, t_start: int, n_traces: int | None = None,
                      want_summary: bool = True, want_base: bool = True, want_decisions: bool = False,
                      want_totals: bool = True) -> ReplayResult:
        """One time chunk: traces[r] = global interval t_base + r; decides
        [t_start, t_base + rows); outputs cover the prefix [0, t_base + rows)."""
        torch = self._torch
        assert traces.is_cuda and traces.dtype == torch.float32 and traces.dim() == 2
        assert traces.stride(1) == 1
        R, ld = traces.shape[0], traces.stride(0)
        N = traces.shape[1] if n_traces is None else n_traces
        arr, C = _policy_array(policies)
        dev = traces.device
        nw = (t_base + R - t_start + 31) // 32
        out = ReplayResult(
            summary=torch.empty((C, N, SUMMARY_DT.itemsize), dtype=torch.uint8, device=dev) if want_summary else None,
            base=torch.empty((N, 32), dtype=torch.uint8, device=dev) if want_base else None,
            decisions=torch.empty((C, max(nw, 0), N), dtype=torch.int32, device=dev) if want_decisions else None,
            totals=torch.empty((C, TOT_WORDS), dtype=torch.int64, device=dev) if want_totals else None,
            n_traces=N, n_configs=C)
        p = lambda t: _vp(t.data_ptr()) if t is not None else None  # noqa: E731
        st = _lib.magus_replay_resume(self._h, _vp(traces.data_ptr()), N, R, ld, t_base, t_start, arr, C,
                                      _vp(state.data_ptr()), p(out.summary), p(out.base), p(out.decisions),
                                      p(out.totals))
        self._check(st, "replay_resume")
        return out

    def replay_levels(self, traces, policies, n_traces: int | None = None, want_totals: bool = True):
        """Per-interval uncore ratios (uint8 [C, T, N]) + summaries (+ totals):
        walk kernels (open loop) or the sequential kernel (closed loop);
        required for the multi-level f4 variant."""
        torch = self._torch
        assert traces.is_cuda and traces.dtype == torch.float32 and traces.stride(1) == 1
        T, ld = traces.shape[0], traces.stride(0)
        N = traces.shape[1] if n_traces is None else n_traces
        arr, C = _policy_array(policies)
        dev = traces.device
        levels = torch.empty((C, T, N), dtype=torch.uint8, device=dev)
        res = ReplayResult(summary=torch.empty((C, N, SUMMARY_DT.itemsize), dtype=torch.uint8, device=dev),
                           base=None, decisions=None,
                           totals=torch.empty((C, TOT_WORDS), dtype=torch.int64, device=dev) if want_totals else None,
                           n_traces=N, n_configs=C)
        st = _lib.magus_replay_levels(self._h, _vp(traces.data_ptr()), N, T, ld, arr, C, _vp(levels.data_ptr()),
                                      _vp(res.summary.data_ptr()),
                                      _vp(res.totals.data_ptr()) if want_totals else None)
        self._check(st, "replay_levels")
        return levels, res

    def offline_bound(self, traces, lambdas, full_grid: bool = False, n_traces: int | None = None):
        """NEXT f2: float64 tensor [N, len(lambdas), 3] = {cost, energy, time}
        of the schedule minimising energy + lambda * time (magus_offline_bound)."""
        torch = self._torch
        assert traces.is_cuda and traces.dtype == torch.float32 and traces.stride(1) == 1
        T, ld = traces.shape[0], traces.stride(0)
        N = traces.shape[1] if n_traces is None else n_traces
        lam = np.ascontiguousarray(lambdas, dtype=np.float64)
        out = torch.empty((N, len(lam), 3), dtype=torch.float64, device=traces.device)
        st = _lib.magus_offline_bound(self._h, _vp(traces.data_ptr()), N, T, ld, _vp(lam.ctypes.data), len(lam),
                                      int(full_grid), _vp(out.data_ptr()))
        self._check(st, "offline_bound")
        return out

    def replay_host(self, traces: np.ndarray, policies, n_traces: int | None = None, want_summary=True,
                    want_base=True, want_decisions=False, want_totals=True):
        """End-to-end path: host arrays in, host arrays out (H2D/D2H inside)."""
        assert traces.dtype == np.float32 and traces.ndim == 2 and traces.strides[1] == 4
        T, ld = traces.shape[0], traces.strides[0] // 4
        N = traces.shape[1] if n_traces is None else n_traces
        arr, C = _policy_array(policies)
        nw = (T + 31) // 32
        s = np.empty((C, N), SUMMARY_DT) if want_summary else None
        b = np.empty(N, BASE_DT) if want_base else None
        d = np.empty((C, nw, N), np.uint32) if want_decisions else None
        t = np.empty((C, TOT_WORDS), np.uint64) if want_totals else None
        p = lambda a: _vp(a.ctypes.data) if a is not None else None  # noqa: E731
        st = _lib.magus_replay_host(self._h, _vp(traces.ctypes.data), N, T, ld, arr, C, p(s), p(b), p(d), p(t))
        self._check(st, "replay_host")
        return s, b, d, t

    def totals_derive(self, totals_row) -> dict:
        w = np.ascontiguousarray(np.asarray(totals_row).view(np.uint64).reshape(TOT_WORDS))
        d = Derived()
        self._check(_lib.magus_totals_derive(self._h, _vp(w.ctypes.data), ctypes.byref(d)), "totals_derive")
        return d.as_dict()

    def pareto_front(self, totals) -> np.ndarray:
        """Sec. 6.4 front over the configs from DEVICE totals [C, W]."""
        C = totals.shape[0]
        on = np.zeros(C, np.int32)
        nf = _i32()
        st = _lib.magus_pareto_front(self._h, _vp(totals.data_ptr()), C, _vp(on.ctypes.data), ctypes.byref(nf))
        self._check(st, "pareto_front")
        return on.astype(bool)

    def sweep_best_async(self, totals, out=None):
        """Enqueue the device-side choice (one D2H copy of a magus_choice into
        a pinned buffer, returned); read it with sweep_result() after a sync."""
        torch = self._torch
        if out is None:
            out = torch.zeros(ctypes.sizeof(Choice), dtype=torch.uint8, pin_memory=True)
        st = _lib.magus_sweep_best_async(self._h, _vp(totals.data_ptr()), totals.shape[0], _vp(out.data_ptr()))
        self._check(st, "sweep_best_async")
        return out

    @staticmethod
    def sweep_result(out) -> tuple[int, dict, bool]:
        ch = Choice.from_buffer_copy(out.numpy().tobytes())
        return int(ch.best), ch.row.as_dict(), bool(ch.feasible)

    def comm_init(self, uid: bytes, nranks: int, rank: int):
        """magus_comm_init: this context's NCCL communicator (collective)."""
        assert len(uid) == COMM_ID_BYTES
        buf = ctypes.create_string_buffer(uid, COMM_ID_BYTES)
        self._check(_lib.magus_comm_init(self._h, ctypes.cast(buf, _vp), nranks, rank), "comm_init")

    def allreduce_totals(self, totals):
        """magus_allreduce_totals: in-place uint64 SUM over the ranks on this
        context's stream (a no-op without comm_init)."""
        assert totals.is_cuda and totals.dtype == self._torch.int64 and totals.shape[-1] == TOT_WORDS
        self._check(_lib.magus_allreduce_totals(self._h, _vp(totals.data_ptr()), totals.shape[0]),
                    "allreduce_totals")
        return totals

    def sweep_best(self, totals) -> tuple[int, dict, bool]:
        """totals: CUDA int64 tensor [C, TOT_WORDS=18] (summed over ranks if sharded).
        Returns (best index, derived row, feasible)."""
        C = totals.shape[0]
        best = _i32()
        d = Derived()
        st = _lib.magus_sweep_best(self._h, _vp(totals.data_ptr()), C, ctypes.byref(best), ctypes.byref(d))
        self._check(st, "sweep_best")
        return int(best.value), d.as_dict(), st == OK
