"""Seeded synthetic memory-throughput traces (input generator only).

Host side of gen/magus_gen.h (built into gen/libmagus_gen.so by
``__graft_entry__.build()``).  The CUDA build of the same header lives in
libmagus (``magus_gen_traces``) and is bit-identical; tests check that.
No method arithmetic lives here: it is shared input plumbing.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libmagus_gen.so")
_lib = None

KIND_MIX = 0
KIND_ADVERSARIAL = 1
CLASS_NAMES = {0: "altis", 1: "ml", 2: "md", 3: "srad", 4: "adv_osc", 5: "adv_burst"}

# Seeds of the BASELINE.json configs.
SEEDS = {1: 0x4D41475553000001, 2: 0x4D41475553000002, 3: 0x4D41475553000003,
         4: 0x4D41475553000004, 5: 0x4D41475553000005}


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(_LIB_PATH)
        lib.magus_gen_traces_host.restype = ctypes.c_int
        lib.magus_gen_traces_host.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64,
                                              ctypes.c_int64, ctypes.c_int64, ctypes.c_int32,
                                              ctypes.c_void_p]
        lib.magus_gen_class_host.restype = ctypes.c_int32
        lib.magus_gen_class_host.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32]
        _lib = lib
    return _lib


def gen_traces(seed: int, n_traces: int, n_steps: int, kind: int = KIND_MIX, id0: int = 0,
               ld: int | None = None) -> np.ndarray:
    """Time-major float32 array [n_steps, ld] (columns >= n_traces are 0)."""
    ld = n_traces if ld is None else ld
    out = np.zeros((n_steps, ld), dtype=np.float32)
    rc = _load().magus_gen_traces_host(seed & 0xFFFFFFFFFFFFFFFF, id0, n_traces, n_steps, ld, kind,
                                       out.ctypes.data)
    if rc != 0:
        raise ValueError("magus_gen_traces_host: bad arguments")
    return out


def trace_class(seed: int, global_id: int, kind: int = KIND_MIX) -> int:
    return int(_load().magus_gen_class_host(seed & 0xFFFFFFFFFFFFFFFF, global_id, kind))
