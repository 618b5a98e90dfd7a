"""Builds libmagus.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

Numerics flags: ``--fmad=false`` (no FMA contraction in device fp64/fp32, so
every product and sum rounds separately, as in the oracle) and no fast-math;
host code gets ``-ffp-contract=off`` for the same reason.
"""
from __future__ import annotations

import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "build")
LIB = os.path.join(HERE, "libmagus.so")
SOURCES = ["api.cu", "precompute.cpp", "kernels_ref.cu", "kernels_seq.cu", "kernels_walk.cu", "kernels_spec.cu", "kernels_stream.cu", "kernels_family.cu", "kernels_post.cu",
           "kernels_bound.cu", "comm.cpp"]

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "--fmad=false", "-Xcompiler", "-fPIC,-ffp-contract=off,-O2",
          "-Xptxas", "-v", "-I", os.path.join(HERE, "..", "include")]


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.isabs(c) and os.path.exists(c) or not os.path.isabs(c)):
            return c
    return "nvcc"


def _compile(src: str) -> tuple[str, str]:
    obj = os.path.join(BUILD, os.path.splitext(src)[0] + ".o")
    extra = os.environ.get("MAGUS_NVCC_FLAGS", "").split()  # developer experiments only
    cmd = [_nvcc(), *ARCH, *COMMON, *extra, "-x", "cu", "-c", os.path.join(CSRC, src), "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    return obj, r.stderr


def build_libmagus(verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    with ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        res = list(ex.map(_compile, SOURCES))
    log = "\n".join(r[1] for r in res)
    with open(os.path.join(BUILD, "ptxas.log"), "w") as f:
        f.write(log)
    if verbose:
        print(log)
    cmd = [_nvcc(), *ARCH, "-shared", "-cudart", "static", "-o", LIB, *[r[0] for r in res], "-ldl"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    print(f"built {LIB}", flush=True)
    return LIB


if __name__ == "__main__":
    build_libmagus(verbose="-v" in sys.argv)
