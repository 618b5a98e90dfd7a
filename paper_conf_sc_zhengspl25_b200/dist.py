"""Multi-GPU glue: trace sharding and the one collective of the sweep.

Traces are independent (north_star (3)), so rank r of G owns the contiguous
block of global trace ids [r*n, (r+1)*n) and runs every config on it.  The
only exchange is ONE all-reduce (sum) of the per-config uint64 totals
[C x 16] over torch.distributed -- NCCL over NVLink/NVSwitch on the GPU box,
gloo in the CPU tests.  The totals are exact integers (limb-split q sums), so
the sum is exact and order-free: totals and the argmin are bit-identical for
any G.  Every rank then derives the fleet energies and picks the config with
the same deterministic rule (no broadcast needed).
"""
from __future__ import annotations

import numpy as np

from . import TOT_WORDS


def shard(n_total: int, world: int, rank: int) -> tuple[int, int]:
    """(first global trace id, count) of `rank`; the remainder goes to the
    first ranks so that every trace is owned exactly once."""
    if world < 1 or not 0 <= rank < world or n_total < 0:
        raise ValueError("bad shard arguments")
    base, extra = divmod(n_total, world)
    n = base + (1 if rank < extra else 0)
    id0 = rank * base + min(rank, extra)
    return id0, n


def allreduce_totals(totals, group=None):
    """In-place SUM all-reduce of an int64 [C, 16] tensor of totals (the
    uint64 words viewed as int64: a wrapping two's-complement sum is the
    same bit pattern as the uint64 sum)."""
    import torch
    import torch.distributed as dist
    assert totals.dtype == torch.int64 and totals.shape[-1] == TOT_WORDS
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(totals, op=dist.ReduceOp.SUM, group=group)
    return totals


def replay_sharded(ctx, traces, policies, group=None, **kw):
    """magus_replay on this rank's shard, then the all-reduce of the totals
    and the (replicated) sweep choice.  Returns (result, best, row, feasible)."""
    res = ctx.replay(traces, policies, want_totals=True, **kw)
    allreduce_totals(res.totals, group)
    best, row, feasible = ctx.sweep_best(res.totals)
    return res, best, row, feasible


def merge_totals_numpy(parts) -> np.ndarray:
    """Host-side merge of per-shard totals (the same arithmetic as the
    all-reduce): uint64 word-wise sum."""
    acc = np.zeros_like(np.asarray(parts[0], dtype=np.uint64))
    for p in parts:
        acc += np.asarray(p, dtype=np.uint64)
    return acc
