"""Multi-GPU glue: trace or config sharding and the one collective of the sweep.

Traces are independent and so are configs (north_star (3)).  Trace sharding
(the default): rank r of G owns the contiguous block of global trace ids
[r*n, (r+1)*n) and runs every config on it.  Config sharding (C >> N/G, e.g.
the Sec. 6.4 threshold sweep, P@43882): rank r runs its contiguous block of
configs over every trace and fills only those rows of the [C x 18] totals.
Either way the only exchange is ONE all-reduce (sum) of the per-config uint64
totals [C x 18] over torch.distributed -- NCCL over NVLink/NVSwitch on the
GPU box, gloo in the CPU tests (rows a rank does not own are zero, so the sum
of disjoint rows is exact too).  The totals are exact integers (limb-split q sums), so
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


def shard_configs(n_configs: int, world: int, rank: int) -> tuple[int, int]:
    """(first config index, count) of `rank` under config sharding (the same
    contiguous split as the traces)."""
    return shard(n_configs, world, rank)


def allreduce_totals(totals, group=None):
    """In-place SUM all-reduce of an int64 [C, 18] tensor of totals (the
    uint64 words viewed as int64: a wrapping two's-complement sum is the
    same bit pattern as the uint64 sum).  gloo reduces host tensors, so a
    CUDA tensor goes through a host copy there (tests only; NCCL reduces
    device memory in place)."""
    import torch
    import torch.distributed as dist
    assert totals.dtype == torch.int64 and totals.shape[-1] == TOT_WORDS
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        if totals.is_cuda and dist.get_backend(group) == "gloo":
            h = totals.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
            totals.copy_(h)
        else:
            dist.all_reduce(totals, op=dist.ReduceOp.SUM, group=group)
    return totals


def replay_sharded(ctx, traces, policies, group=None, shard_by: str = "traces", **kw):
    """magus_replay on this rank's shard, then the all-reduce of the totals
    and the (replicated) sweep choice.  Returns (result, best, row, feasible).

    shard_by="traces": `traces` is this rank's block of traces (dist.shard),
    every config runs here.  shard_by="configs": `traces` is the whole fleet,
    this rank runs configs shard_configs(C, G, r) and the result's totals are
    the full [C x 18] table (this rank's rows + the all-reduce)."""
    import torch
    import torch.distributed as dist
    if shard_by == "traces":
        res = ctx.replay(traces, policies, want_totals=True, **kw)
        allreduce_totals(res.totals, group)
        best, row, feasible = ctx.sweep_best(res.totals)
        return res, best, row, feasible
    if shard_by != "configs":
        raise ValueError(f"shard_by must be 'traces' or 'configs', not {shard_by!r}")
    pols = list(policies)
    C = len(pols)
    world = dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1
    rank = dist.get_rank(group) if world > 1 else 0
    c0, nc = shard_configs(C, world, rank)
    full = torch.zeros((C, TOT_WORDS), dtype=torch.int64, device=traces.device)
    res = None
    if nc > 0:
        res = ctx.replay(traces, pols[c0:c0 + nc], want_totals=True, **kw)
        full[c0:c0 + nc].copy_(res.totals)
    allreduce_totals(full, group)
    best, row, feasible = ctx.sweep_best(full)
    if res is not None:
        res.totals = full
    return res, best, row, feasible


def merge_totals_numpy(parts) -> np.ndarray:
    """Host-side merge of per-shard totals (the same arithmetic as the
    all-reduce): uint64 word-wise sum."""
    acc = np.zeros_like(np.asarray(parts[0], dtype=np.uint64))
    for p in parts:
        acc += np.asarray(p, dtype=np.uint64)
    return acc
