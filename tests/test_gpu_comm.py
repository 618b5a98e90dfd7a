"""The optional native NCCL path of the C-ABI (magus_comm_unique_id /
magus_comm_init / magus_allreduce_totals) on one GPU: a
single-rank communicator makes the all-reduce an identity on the exact
integer totals, so the choice is unchanged; bad arguments are rejected; a
context without a communicator treats the all-reduce as a no-op.  (Several
ranks need several GPUs: the multi-rank path is the driver's scaling run;
its host logic -- sharding and the integer sum -- is covered on gloo in
test_dist_gloo.py.)"""
from __future__ import annotations

import numpy as np
import pytest

import gen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
magus = pytest.importorskip("paper_conf_sc_zhengspl25_b200")


def test_single_rank_allreduce_is_identity():
    x = gen.gen_traces(gen.SEEDS[3], 300, 4000)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    pols = magus.grid_fleet64()[:8]
    with magus.Context(device=0) as ctx:
        r = ctx.replay(xd, pols, want_summary=False, want_base=False)
        torch.cuda.synchronize()
        before = r.totals.clone()
        best0 = ctx.sweep_best(r.totals)
        ctx.allreduce_totals(r.totals)            # no communicator yet: a no-op
        torch.cuda.synchronize()
        assert torch.equal(before, r.totals)
        uid = magus.comm_unique_id()
        assert len(uid) == magus.COMM_ID_BYTES
        ctx.comm_init(uid, 1, 0)
        ctx.allreduce_totals(r.totals)            # one rank: the sum is the identity
        torch.cuda.synchronize()
        assert torch.equal(before, r.totals)
        best1 = ctx.sweep_best(r.totals)
        assert best0[0] == best1[0] and best0[2] == best1[2]
        # the communicator is per context and survives further replays
        r2 = ctx.replay(xd, pols, want_summary=False, want_base=False)
        ctx.allreduce_totals(r2.totals)
        torch.cuda.synchronize()
        assert torch.equal(r2.totals, before)


def test_comm_init_rejects_bad_arguments():
    with magus.Context(device=0) as ctx:
        uid = magus.comm_unique_id()
        with pytest.raises(magus.MagusError) as e:
            ctx.comm_init(uid, 1, 1)                  # rank >= nranks
        assert e.value.status == magus.ERR_INVALID_ARG
        with pytest.raises(magus.MagusError):
            ctx.comm_init(uid, 0, 0)
