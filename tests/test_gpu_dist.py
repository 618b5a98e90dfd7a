"""Multi-rank replay THROUGH THE CUDA KERNELS: two processes share cuda:0 and
talk over gloo (the only GPU this build gets), each runs
``dist.replay_sharded`` on its shard -- by traces (north_star (3), SURVEY.md
8(e)) and by configs (C >> N/G, the Sec. 6.4 sweep, P@43882) -- and the
all-reduced totals and the replicated choice must be bit-identical to one
process replaying everything, and to the CPU oracle."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

N_TOTAL, T, SEED = 300, 5000, gen.SEEDS[5]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _pols():
    import paper_conf_sc_zhengspl25_b200 as m
    return m.grid_fleet64()[::4]  # 16 configs, both defaults' neighbours included


def _worker(rank, world, port, out_dir, shard_by):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sc_zhengspl25_b200 as m
    from paper_conf_sc_zhengspl25_b200 import dist as mdist
    torch.cuda.set_device(0)
    pols = _pols()
    with m.Context(device=0) as ctx:
        if shard_by == "traces":
            id0, n = mdist.shard(N_TOTAL, world, rank)
        else:
            id0, n = 0, N_TOTAL
        x = ctx.gen_traces(SEED, n, T, kind=gen.KIND_ADVERSARIAL, id0=id0)
        res, best, row, feas = mdist.replay_sharded(ctx, x, pols, shard_by=shard_by, want_summary=False,
                                                    want_base=False)
        torch.cuda.synchronize()
        tot = res.totals.cpu().numpy().view(np.uint64)
        launches = ctx.stats()["launches_total"]
    np.save(os.path.join(out_dir, f"tot{rank}.npy"), tot)
    np.save(os.path.join(out_dir, f"best{rank}.npy"), np.array([best, int(feas), launches]))
    dist.destroy_process_group()


@pytest.mark.parametrize("shard_by", ["traces", "configs"])
def test_two_ranks_through_the_kernels_equal_one_process(tmp_path, shard_by):
    import torch
    import torch.multiprocessing as mp

    import paper_conf_sc_zhengspl25_b200 as m
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path), shard_by), nprocs=world, join=True)
    pols = _pols()
    with m.Context(device=0) as ctx:
        x = ctx.gen_traces(SEED, N_TOTAL, T, kind=gen.KIND_ADVERSARIAL)
        res = ctx.replay(x, pols, want_summary=False, want_base=False, want_totals=True)
        best1, _, feas1 = ctx.sweep_best(res.totals)
        torch.cuda.synchronize()
        single = res.totals.cpu().numpy().view(np.uint64)
    # the oracle over the whole fleet (independent of the CUDA path)
    xh = gen.gen_traces(SEED, N_TOTAL, T, kind=gen.KIND_ADVERSARIAL)
    pols_o = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                   tau_dec=p.tau_dec, t_hi=p.t_hi) for p in pols])
    r = oracle.replay(xh, pols_o)
    ref = np.stack([oracle.totals(r.summary[c], r.base, T)[0] for c in range(len(pols_o))])
    assert np.array_equal(single, ref)
    for rank in range(world):
        tot = np.load(tmp_path / f"tot{rank}.npy")
        best, feas, launches = np.load(tmp_path / f"best{rank}.npy")
        assert launches > 0                      # the rank really ran the kernels
        assert np.array_equal(tot, single), (shard_by, rank)
        assert (int(best), bool(feas)) == (best1, feas1)
