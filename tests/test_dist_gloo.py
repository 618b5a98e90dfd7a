"""Multi-process (world_size 2, gloo, CPU) checks of the sharded sweep logic:
shard ownership, the all-reduce of the integer totals, and the replicated
sweep choice.  Per-rank totals come from the CPU oracle on that rank's shard
(the GPU kernels are covered by tests/test_gpu_parity.py); the reduced result
must equal the oracle's totals over all traces, bit for bit."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle

N_TOTAL, T = 90, 1500


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _pols():
    import paper_conf_sc_zhengspl25_b200 as m
    return m.grid_fleet64()[::4]


def _oracle_totals(x, pols_o):
    r = oracle.replay(x, pols_o)
    return np.stack([oracle.totals(r.summary[c], r.base, x.shape[0])[0] for c in range(len(pols_o))])


def _worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sc_zhengspl25_b200 as m
    from paper_conf_sc_zhengspl25_b200 import dist as mdist
    pols = _pols()
    pols_o = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                   tau_dec=p.tau_dec, t_hi=p.t_hi) for p in pols])
    id0, n = mdist.shard(N_TOTAL, world, rank)
    x = gen.gen_traces(gen.SEEDS[4], n, T, id0=id0)
    tot = torch.from_numpy(_oracle_totals(x, pols_o).view(np.int64).copy())
    mdist.allreduce_totals(tot)
    best, row, feas = m.sweep_best_host(tot.numpy().view(np.uint64))
    np.save(os.path.join(out_dir, f"tot{rank}.npy"), tot.numpy().view(np.uint64))
    np.save(os.path.join(out_dir, f"best{rank}.npy"), np.array([best, int(feas)]))
    dist.destroy_process_group()


def test_shard_covers_every_trace_once():
    from paper_conf_sc_zhengspl25_b200 import dist as mdist
    for n_total in (0, 1, 7, 90, 4096, 65536):
        for world in (1, 2, 3, 4, 8):
            got = [mdist.shard(n_total, world, r) for r in range(world)]
            ids = [i for id0, n in got for i in range(id0, id0 + n)]
            assert ids == list(range(n_total))


def test_allreduce_of_totals_is_exact_world2(tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    import paper_conf_sc_zhengspl25_b200 as m
    pols = _pols()
    pols_o = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                   tau_dec=p.tau_dec, t_hi=p.t_hi) for p in pols])
    full = _oracle_totals(gen.gen_traces(gen.SEEDS[4], N_TOTAL, T), pols_o)
    b_full = m.sweep_best_host(full)
    for r in range(world):
        tot = np.load(tmp_path / f"tot{r}.npy")
        assert np.array_equal(tot, full)
        best, feas = np.load(tmp_path / f"best{r}.npy")
        assert (int(best), bool(feas)) == (b_full[0], b_full[2])


def test_host_derivation_matches_oracle():
    import paper_conf_sc_zhengspl25_b200 as m
    x = gen.gen_traces(gen.SEEDS[2], 64, 2000)
    r = oracle.replay(x, oracle.policy())
    w, f = oracle.totals(r.summary[0], r.base, 2000)
    d = m.derive_host(w)
    assert d["energy_j"] == f[0] and d["time_s"] == f[1]
    assert d["base_energy_j"] == f[2] and d["base_time_s"] == f[3]
    assert d["saving"] == f[4] and d["slowdown"] == f[5]


def _worker_cfg(rank, world, port, out_dir):
    """Config sharding: every rank holds every trace and fills only its rows."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sc_zhengspl25_b200 as m
    from paper_conf_sc_zhengspl25_b200 import dist as mdist
    pols = _pols()
    pols_o = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                   tau_dec=p.tau_dec, t_hi=p.t_hi) for p in pols])
    c0, nc = mdist.shard_configs(len(pols), world, rank)
    x = gen.gen_traces(gen.SEEDS[4], N_TOTAL, T)
    full = torch.zeros((len(pols), m.TOT_WORDS), dtype=torch.int64)
    full[c0:c0 + nc] = torch.from_numpy(_oracle_totals(x, pols_o[c0:c0 + nc]).view(np.int64).copy())
    mdist.allreduce_totals(full)
    best, row, feas = m.sweep_best_host(full.numpy().view(np.uint64))
    np.save(os.path.join(out_dir, f"tot{rank}.npy"), full.numpy().view(np.uint64))
    np.save(os.path.join(out_dir, f"best{rank}.npy"), np.array([best, int(feas)]))
    dist.destroy_process_group()


def test_config_sharded_allreduce_world2(tmp_path):
    world = 2
    mp.spawn(_worker_cfg, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    import paper_conf_sc_zhengspl25_b200 as m
    pols = _pols()
    pols_o = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                   tau_dec=p.tau_dec, t_hi=p.t_hi) for p in pols])
    full = _oracle_totals(gen.gen_traces(gen.SEEDS[4], N_TOTAL, T), pols_o)
    b_full = m.sweep_best_host(full)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"tot{r}.npy"), full)
        best, feas = np.load(tmp_path / f"best{r}.npy")
        assert (int(best), bool(feas)) == (b_full[0], b_full[2])


def test_shard_configs_covers_every_config_once():
    from paper_conf_sc_zhengspl25_b200 import dist as mdist
    for C in (1, 16, 64, 256):
        for world in (1, 2, 3, 8):
            got = [mdist.shard_configs(C, world, r) for r in range(world)]
            assert [c for c0, n in got for c in range(c0, c0 + n)] == list(range(C))
