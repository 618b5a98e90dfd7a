#!/usr/bin/env python3
"""Benchmark of the MAGUS replay hot path on B200.

One "step" = one pass of the whole hot path over the workload resident in
HBM: Alg. 1-3 for every interval x trace x config + model M (stream kernel),
the segment fix-up, the per-config totals, the NCCL sum of the totals when
sharded, and magus_sweep_best (device->host read of the totals, argmin).

  python bench.py [--gpus N --steps K --warmup W] [--config 2|3|5] [--impl reference]
  torchrun --nproc-per-node N bench.py --gpus N ...   (one process per GPU)

Metric (BASELINE.json): trace-samples x configs per second, whole job; plus
the dominant kernel's achieved HBM GB/s against the measured copy peak.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

SEED_BASE = 0x4D41475553000000
WORKLOADS = {
    # cfg: (n_traces per GPU, n_steps, grid, kind, decisions, description)
    1: (1, 10_000, "default", 0, True, "cfg1: 1 trace x 10,000 intervals x 1 config (paper_default)"),
    2: (4096, 100_000, "default", 0, True, "cfg2: 4,096 traces x 100,000 intervals x 1 config (paper_default)"),
    3: (4096, 100_000, "sweep256", 0, False, "cfg3: 4,096 traces x 100,000 intervals x 256 configs (SWEEP256)"),
    4: (65536, 1_000_000, "fleet64", 0, False,
        "cfg4: 65,536 traces x 1,000,000 intervals x 64 configs (FLEET64), traces sharded over the GPUs"),
    5: (16384, 1_000_000, "default", 1, False,
        "cfg5: 16,384 adversarial traces x 1,000,000 intervals x 1 config (paper_default)"),
}
METRIC = "trace-samples x configs/sec"
UNIT = "trace-samples*configs/s"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled in the background."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.marks = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "50", "-i", str(self.index)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read, daemon=True).start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append((time.time(), line.strip()))

    def mark(self):
        self.marks.append(time.time())

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        t0, t1 = (self.marks + [0, 0])[:2] if len(self.marks) >= 2 else (0, 1e18)
        inside = [r for r in self.rows if t0 <= r[0] <= t1]
        note = None
        if len(inside) < 3:
            inside, note = self.rows, "timed region shorter than 3 samples: whole-run samples"
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for _, line in inside:
            f = [x.strip() for x in line.split(",")]
            try:
                sm.append(float(f[0]))
                smax.append(float(f[1]))
            except Exception:
                continue
            for name, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(name)
        out = {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
               "reasons": sorted(reasons), "samples": len(inside)}
        if note:
            out["note"] = note
        return out


def setup_dist(world: int, local: int) -> int:
    """One process per GPU; returns this rank's CUDA device index.  The
    backend is NCCL; MAGUS_DIST_BACKEND=gloo (with several ranks sharing a
    GPU, device = local rank mod the GPU count) exercises the multi-rank path
    of this script on a single-GPU box."""
    import torch
    import torch.distributed as dist
    devidx = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(devidx)
    if world > 1:
        dist.init_process_group(os.environ.get("MAGUS_DIST_BACKEND", "nccl"), init_method="env://")
    return devidx


def dist_backend(world: int) -> str:
    return "none" if world == 1 else os.environ.get("MAGUS_DIST_BACKEND", "nccl")


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


class OraclePool:
    """The oracle as it stands, run on several host cores at once over a
    static partition of the traces (traces are independent; the ctypes call
    releases the GIL, and the C++ replay keeps no shared state)."""

    def __init__(self, threads: int):
        from concurrent.futures import ThreadPoolExecutor
        self.threads = max(1, threads)
        self.ex = ThreadPoolExecutor(self.threads)

    def replay(self, xs, pols):
        """xs: [T, N] -> per-config summaries [C, N] (trace order kept)."""
        import oracle
        N = xs.shape[1]
        k = max(1, min(self.threads, N))
        parts = [np.ascontiguousarray(xs[:, i * N // k:(i + 1) * N // k]) for i in range(k)]
        res = list(self.ex.map(lambda part: oracle.replay(part, pols), parts))
        return np.concatenate([r.summary for r in res], axis=1)

    def close(self):
        self.ex.shutdown()


def cpu_oracle_sample(cfg, T, pols_oracle, budget_s, kind, max_traces=None, threads=1):
    """Times the oracle, as it stands, on a bounded sample of the workload,
    on `threads` host cores (a static partition of the sampled traces)."""
    import gen
    import oracle
    seed = SEED_BASE + cfg
    # probe on a sample of the same shape class (time-major, ld = n): the
    # oracle reads each trace with stride ld, so a tiny probe under-estimates
    probe_n = max(1, min(64, int(2e7 / (T * len(pols_oracle)))))  # ~2 s of probe
    if max_traces:
        probe_n = min(probe_n, max_traces)
    xs = gen.gen_traces(seed, probe_n, T, kind=kind)
    t = time.perf_counter()
    oracle.replay(xs, pols_oracle)
    per_trace = (time.perf_counter() - t) / probe_n
    n = max(1, int(budget_s * threads / max(per_trace, 1e-9)))
    if max_traces:
        n = min(n, max_traces)
    n = min(n, 1024 * threads)  # keeps each part's ld (the oracle's stride) in the probed regime
    if T > 100_000:             # long traces: wide parts stride badly, the probe under-estimates
        n = min(n, 64 * threads)
    n = max(n, min(threads, max_traces or threads))
    xs = gen.gen_traces(seed, n, T, kind=kind)
    pool = OraclePool(threads)
    pool.replay(xs[:64, :pool.threads], pols_oracle)  # threads started, library loaded
    t = time.perf_counter()
    summ = pool.replay(xs, pols_oracle)
    dt = time.perf_counter() - t
    pool.close()
    units = n * T * len(pols_oracle)
    return units / dt, n, dt, summ


def policies_for(grid):
    import paper_conf_sc_zhengspl25_b200 as magus
    if grid == "sweep256":
        return magus.grid_sweep256()
    if grid == "fleet64":
        return magus.grid_fleet64()
    return [magus.policy_preset(magus.POLICY_PAPER_DEFAULT)]


def oracle_policies(pols):
    import oracle
    return oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                 tau_dec=p.tau_dec, t_hi=p.t_hi, variant=p.variant, step=p.step)
                            for p in pols])


def run_reference(args):
    """--impl reference: the oracle timed on the host cores, bounded samples."""
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    N, T, grid, kind, _, desc = WORKLOADS[args.config]
    import gen
    import oracle
    pols = oracle_policies(policies_for(grid))
    seed = SEED_BASE + args.config
    threads = args.cpu_threads or host_cores()
    per_thread = 4 if args.config not in (4, 5) else 1
    per_step = max(1, min(N, per_thread * threads))
    xs = gen.gen_traces(seed, per_step, T, kind=kind)
    if args.config in (3, 4):
        pols = pols[:16]  # bounded: 16 of the 256 / 64 configs per step
    pool = OraclePool(threads)
    for _ in range(args.warmup):
        pool.replay(xs, pols)
    t = time.perf_counter()
    for _ in range(args.steps):
        pool.replay(xs, pols)
    dt = (time.perf_counter() - t) / args.steps
    pool.close()
    cores = min(threads, per_step)
    value = per_step * T * len(pols) / dt
    sample = (f"{per_step} trace(s) x {T} intervals x {len(pols)} config(s) per step (seed {seed:#x}), "
              f"statically partitioned over {cores} host thread(s)")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": desc, "n_steps": T, "n_configs": len(pols), "kind": kind},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_sc_zhengspl25_b200 as magus
    from paper_conf_sc_zhengspl25_b200 import dist as mdist

    world, rank, local = dist_env()
    if world != args.gpus:
        print(f"warning: --gpus {args.gpus} but WORLD_SIZE {world}", file=sys.stderr)
    local = setup_dist(world, local)
    dev = torch.device(f"cuda:{local}")
    stream = torch.cuda.current_stream(dev)

    N, T, grid, kind, want_dec, desc = WORKLOADS[args.config]
    if args.n_traces:
        N = args.n_traces
    if args.n_steps:
        T = args.n_steps
    if args.no_decisions:
        want_dec = False
    pols = policies_for(grid)
    if args.variant:  # NEXT f3 / f4: closed loop (seq_kernel) / gradual step (walk kernels)
        for p in pols:
            p.variant = args.variant
            p.step = args.step if args.variant & magus.VARIANT_GRADUAL else 0
    C = len(pols)
    seed = SEED_BASE + args.config
    plat = magus.platform_preset()
    if args.burst > 0:  # NEXT f1: Sec. 6.3 burst Jaccard counters in the same pass
        plat.burst_mbs = args.burst
    ctx = magus.Context(device=local, stream=stream, platform=plat)
    if args.waves:
        ctx.set_option(magus.OPT_WAVES, args.waves)
    if args.segments:
        ctx.set_option(magus.OPT_SEGMENTS, args.segments)
    if args.bundle:
        ctx.set_option(magus.OPT_BUNDLE, args.bundle)
    if args.spec_warm:
        ctx.set_option(magus.OPT_SPEC_WARM, args.spec_warm)
    if args.kernel:
        ctx.set_option(magus.OPT_KERNEL, args.kernel)
    id0, _ = mdist.shard(N * world, world, rank)     # weak scaling: N traces per GPU
    x = ctx.gen_traces(seed, N, T, kind=kind, id0=id0)
    torch.cuda.synchronize()

    out = None
    sweep_buf = None
    # --inflight 2: consecutive steps alternate between two contexts on two
    # streams (own scratch, outputs and choice buffers; the traces are
    # shared, read-only), so one step's tail overlaps the next step's head
    lanes = [[ctx, stream, None, None]]
    if args.inflight > 1:
        s2 = torch.cuda.Stream(dev)
        ctx2 = magus.Context(device=local, stream=s2, platform=plat)
        for k, v in ((magus.OPT_WAVES, args.waves), (magus.OPT_SEGMENTS, args.segments),
                     (magus.OPT_BUNDLE, args.bundle), (magus.OPT_KERNEL, args.kernel)):
            if v:
                ctx2.set_option(k, v)
        lanes.append([ctx2, s2, None, None])
    nstep = [0]
    if args.comm == "native" and world > 1:
        # rank 0's NCCL id reaches every rank through the process group
        uids = [magus.comm_unique_id() if rank == 0 else None for _ in lanes]
        dist.broadcast_object_list(uids, src=0)
        for ln, uid in zip(lanes, uids):  # one communicator (and id) per context
            ln[0].comm_init(uid, world, rank)

    def step():
        # replay (one fused launch per W group) -> NCCL sum of the integer
        # totals -> device-side choice + async device->host copy of the result
        # into pinned memory (no host sync inside a step; --sync-sweep restores
        # the synchronous magus_sweep_best)
        nonlocal out, sweep_buf
        ln = lanes[nstep[0] % len(lanes)]
        nstep[0] += 1
        c_, s_, o_, b_ = ln
        with torch.cuda.stream(s_):
            o_ = c_.replay(x, pols, want_summary=False, want_base=False, want_decisions=want_dec,
                           want_totals=True, out=o_)
            if args.comm == "native":          # the library's own NCCL communicator
                c_.allreduce_totals(o_.totals)
            else:
                mdist.allreduce_totals(o_.totals)  # the one collective; exact (integer words)
            if args.sync_sweep:
                ln[2] = o_
                return c_.sweep_best(o_.totals)
            b_ = c_.sweep_best_async(o_.totals, b_)
        ln[2], ln[3] = o_, b_
        out, sweep_buf = o_, b_
        return b_

    def result(r):
        return r if args.sync_sweep else ctx.sweep_result(r)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    for ln in lanes:
        ln[0].set_option(magus.OPT_TIMING, 1)
        ln[0].reset_stats()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clocks.mark()
    e0.record(stream)
    for ln in lanes[1:]:
        ln[1].wait_event(e0)
    for _ in range(args.steps):
        best = step()
    for ln in lanes[1:]:
        done_ev = torch.cuda.Event()
        done_ev.record(ln[1])
        stream.wait_event(done_ev)
    e1.record(stream)
    torch.cuda.synchronize()
    best = result(best)
    clocks.mark()
    if world > 1:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    st = ctx.stats()
    for ln in lanes[1:]:  # launches of every context in flight
        s2 = ln[0].stats()
        for key in ("launches_total", "main_launches", "main_ms_total"):
            st[key] += s2[key]
        ln[0].set_option(magus.OPT_TIMING, 0)
    ctx.set_option(magus.OPT_TIMING, 0)
    time.sleep(0.2)
    clocks.stop()
    # with steps in flight, also time the dominant kernel alone: a few serial
    # steps on one context, untimed for `value`, CUDA events per launch
    serial_ms = None
    if len(lanes) > 1:
        torch.cuda.synchronize()
        ctx.set_option(magus.OPT_TIMING, 1)
        ctx.reset_stats()
        for _ in range(min(50, max(5, args.steps))):
            o = ctx.replay(x, pols, want_summary=False, want_base=False, want_decisions=want_dec,
                           want_totals=True, out=lanes[0][2])
            lanes[0][2] = o
            torch.cuda.synchronize()
        s1 = ctx.stats()
        ctx.set_option(magus.OPT_TIMING, 0)
        serial_ms = s1["main_ms_total"] / max(1, s1["main_launches"])
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        kt = torch.tensor([st["main_ms_total"]], dtype=torch.float64, device=dev)
        dist.all_reduce(kt, op=dist.ReduceOp.MAX)
        st["main_ms_total"] = float(kt.item())
    ms_per_step = ms / args.steps
    units_per_step = N * world * T * C
    value = units_per_step / (ms_per_step * 1e-3)

    # roofline of the dominant kernel (stream kernel), from live CUDA events
    peak, peak_src = _peaks()
    kern_ms = st["main_ms_total"] / max(1, st["main_launches"])
    alg_bytes = N * T * 4 + (C * N * T / 8 if want_dec else 0)
    achieved = alg_bytes / (kern_ms * 1e-3) / 1e9
    roof_method = "algorithmic bytes per launch / mean launch duration (CUDA events on the launching stream)"
    if len(lanes) > 1:
        # consecutive steps' kernels overlap on two streams, so each launch's
        # event-timed duration includes the other's share of the GPU: the
        # dominant kernel's rate is the aggregate over the timed region
        achieved = alg_bytes * args.steps / (ms * 1e-3) / 1e9
        roof_method = (f"{len(lanes)} launches in flight on separate streams: algorithmic bytes of all launches / "
                       f"timed region (per-launch event duration {kern_ms:.4f} ms includes the overlap)")
    traffic = None
    kname = {1: "ref_kernel", 2: "stream_kernel", 3: "seq_kernel", 4: "walk_map_kernel + walk_replay_kernel + walk_final_kernel", 5: "spec_kernel + spec_fix_kernel"}.get(st["last_kernel"], "?")
    vtag = {0: "", 1: "_f3", 2: "_f4"}.get(args.variant, f"_v{args.variant}")
    # traffic only from an ncu capture of this very kernel and workload
    prof = os.path.join(ROOT, "profiles", f"ncu_cfg{args.config}{vtag}.json")
    if os.path.exists(prof):
        try:
            with open(prof) as f:
                traffic = json.load(f).get("dram_bytes_per_launch")
        except Exception:
            traffic = None

    # e2e: through the C-ABI with HOST buffers (H2D of the traces + D2H of the totals per step)
    e2e = None
    if not args.no_e2e:
        xh = torch.empty((T, N), dtype=torch.float32, pin_memory=True)
        xh.copy_(x.cpu())
        xn = xh.numpy()
        e2e_steps = max(1, min(args.steps, args.e2e_steps))
        ctx.replay_host(xn, pols, want_summary=False, want_base=False, want_totals=True)
        if world > 1:
            dist.barrier()
        t = time.perf_counter()
        for _ in range(e2e_steps):
            _, _, _, tot = ctx.replay_host(xn, pols, want_summary=False, want_base=False, want_totals=True)
            if world > 1:
                tt = torch.from_numpy(tot.view(np.int64)).to(dev)
                dist.all_reduce(tt, op=dist.ReduceOp.SUM)
                tt.cpu()
        el = time.perf_counter() - t
        if world > 1:
            tmax = torch.tensor([el], dtype=torch.float64, device=dev)
            dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
            el = float(tmax.item())
        e2e = {"value": units_per_step * e2e_steps / el, "unit": UNIT,
               "h2d_bytes_per_step": N * T * 4 * world, "d2h_bytes_per_step": C * 16 * 8 * world,
               "steps": e2e_steps, "path": "magus_replay_host (pinned host traces)"}

    cpu = None
    parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        pol_o = oracle_policies(pols)
        if C > 16:
            pol_o = pol_o[:16]
        threads = args.cpu_threads or host_cores()
        v, n_s, dt_s, ref_summ = cpu_oracle_sample(args.config, T, pol_o, args.cpu_budget, kind, max_traces=N,
                                                   threads=threads)
        cpu = {"value": v, "unit": UNIT, "cores": min(threads, n_s), "kind": "oracle",
               "sample": f"first {n_s} traces x {T} intervals x {len(pol_o)} config(s) of the same workload, "
                         f"statically partitioned over {min(threads, n_s)} host thread(s) ({dt_s:.1f} s)"}
        # parity of that sample against the GPU path (untimed)
        r = ctx.replay(x[:, :n_s], pols[:len(pol_o)], n_traces=n_s, want_totals=False)
        torch.cuda.synchronize()
        got = r.summary_numpy()
        parity = bool(all(np.array_equal(got[g], ref_summ[o]) for g, o in
                          [("n_events", "n_events"), ("n_changes", "n_changes"), ("digest", "digest"),
                           ("energy_j", "energy"), ("time_s", "time")]))

    # C > 1 sweeps are ALU-bound: algorithmic work = 8 lane-ops
    # per decision (lag difference, 2 threshold compares, event
    # log, count compare, priority select, change compare, accumulate); peak =
    # 148 SMs x 4 SMSPs x 32 lanes x max SM clock (one lane-op per lane-cycle).
    clk = clocks.summary()
    hbm_roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                "kernel": kname, "kernel_ms": kern_ms, "alg_bytes_per_launch": alg_bytes,
                "method": roof_method}
    if serial_ms is not None:
        hbm_roof["serial_launch"] = {"kernel_ms": serial_ms, "achieved": alg_bytes / (serial_ms * 1e-3) / 1e9,
                                     "frac": alg_bytes / (serial_ms * 1e-3) / 1e9 / peak,
                                     "note": "the kernel timed alone (serial steps after the timed region)"}
    roof = hbm_roof
    if C > 1:
        sm_mhz = clk.get("sm_max_mhz") or 1965.0
        alu_peak = 148 * 4 * 32 * sm_mhz * 1e6 / 1e9   # Gop/s
        alu_ach = 8.0 * N * T * C / (kern_ms * 1e-3) / 1e9
        if len(lanes) > 1:
            alu_ach = 8.0 * N * T * C * args.steps / (ms * 1e-3) / 1e9
        roof = {"bound": "alu", "achieved": alu_ach, "peak": alu_peak, "unit": "Gop/s",
                "frac": alu_ach / alu_peak, "traffic": traffic,
                "peak_source": f"148 SMs x 128 lanes x {sm_mhz:.0f} MHz (B200_PROFILING.md unit counts)",
                "kernel": kname, "kernel_ms": kern_ms, "alg_ops_per_decision": 8, "method": roof_method}
        if serial_ms is not None:
            sa = 8.0 * N * T * C / (serial_ms * 1e-3) / 1e9
            roof["serial_launch"] = {"kernel_ms": serial_ms, "achieved": sa, "frac": sa / alu_peak,
                                     "note": "the kernel timed alone (serial steps after the timed region)"}
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": desc, "n_traces_per_gpu": N, "n_traces_total": N * world, "n_steps": T,
                       "n_configs": C, "decisions_emitted": want_dec, "seed": hex(seed),
                       "l2": f"inputs {N * T * 4 / 1e9:.2f} GB per GPU > 126 MB L2 (no flush needed)",
                       "parallelism": f"traces sharded over {world} GPU(s); 1 all-reduce of int64 totals "
                                      f"({'native NCCL' if args.comm == 'native' and world > 1 else dist_backend(world)})",
                       "steps_in_flight": len(lanes),
                       "segments": st["last_segments"], "kernel": {1: "reference", 2: "stream", 3: "sequential", 4: "walk", 5: "spec"}.get(st["last_kernel"], "?"),
                       "variant": args.variant, "step": args.step if args.variant & 2 else 0},
            "roofline": roof,
            "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": int(st["launches_total"]), "clocks": clk,
            "best_config": best[0], "feasible": best[2]}
    if args.burst > 0:
        line["config"]["burst_mbs"] = args.burst
        line["best_jaccard"] = best[1]["jaccard"]
        line["pareto_front"] = [int(i) for i in np.flatnonzero(ctx.pareto_front(out.totals))]
    if roof is not hbm_roof:
        line["roofline_hbm"] = hbm_roof
    if parity is not None:
        line["parity_sample_ok"] = parity
    if rank == 0:
        print(json.dumps(line), flush=True)
    for ln in lanes[1:]:
        ln[0].close()
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_fleet(args):
    """Config 4: 65,536 traces x 10^6 intervals x FLEET64, traces sharded over
    the GPUs (strong scaling: the fleet is fixed).  One GPU holds 262 GB of
    traces only in time chunks: each step streams the fleet through HBM in
    chunks of R intervals, generated on the device (untimed, SURVEY 8(d):
    "trace generation is excluded") and replayed with magus_replay_resume
    (timed: CUDA events around every replay call + the final all-reduce and
    device-side choice).  The chunked replay is bit-identical to a one-shot
    replay (tests/test_gpu_resume.py)."""
    import torch
    import torch.distributed as dist

    import paper_conf_sc_zhengspl25_b200 as magus
    from paper_conf_sc_zhengspl25_b200 import dist as mdist

    world, rank, local = dist_env()
    local = setup_dist(world, local)
    dev = torch.device(f"cuda:{local}")
    stream = torch.cuda.current_stream(dev)
    N_tot, T, grid, kind, _, desc = WORKLOADS[4]
    if args.n_traces:
        N_tot = args.n_traces
    if args.n_steps:
        T = args.n_steps
    id0, N = mdist.shard(N_tot, world, rank)
    pols = policies_for(grid)
    C = len(pols)
    seed = SEED_BASE + 4
    ctx = magus.Context(device=local, stream=stream)
    halo = magus.resume_halo(pols)
    ld = (N + 3) // 4 * 4
    R = args.chunk if args.chunk else min(T, (32 << 30) // (ld * 4))
    R = max(halo, R // 32 * 32)
    buf = torch.empty((halo + R, ld), dtype=torch.float32, device=dev)
    gstate = ctx.gen_state(N)
    state = ctx.resume_state(N, pols)
    chunks = [(t, min(T, t + R)) for t in range(0, T, R)]
    sweep_buf = None

    def step(timed):
        nonlocal sweep_buf
        evs = []
        out = None
        for i, (t0, t1) in enumerate(chunks):
            n = t1 - t0
            if i > 0:  # the halo: the previous chunk's last rows
                buf[:halo].copy_(buf[R:R + halo])
            ctx.gen_traces_resume(seed, N, t0, n, gstate, buf[halo:halo + n], kind=kind, id0=id0)
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            if i == 0:
                state.zero_()   # fresh accumulators for this pass
                xs, tb = buf[halo:halo + n], 0
            else:
                xs, tb = buf[:halo + n], t0 - halo
            last = i == len(chunks) - 1
            out = ctx.replay_resume(xs, pols, state, t_base=tb, t_start=t0, n_traces=N, want_summary=False,
                                    want_base=False, want_decisions=False, want_totals=last)
            if last:
                mdist.allreduce_totals(out.totals)
                sweep_buf = ctx.sweep_best_async(out.totals, sweep_buf)
            b.record(stream)
            evs.append((a, b))
        return evs, out

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    ctx.set_option(magus.OPT_TIMING, 1)
    ctx.reset_stats()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.mark()
    all_evs = []
    for _ in range(args.steps):
        evs, out = step(True)
        all_evs += evs
    torch.cuda.synchronize()
    clocks.mark()
    best = ctx.sweep_result(sweep_buf)
    if world > 1:
        dist.barrier()
    ms = sum(a.elapsed_time(b) for a, b in all_evs)
    st = ctx.stats()
    ctx.set_option(magus.OPT_TIMING, 0)
    time.sleep(0.2)
    clocks.stop()
    kern_ms = st["main_ms_total"]
    if world > 1:
        t = torch.tensor([ms, kern_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms, kern_ms = float(t[0].item()), float(t[1].item())
    ms_per_step = ms / args.steps
    value = N_tot * T * C / (ms_per_step * 1e-3)
    clk = clocks.summary()
    sm_mhz = clk.get("sm_max_mhz") or 1965.0
    alu_peak = 148 * 4 * 32 * sm_mhz * 1e6 / 1e9
    alu_ach = 8.0 * N * T * C * args.steps / (kern_ms * 1e-3) / 1e9

    # bounded oracle sample + parity of the chunked path at full T (untimed)
    cpu = None
    parity = None
    if rank == 0 and not args.no_cpu_baseline:
        import oracle
        pol_o = oracle_policies(pols)[:16]
        threads = args.cpu_threads or host_cores()
        v, n_s, dt_s, ref_summ = cpu_oracle_sample(4, T, pol_o, args.cpu_budget, kind, max_traces=64,
                                                   threads=threads)
        cpu = {"value": v, "unit": UNIT, "cores": min(threads, n_s), "kind": "oracle",
               "sample": f"first {n_s} traces x {T} intervals x {len(pol_o)} configs of the fleet, "
                         f"statically partitioned over {min(threads, n_s)} host thread(s) ({dt_s:.1f} s)"}
        if world == 1:
            ld_s = (n_s + 3) // 4 * 4
            sb = torch.empty((halo + R, ld_s), dtype=torch.float32, device=dev)
            gs = ctx.gen_state(n_s)
            rs = ctx.resume_state(n_s, pols[:16])
            for i, (t0, t1) in enumerate(chunks):
                n = t1 - t0
                if i > 0:
                    sb[:halo].copy_(sb[R:R + halo])
                ctx.gen_traces_resume(seed, n_s, t0, n, gs, sb[halo:halo + n], kind=kind, id0=0)
                xs, tb = (sb[halo:halo + n], 0) if i == 0 else (sb[:halo + n], t0 - halo)
                r = ctx.replay_resume(xs, pols[:16], rs, t_base=tb, t_start=t0, n_traces=n_s,
                                      want_summary=i == len(chunks) - 1, want_base=False, want_totals=False)
            torch.cuda.synchronize()
            got = r.summary_numpy()
            parity = bool(all(np.array_equal(got[g], ref_summ[o]) for g, o in
                              [("n_events", "n_events"), ("n_changes", "n_changes"), ("digest", "digest"),
                               ("energy_j", "energy"), ("time_s", "time")]))
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": desc, "n_traces_total": N_tot, "n_traces_per_gpu": N, "n_steps": T,
                       "n_configs": C, "decisions_emitted": False, "seed": hex(seed),
                       "chunk_intervals": R, "chunks": len(chunks), "halo_rows": halo,
                       "l2": f"chunks of {N * R * 4 / 1e9:.1f} GB > 126 MB L2 (no flush needed)",
                       "timed": "replay calls + all-reduce + device choice; on-device generation of each "
                                "chunk and the halo copy untimed (SURVEY 8(d))",
                       "parallelism": f"traces sharded over {world} GPU(s); 1 all-reduce of int64 totals ({dist_backend(world)})"},
            "roofline": {"bound": "alu", "achieved": alu_ach, "peak": alu_peak, "unit": "Gop/s",
                         "frac": alu_ach / alu_peak, "traffic": None,
                         "peak_source": f"148 SMs x 128 lanes x {sm_mhz:.0f} MHz (B200_PROFILING.md unit counts)",
                         "kernel": "stream_kernel", "kernel_ms": kern_ms / max(1, st["main_launches"]),
                         "alg_ops_per_decision": 8},
            "cpu_baseline": cpu,
            "e2e": None, "e2e_note": "the fleet (262 GB) does not fit in host pinned memory; see cfg2 e2e",
            "gpu_launches": int(st["launches_total"]), "clocks": clk,
            "best_config": best[0], "feasible": best[2]}
    if parity is not None:
        line["parity_sample_ok"] = parity
    if rank == 0:
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_bound(args):
    """NEXT f2: offline-optimal schedules (DP) on the workload, n_lambda weights.
    Unit: trace-sample x lambda.  ALU-bound on the fp64 pipe: ~12 fp64 ops per
    (trace-sample, lambda, level) (stretch, tau, energy, cost, 3 path sums);
    peak = 148 SMs x 64 fp64 lanes x clock (B200 fp64 rate, half of fp32)."""
    import torch

    import oracle
    import paper_conf_sc_zhengspl25_b200 as magus
    N, T, _, kind, _, desc = WORKLOADS[args.config]
    if args.n_traces:
        N = args.n_traces
    if args.n_steps:
        T = args.n_steps
    lams = [0.0] + [10.0 * 4 ** i for i in range(args.bound - 1)]
    L = (22 - 8 + 1) if args.full_grid else 2
    ctx = magus.Context(device=0)
    x = ctx.gen_traces(SEED_BASE + args.config, N, T, kind=kind)
    for _ in range(args.warmup):
        out = ctx.offline_bound(x, lams, full_grid=args.full_grid)
    torch.cuda.synchronize()
    clocks = ClockSampler(0)
    clocks.start()
    time.sleep(0.2)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clocks.mark()
    e0.record()
    for _ in range(args.steps):
        out = ctx.offline_bound(x, lams, full_grid=args.full_grid)
        out[0, 0, 0].item()  # device->host read of the result
    e1.record()
    torch.cuda.synchronize()
    clocks.mark()
    clocks.stop()
    ms = e0.elapsed_time(e1) / args.steps
    units = N * T * len(lams)
    value = units / (ms * 1e-3)
    clk = clocks.summary()
    sm_mhz = clk.get("sm_max_mhz") or 1965.0
    peak = 148 * 64 * sm_mhz * 1e6 / 1e9
    ach = 12.0 * L * units / (ms * 1e-3) / 1e9
    # parity of a few traces against the oracle's DP (untimed)
    got = out.cpu().numpy()
    xs = x[:, :4].cpu().numpy()
    parity = all(np.array_equal(got[n, j], oracle.offline_bound(xs[:, n], lam, full_grid=args.full_grid))
                 for n in range(4) for j, lam in enumerate(lams))
    line = {"metric": "trace-samples x lambdas/sec (NEXT f2 offline-optimal DP)", "value": value,
            "unit": "trace-samples*lambdas/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": desc, "n_traces": N, "n_steps": T, "lambdas": lams,
                                             "levels": L},
            "roofline": {"bound": "alu", "achieved": ach, "peak": peak, "unit": "Gop/s (fp64)",
                         "frac": ach / peak, "traffic": None, "alg_ops_per_unit_level": 12,
                         "peak_source": f"148 SMs x 64 fp64 lanes x {sm_mhz:.0f} MHz"},
            "gpu_launches": int(ctx.stats()["launches_total"]), "clocks": clk, "parity_sample_ok": bool(parity)}
    print(json.dumps(line), flush=True)
    ctx.close()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", type=int, default=2, choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n-traces", type=int, default=0)
    ap.add_argument("--n-steps", type=int, default=0)
    ap.add_argument("--no-decisions", action="store_true")
    ap.add_argument("--waves", type=int, default=0, help="MAGUS_OPT_WAVES (0 = library default)")
    ap.add_argument("--segments", type=int, default=0, help="MAGUS_OPT_SEGMENTS (0 = auto)")
    ap.add_argument("--bundle", type=int, default=0, help="MAGUS_OPT_BUNDLE (0 = auto, 1, 2, 4)")
    ap.add_argument("--sync-sweep", action="store_true",
                    help="host-synchronous magus_sweep_best each step (default: the async device choice)")
    ap.add_argument("--bound", type=int, default=0,
                    help="NEXT f2: time magus_offline_bound with this many lambdas instead of the replay")
    ap.add_argument("--full-grid", action="store_true", help="f2 over every ratio, not {min, max}")
    ap.add_argument("--variant", type=int, default=0, help="NEXT f3 (1 closed loop) / f4 (2 gradual)")
    ap.add_argument("--step", type=int, default=1, help="ratio step of the gradual variant")
    ap.add_argument("--spec-warm", type=int, default=0, help="f3 speculation warm-up rounds (0 auto)")
    ap.add_argument("--kernel", type=int, default=0, help="MAGUS_OPT_KERNEL (0 auto; 5 = speculative f3)")
    ap.add_argument("--cpu-threads", type=int, default=0, help="host threads of the oracle legs (0 = all cores)")
    ap.add_argument("--comm", choices=["torch", "native"], default="torch",
                    help="the totals all-reduce: torch.distributed NCCL, or the library's own (magus_comm_init)")
    ap.add_argument("--inflight", type=int, default=2,
                    help="consecutive steps in flight on separate streams/contexts (1 = strictly serial)")
    ap.add_argument("--burst", type=float, default=0.0,
                    help="NEXT f1: Sec. 6.3 burst threshold (MB/s); > 0 enables the Jaccard counters")
    ap.add_argument("--chunk", type=int, default=0, help="cfg4: intervals per time chunk (0 = fit ~32 GiB)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.bound > 0 and args.impl == "ours":
        return run_bound(args)
    if args.impl == "reference":
        return run_reference(args)
    if args.config == 4:
        return run_fleet(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
