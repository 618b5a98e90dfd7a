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
    # cfg: (n_traces, n_steps, grid, kind, decisions, scaling, what)
    #   scaling "weak": n_traces per GPU (BASELINE quotes configs 1-3 on one B200);
    #   "strong": n_traces is the whole fleet, sharded over the GPUs (configs 4, 5)
    1: (1, 10_000, "default", 0, True, "weak", "1 config (paper_default)"),
    2: (4096, 100_000, "default", 0, True, "weak", "1 config (paper_default)"),
    3: (4096, 100_000, "sweep256", 0, False, "weak", "256 configs (SWEEP256)"),
    4: (65536, 1_000_000, "fleet64", 0, False, "strong", "64 configs (FLEET64)"),
    5: (16384, 1_000_000, "default", 1, False, "strong", "1 config (paper_default), adversarial traces"),
}
METRIC = "trace-samples x configs/sec"
UNIT = "trace-samples*configs/s"


def shape_for(cfg: int, world: int, shard_by: str, n_traces: int = 0, n_steps: int = 0):
    """(n_traces_total, n_steps, scaling) of a workload at `world` GPUs."""
    N, T, _, _, _, scaling, _ = WORKLOADS[cfg]
    N = n_traces or N
    T = n_steps or T
    if shard_by == "configs":
        return N, T, "strong"          # every rank holds the whole fleet, configs are split
    return (N * world if scaling == "weak" else N), T, scaling


def workload_config(cfg: int, world: int, shard_by: str, n_traces: int = 0, n_steps: int = 0,
                    no_decisions: bool = False, n_configs: int | None = None) -> dict:
    """The `config` object of the JSON line; both arms build it with this
    function, so the reference arm reports exactly our arm's config."""
    _, _, grid, kind, want_dec, _, what = WORKLOADS[cfg]
    N_tot, T, scaling = shape_for(cfg, world, shard_by, n_traces, n_steps)
    C = n_configs if n_configs is not None else {"default": 1, "sweep256": 256, "fleet64": 64}[grid]
    want_dec = want_dec and not no_decisions
    per_gpu = N_tot if shard_by == "configs" else -(-N_tot // world)
    return {"workload": f"cfg{cfg}: {N_tot:,} traces x {T:,} intervals x {what}"
                        + ("" if world == 1 else f" over {world} GPUs"),
            "n_traces_total": N_tot, "n_traces_per_gpu": per_gpu, "n_steps": T, "n_configs": C,
            "decisions_emitted": want_dec, "seed": hex(SEED_BASE + cfg),
            "generator": "adversarial" if kind == 1 else "mix",
            "l2": f"inputs {per_gpu * T * 4 / 1e9:.2f} GB per GPU vs 126 MB L2 (no flush needed)"
                  if per_gpu * T * 4 > 4 * 126e6 else "inputs fit in L2: L2 flushed between steps",
            "parallelism": "1 GPU" if world == 1 else
                           f"{shard_by} sharded over {world} GPUs; 1 all-reduce of the int64 totals",
            "scaling": scaling}


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """SM clock + throttle reasons sampled DURING the timed region.

    NVML (pynvml) polled every ~2 ms from a thread, so even a few-ms timed
    region gets samples; falls back to `nvidia-smi -lms 50` without NVML.
    mark() brackets a window; summary() reports the samples inside the
    window(s) marked so far."""
    # nvmlClocksEventReason* bits
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int, period_s: float = 0.002):
        self.index = index
        self.period = period_s
        self.rows = []      # (time, sm_mhz, reasons set)
        self.smax = None
        self.proc = None
        self.stop_ev = threading.Event()
        self.marks = []
        self.source = None

    def _nvml_handle(self):
        import pynvml
        pynvml.nvmlInit()
        try:
            import torch
            p = torch.cuda.get_device_properties(self.index)
            bus = f"{p.pci_domain_id:08x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
            return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId(bus.encode())
        except Exception:
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.index)

    def start(self):
        try:
            nv, h = self._nvml_handle()
            self.smax = float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM))
            get_r = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons",
                            getattr(nv, "nvmlDeviceGetCurrentClocksThrottleReasons", None))

            def loop():
                while not self.stop_ev.is_set():
                    try:
                        sm = float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM))
                        r = int(get_r(h)) if get_r else 0
                        self.rows.append((time.time(), sm, {n for b, n in self.REASONS.items() if r & b}))
                    except Exception:
                        pass
                    self.stop_ev.wait(self.period)
            threading.Thread(target=loop, daemon=True).start()
            self.source = f"NVML every {self.period * 1e3:.0f} ms"
            return
        except Exception:
            pass
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "50", "-i", str(self.index)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read_smi, daemon=True).start()
            self.source = "nvidia-smi -lms 50"
        except Exception:
            self.proc = None

    def _read_smi(self):
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.proc.stdout:
            f = [x.strip() for x in line.strip().split(",")]
            try:
                sm, smax = float(f[0]), float(f[1])
            except Exception:
                continue
            self.smax = smax
            self.rows.append((time.time(), sm, {n for n, v in zip(names, f[4:8]) if v.lower() == "active"}))

    def mark(self):
        self.marks.append(time.time())

    def stop(self):
        self.stop_ev.set()
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def window(self, i0: int, i1: int):
        t0, t1 = self.marks[i0], self.marks[i1]
        return [r for r in self.rows if t0 <= r[0] <= t1]

    def summarize(self, rows, note=None):
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": self.smax, "reasons": ["no clock samples"], "samples": 0,
                    "source": self.source}
        sm = [r[1] for r in rows]
        reasons = set().union(*[r[2] for r in rows])
        out = {"sm_mhz": statistics.median(sm), "sm_min_mhz": min(sm), "sm_max_mhz": self.smax,
               "reasons": sorted(reasons), "samples": len(rows), "source": self.source}
        if note:
            out["note"] = note
        return out

    def summary(self):
        """Samples of the first marked window (the timed region)."""
        if len(self.marks) < 2:
            return self.summarize(self.rows, "no marked window: whole-run samples")
        return self.summarize(self.window(0, 1))


def clocks_line(clocks: ClockSampler, soak: bool):
    """The timed region's clocks; when it held fewer than 3 samples, the same
    steps were re-run untimed for >= 0.3 s right after (window 2-3) and those
    samples are reported with the timed ones."""
    c = clocks.summary()
    if soak and len(clocks.marks) >= 4 and c["samples"] < 3:
        rows = clocks.window(0, 1) + clocks.window(2, 3)
        c = clocks.summarize(rows, f"timed region held {c['samples']} sample(s): plus an untimed re-run of the "
                                   f"same steps for >= 0.3 s right after it")
    return c


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


def cpu_oracle_single(cfg, T, pols_oracle, kind, max_traces, budget_s=20.0, chunk=256):
    """SURVEY 8(d) protocol: the oracle on ONE host thread (no pool), over the
    first traces of the workload in blocks of `chunk` traces until the time
    budget is spent -- the whole of config 1, and of config 2 when the host is
    fast enough (the line says which)."""
    import gen
    import oracle
    n_done, dt = 0, 0.0
    while n_done < max_traces and dt < budget_s:
        n = min(chunk, max_traces - n_done)
        xs = gen.gen_traces(SEED_BASE + cfg, n, T, kind=kind, id0=n_done)
        t = time.perf_counter()
        oracle.replay(xs, pols_oracle)
        dt += time.perf_counter() - t
        n_done += n
    return n_done * T * len(pols_oracle) / dt, n_done, dt


def policies_for(grid):
    import paper_conf_sc_zhengspl25_b200 as magus
    if grid == "sweep256":
        return magus.grid_sweep256()
    if grid == "fleet64":
        return magus.grid_fleet64()
    return [magus.policy_preset(magus.POLICY_PAPER_DEFAULT)]


def oracle_grid(grid):
    """The oracle's own restatement of the grids (never the product's)."""
    import oracle
    if grid == "sweep256":
        return oracle.grid_sweep256()
    if grid == "fleet64":
        return oracle.grid_fleet64()
    return oracle.policy()


def oracle_policies(pols):
    import oracle
    return oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc,
                                 tau_dec=p.tau_dec, t_hi=p.t_hi, variant=p.variant, step=p.step)
                            for p in pols])


def host_info() -> dict:
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.lower().startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    if model is None:
        try:
            for ln in open("/proc/cpuinfo"):
                if ln.startswith("model name"):
                    model = ln.split(":", 1)[1].strip()
                    break
        except Exception:
            pass
    return {"cpu_model": model, "nproc": os.cpu_count(), "affinity_cores": host_cores()}


def run_reference(args):
    """--impl reference: the oracle, as it stands, timed on the host cores on
    our arm's config / metric / unit.  Each step replays as much of the
    workload as fits the time budget (the whole of config 2 on a 16-core
    host); the line says whether that is the whole workload.  Only oracle/
    and gen/ are loaded: the product library is not touched."""
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    import gen
    import oracle
    _, _, grid, kind, _, _, _ = WORKLOADS[args.config]
    cfgd = workload_config(args.config, world, args.shard, args.n_traces, args.n_steps, args.no_decisions)
    N, T, C = cfgd["n_traces_total"], cfgd["n_steps"], cfgd["n_configs"]
    pols = oracle_grid(grid)
    seed = SEED_BASE + args.config
    threads = args.cpu_threads or host_cores()
    # probe: single-thread time per trace x config on a small sample of this workload
    pc = pols[:min(len(pols), 4)]
    probe_n = max(1, min(N, 8))
    xp = gen.gen_traces(seed, probe_n, T, kind=kind)
    t = time.perf_counter()
    oracle.replay(xp, pc)
    per_unit = (time.perf_counter() - t) / (probe_n * len(pc))      # s per trace x config, 1 thread
    budget = args.ref_budget / max(1, args.steps + args.warmup)       # s per step
    n_cfg = C if per_unit * C * threads <= budget * threads else max(1, min(C, 16))
    n_tr = int(budget * threads / max(per_unit * n_cfg, 1e-12))
    n_tr = max(min(threads, N), min(N, n_tr))
    xs = gen.gen_traces(seed, n_tr, T, kind=kind)
    use = pols[:n_cfg]
    pool = OraclePool(threads)
    # the first warm-up step re-calibrates at the step's real stride (the
    # oracle reads each trace with stride ld, so the small probe is optimistic)
    t = time.perf_counter()
    pool.replay(xs, use)
    per_trace = (time.perf_counter() - t) / n_tr
    n_new = max(min(threads, N), min(N, int(budget / max(per_trace, 1e-12))))
    if n_new < n_tr:
        n_tr = n_new
        xs = gen.gen_traces(seed, n_tr, T, kind=kind)
    for _ in range(args.warmup - 1):
        pool.replay(xs, use)
    times = []
    for _ in range(args.steps):
        t = time.perf_counter()
        pool.replay(xs, use)
        times.append(time.perf_counter() - t)
    pool.close()
    dt = sum(times) / len(times)
    cores = min(threads, n_tr)
    value = n_tr * T * n_cfg / dt
    whole = n_tr == N and n_cfg == C
    sample = (f"{n_tr} of {N} trace(s) x {T} intervals x {n_cfg} of {C} config(s) per step (seed {seed:#x}), "
              f"statically partitioned over {cores} host thread(s)" + (" -- the whole workload" if whole else ""))
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3,
            "step_ms": {"mean": dt * 1e3, "median": statistics.median(times) * 1e3, "best": min(times) * 1e3,
                        "n": len(times)},
            "higher_is_better": True, "scaling": cfgd["scaling"], "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": cfgd, "whole_workload_per_step": whole,
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                             "host": host_info()},
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

    _, _, grid, kind, _, _, _ = WORKLOADS[args.config]
    cfgd = workload_config(args.config, world, args.shard, args.n_traces, args.n_steps, args.no_decisions)
    N_tot, T, want_dec, scaling = cfgd["n_traces_total"], cfgd["n_steps"], cfgd["decisions_emitted"], cfgd["scaling"]
    pols_all = policies_for(grid)
    if args.variant:  # NEXT f3 / f4: closed loop (seq_kernel) / gradual step (walk kernels)
        for p in pols_all:
            p.variant = args.variant
            p.step = args.step if args.variant & magus.VARIANT_GRADUAL else 0
    C_all = len(pols_all)
    if args.shard == "configs":      # this rank: every trace, its block of configs
        id0, N = 0, N_tot
        c0, nc = mdist.shard_configs(C_all, world, rank)
    else:                            # this rank: its block of traces, every config
        id0, N = mdist.shard(N_tot, world, rank)
        c0, nc = 0, C_all
    pols = pols_all[c0:c0 + nc]
    C = len(pols)
    seed = SEED_BASE + args.config
    plat = magus.platform_preset()
    if args.burst > 0:  # NEXT f1: Sec. 6.3 burst Jaccard counters in the same pass
        plat.burst_mbs = args.burst
    opts = [(magus.OPT_WAVES, args.waves), (magus.OPT_SEGMENTS, args.segments), (magus.OPT_BUNDLE, args.bundle),
            (magus.OPT_SPEC_WARM, args.spec_warm), (magus.OPT_KERNEL, args.kernel), (magus.OPT_WALK1, args.walk1)]
    ctx = magus.Context(device=local, stream=stream, platform=plat)
    for k, v in opts:
        if v:
            ctx.set_option(k, v)
    x = ctx.gen_traces(seed, N, T, kind=kind, id0=id0)
    torch.cuda.synchronize()
    # inputs that fit in L2 are flushed before every step (outside the step's events)
    flush = None
    if N * T * 4 <= 4 * 126e6:
        flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)   # 256 MB > L2

    # --inflight 2: consecutive steps alternate between two contexts on two
    # streams (own scratch, outputs and choice buffers; the traces are
    # shared, read-only), so one step's tail overlaps the next step's head
    lanes = [[ctx, stream, None, None, None]]
    if args.inflight > 1 and flush is None:
        s2 = torch.cuda.Stream(dev)
        ctx2 = magus.Context(device=local, stream=s2, platform=plat)
        for k, v in opts:
            if v:
                ctx2.set_option(k, v)
        lanes.append([ctx2, s2, None, None, None])
    if args.shard == "configs":
        for ln in lanes:
            ln[4] = torch.zeros((C_all, magus.TOT_WORDS), dtype=torch.int64, device=dev)
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
        # the synchronous magus_sweep_best).  Returns (lane stream, choice).
        ln = lanes[nstep[0] % len(lanes)]
        nstep[0] += 1
        c_, s_, o_, b_, full = ln
        with torch.cuda.stream(s_):
            o_ = c_.replay(x, pols, want_summary=False, want_base=False, want_decisions=want_dec,
                           want_totals=True, out=o_)
            tot = o_.totals
            if full is not None:               # config shard: this rank's rows of [C_all x 18]
                full.zero_()
                full[c0:c0 + nc].copy_(tot)
                tot = full
            if args.comm == "native":          # the library's own NCCL communicator
                c_.allreduce_totals(tot)
            else:
                mdist.allreduce_totals(tot)    # the one collective; exact (integer words)
            ln[2] = o_
            if args.sync_sweep:
                return s_, c_.sweep_best(tot)
            b_ = c_.sweep_best_async(tot, b_)
        ln[3] = b_
        return s_, b_

    def result(r):
        return r if args.sync_sweep else ctx.sweep_result(r)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.2)
    for ln in lanes:
        ln[0].set_option(magus.OPT_TIMING, 1)
        ln[0].reset_stats()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    e0, e1 = ev(), ev()
    ends = []
    per_step = []     # (start, end) events of each step when L2 is flushed between steps
    clocks.mark()
    e0.record(stream)
    for ln in lanes[1:]:
        ln[1].wait_event(e0)
    for _ in range(args.steps):
        if flush is not None:
            flush.zero_()
            a = ev()
            a.record(stream)
        s_, best = step()
        d = ev()
        d.record(s_)
        ends.append(d)
        if flush is not None:
            per_step.append((a, d))
    for ln in lanes[1:]:
        done_ev = torch.cuda.Event()
        done_ev.record(ln[1])
        stream.wait_event(done_ev)
    e1.record(stream)
    torch.cuda.synchronize()
    clocks.mark()
    best = result(best)
    if world > 1:
        dist.barrier()
    if per_step:
        steps_ms = [a.elapsed_time(d) for a, d in per_step]
        ms = sum(steps_ms)
    else:
        ms = e0.elapsed_time(e1)
        done = [0.0] + sorted(e0.elapsed_time(d) for d in ends)
        # the step period over a window of as many steps as are in flight
        # (consecutive completions of overlapping steps alternate short / long)
        L = max(1, len(lanes))
        steps_ms = [(done[i] - done[max(0, i - L)]) / min(i, L) for i in range(1, len(done))]
    st = ctx.stats()
    for ln in lanes[1:]:  # launches of every context in flight
        s2 = ln[0].stats()
        for key in ("launches_total", "main_launches", "main_ms_total"):
            st[key] += s2[key]
    for ln in lanes:
        ln[0].set_option(magus.OPT_TIMING, 0)
    soak = ms < 100.0
    if soak:  # the same steps, untimed, for >= 0.3 s: clock samples under this load
        clocks.mark()
        t = time.time()
        while time.time() - t < 0.3:
            for _ in range(8):
                step()
            torch.cuda.synchronize()
        clocks.mark()
    time.sleep(0.05)
    clocks.stop()
    # the dominant kernel ALONE: serial steps on one context after the timed
    # region, CUDA events around each launch on its stream (this is the
    # roofline's kernel time; with steps in flight the in-region event times
    # include the other stream's share of the GPU)
    serial_ms = None
    if len(lanes) > 1:
        torch.cuda.synchronize()
        ctx.set_option(magus.OPT_TIMING, 1)
        ctx.reset_stats()
        for _ in range(min(50, max(10, args.steps))):
            o = ctx.replay(x, pols, want_summary=False, want_base=False, want_decisions=want_dec,
                           want_totals=True, out=lanes[0][2])
            lanes[0][2] = o
            torch.cuda.synchronize()
        s1 = ctx.stats()
        ctx.set_option(magus.OPT_TIMING, 0)
        serial_ms = s1["main_ms_total"] / max(1, s1["main_launches"])
    kern_ms = st["main_ms_total"] / max(1, st["main_launches"])
    if world > 1:
        t = torch.tensor([ms, kern_ms, serial_ms or 0.0], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms, kern_ms = float(t[0].item()), float(t[1].item())
        serial_ms = float(t[2].item()) if serial_ms is not None else None
    ms_per_step = ms / args.steps
    units_per_step = N_tot * T * C_all
    value = units_per_step / (ms_per_step * 1e-3)

    # roofline of the dominant kernel, from live CUDA events
    peak, peak_src = _peaks()
    alone_ms = serial_ms if serial_ms is not None else kern_ms
    alg_bytes = N * T * 4 + (C * N * T / 8 if want_dec else 0)      # per launch on this rank
    traffic = None
    kname = {1: "ref_kernel", 2: "family_kernel" if st.get("last_family") else "stream_kernel", 3: "seq_kernel",
             4: ("walk_fused_kernel + walk_final_kernel" if args.walk1
                 else "walk_map_kernel + walk_replay_kernel + walk_final_kernel"),
             5: "spec_kernel + spec_fix_kernel"}.get(st["last_kernel"], "?")
    vtag = {0: "", 1: "_f3", 2: "_f4"}.get(args.variant, f"_v{args.variant}")
    # traffic only from an ncu capture of this very kernel and workload
    prof = os.path.join(ROOT, "profiles", f"ncu_cfg{args.config}{vtag}.json")
    ncu = {}
    if os.path.exists(prof) and world == 1:
        try:
            with open(prof) as f:
                ncu = json.load(f)
            traffic = ncu.get("dram_bytes_per_launch")
        except Exception:
            ncu = {}
    clk = clocks_line(clocks, soak)
    method = ("algorithmic bytes per launch / the launch's CUDA-event duration on its stream, the kernel "
              "timed alone" + (" (serial launches after the timed region)" if serial_ms is not None else ""))
    hbm_roof = {"bound": "hbm", "achieved": alg_bytes / (alone_ms * 1e-3) / 1e9, "peak": peak, "unit": "GB/s",
                "traffic": traffic, "peak_source": peak_src, "kernel": kname, "kernel_ms": alone_ms,
                "alg_bytes_per_launch": alg_bytes, "method": method}
    hbm_roof["frac"] = hbm_roof["achieved"] / peak
    if len(lanes) > 1:
        agg = alg_bytes * args.steps / (ms * 1e-3) / 1e9
        hbm_roof["aggregate"] = {"achieved": agg, "frac": agg / peak, "steps_in_flight": len(lanes),
                                 "note": "algorithmic bytes of all launches / timed region with consecutive "
                                         "steps overlapping on two streams (not a per-kernel number)"}
    roof = hbm_roof
    if C > 1:
        # C > 1 sweeps are ALU-bound: 8 lane-ops per decision
        # (SURVEY 8(d)); peak = 148 SMs x 4 SMSPs x 32 lanes x max SM clock
        sm_mhz = clk.get("sm_max_mhz") or 1965.0
        alu_peak = 148 * 4 * 32 * sm_mhz * 1e6 / 1e9   # Gop/s
        ach = 8.0 * N * T * C / (alone_ms * 1e-3) / 1e9
        roof = {"bound": "alu", "achieved": ach, "peak": alu_peak, "unit": "Gop/s", "frac": ach / alu_peak,
                "traffic": traffic,
                "peak_source": f"148 SMs x 128 lanes x {sm_mhz:.0f} MHz (B200_PROFILING.md unit counts)",
                "kernel": kname, "kernel_ms": alone_ms, "alg_ops_per_decision": 8, "method": method}
        if ncu.get("metrics", {}).get("smsp__issue_active.avg.pct_of_peak_sustained_active"):
            roof["ncu_issue_active_frac"] = float(
                ncu["metrics"]["smsp__issue_active.avg.pct_of_peak_sustained_active"]["value"]) / 100
            roof["ncu_thread_inst_per_decision"] = ncu.get("thread_instructions_per_unit")
        if len(lanes) > 1:
            agg = 8.0 * N * T * C * args.steps / (ms * 1e-3) / 1e9
            roof["aggregate"] = {"achieved": agg, "frac": agg / alu_peak, "steps_in_flight": len(lanes)}

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
                full = torch.zeros((C_all, magus.TOT_WORDS), dtype=torch.int64)
                full[c0:c0 + nc] = torch.from_numpy(tot.view(np.int64))
                mdist.allreduce_totals(full.to(dev)).cpu()
        el = time.perf_counter() - t
        if world > 1:
            tmax = torch.tensor([el], dtype=torch.float64, device=dev)
            dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
            el = float(tmax.item())
        e2e = {"value": units_per_step * e2e_steps / el, "unit": UNIT,
               "h2d_bytes_per_step": N * T * 4 * world, "d2h_bytes_per_step": C * magus.TOT_WORDS * 8 * world,
               "steps": e2e_steps, "path": "magus_replay_host (pinned host traces; wall clock, max over ranks)"}

    cpu = None
    parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        pol_o = oracle_policies(pols)
        if C > 16:
            pol_o = pol_o[:16]
        threads = args.cpu_threads or host_cores()
        v, n_s, dt_s, ref_summ = cpu_oracle_sample(args.config, T, pol_o, args.cpu_budget, kind, max_traces=N,
                                                   threads=threads)
        v1, n1, dt1 = cpu_oracle_single(args.config, T, pol_o, kind, max_traces=N)
        cpu = {"value": v, "unit": UNIT, "cores": min(threads, n_s), "kind": "oracle",
               "sample": f"first {n_s} traces x {T} intervals x {len(pol_o)} config(s) of the same workload, "
                         f"statically partitioned over {min(threads, n_s)} host thread(s) ({dt_s:.1f} s)",
               "single_thread": {"value": v1, "unit": UNIT, "whole_workload": n1 == N and len(pol_o) == C,
                                 "sample": f"first {n1} of {N} traces x {T} intervals x {len(pol_o)} config(s), "
                                           f"one thread, blocks of 256 traces, 20 s budget ({dt1:.1f} s)"},
               "host": host_info()}
        # parity of that sample against the GPU path (untimed)
        r = ctx.replay(x[:, :n_s], pols[:len(pol_o)], n_traces=n_s, want_totals=False)
        torch.cuda.synchronize()
        got = r.summary_numpy()
        parity = bool(all(np.array_equal(got[g], ref_summ[o]) for g, o in
                          [("n_events", "n_events"), ("n_changes", "n_changes"), ("digest", "digest"),
                           ("energy_j", "energy"), ("time_s", "time")]))

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step,
            "step_ms": {"mean": ms_per_step, "median": statistics.median(steps_ms), "best": min(steps_ms),
                        "n": len(steps_ms),
                        "method": "per-step CUDA events around each step" if per_step else
                                  "step-completion events: (t_i - t_(i-L)) / L over L = steps in flight"},
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": cfgd,
            "run": {"steps_in_flight": len(lanes), "segments": st["last_segments"],
                    "kernel": {1: "reference", 2: "stream", 3: "sequential", 4: "walk", 5: "spec"}.get(
                        st["last_kernel"], "?"),
                    "variant": args.variant, "step": args.step if args.variant & 2 else 0,
                    "comm": "native NCCL" if args.comm == "native" and world > 1 else dist_backend(world),
                    "configs_this_rank": [c0, nc], "traces_this_rank": [id0, N],
                    "ranks_per_gpu": max(1, world // max(1, torch.cuda.device_count())),
                    "l2_flush": flush is not None},
            "roofline": roof,
            "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": int(st["launches_total"]), "clocks": clk,
            "best_config": best[0], "feasible": best[2]}
    if args.t1_ms:
        line["scaling_efficiency"] = {
            "value": args.t1_ms / ((world if scaling == "strong" else 1) * ms_per_step),
            "t1_ms": args.t1_ms, "tN_ms": ms_per_step,
            "formula": "t1 / (G * tG)" if scaling == "strong" else "t1 / tG (weak)"}
    if args.burst > 0:
        line["config"]["burst_mbs"] = args.burst
        line["best_jaccard"] = best[1]["jaccard"]
        line["pareto_front"] = [int(i) for i in np.flatnonzero(ctx.pareto_front(lanes[0][2].totals))]
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
    N_tot, T, grid, kind, _, _, _ = WORKLOADS[4]
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
            "config": workload_config(4, world, "traces", args.n_traces, args.n_steps),
            "run": {"chunk_intervals": R, "chunks": len(chunks), "halo_rows": halo,
                    "l2": f"chunks of {N * R * 4 / 1e9:.1f} GB > 126 MB L2 (no flush needed)",
                    "timed": "replay calls + all-reduce + device choice; on-device generation of each "
                             "chunk and the halo copy untimed (SURVEY 8(d))",
                    "comm": dist_backend(world), "traces_this_rank": [id0, N]},
            "roofline": {"bound": "alu", "achieved": alu_ach, "peak": alu_peak, "unit": "Gop/s",
                         "frac": alu_ach / alu_peak, "traffic": None,
                         "peak_source": f"148 SMs x 128 lanes x {sm_mhz:.0f} MHz (B200_PROFILING.md unit counts)",
                         "kernel": "family_kernel" if st.get("last_family") else "stream_kernel",
                         "kernel_ms": kern_ms / max(1, st["main_launches"]),
                         "alg_ops_per_decision": 8,
                         "note": "the 8-op model of SURVEY 8(d) per decision; the kernel shares Alg. 1 work "
                                 "across the family, so the model rate can exceed the lane peak"},
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
    N, T, _, kind, _, _, _ = WORKLOADS[args.config]
    desc = workload_config(args.config, 1, "traces", args.n_traces, args.n_steps)["workload"]
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
    ctx.reset_stats()
    ctx.set_option(magus.OPT_TIMING, 1)  # CUDA events around each DP kernel (kernel alone)
    clocks.mark()
    e0.record()
    for _ in range(args.steps):  # steps queued back to back (inputs resident; one result read after)
        out = ctx.offline_bound(x, lams, full_grid=args.full_grid)
    e1.record()
    out[0, 0, 0].item()  # device->host read of the result
    torch.cuda.synchronize()
    clocks.mark()
    clocks.stop()
    ctx.set_option(magus.OPT_TIMING, 0)
    ms = e0.elapsed_time(e1) / args.steps
    stb = ctx.stats()
    kern_ms = stb["main_ms_total"] / max(1, stb["main_launches"])
    units = N * T * len(lams)
    value = units / (ms * 1e-3)
    clk = clocks.summary()
    sm_mhz = clk.get("sm_max_mhz") or 1965.0
    peak = 148 * 64 * sm_mhz * 1e6 / 1e9
    ach = 12.0 * L * units / (kern_ms * 1e-3) / 1e9  # the DP's algorithmic fp64 ops / the kernel alone
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
                         "peak_source": f"148 SMs x 64 fp64 lanes x {sm_mhz:.0f} MHz",
                         "kernel_ms": kern_ms, "kernel": {True: "bound_grid_free_kernel / bound_dp_kernel",
                                                          False: "bound_binary_shared_kernel"}[bool(args.full_grid)],
                         "method": "the DP's fp64 ops (12 per trace-sample, lambda and level, every level "
                                   "evaluated) / the kernel's CUDA-event time; the kernels skip most of that "
                                   "work (one add per step without a tie, DESIGN.md 11), so this is an "
                                   "algorithmic rate, not the fp64 pipe's utilisation"},
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
    ap.add_argument("--walk1", type=int, default=0, help="MAGUS_OPT_WALK1: 1 = the one-pass f4 walk (A/B)")
    ap.add_argument("--cpu-threads", type=int, default=0, help="host threads of the oracle legs (0 = all cores)")
    ap.add_argument("--comm", choices=["torch", "native"], default="torch",
                    help="the totals all-reduce: torch.distributed NCCL, or the library's own (magus_comm_init)")
    ap.add_argument("--inflight", type=int, default=2,
                    help="consecutive steps in flight on separate streams/contexts (1 = strictly serial)")
    ap.add_argument("--burst", type=float, default=0.0,
                    help="NEXT f1: Sec. 6.3 burst threshold (MB/s); > 0 enables the Jaccard counters")
    ap.add_argument("--chunk", type=int, default=0, help="cfg4: intervals per time chunk (0 = fit ~32 GiB)")
    ap.add_argument("--shard", choices=["traces", "configs"], default="traces",
                    help="multi-GPU split: trace blocks (default) or config blocks (every rank holds every trace)")
    ap.add_argument("--t1-ms", type=float, default=0.0,
                    help="1-GPU ms/step of the same workload: adds scaling_efficiency = t1/(G*tG) (strong) "
                         "or t1/tG (weak)")
    ap.add_argument("--ref-budget", type=float, default=150.0,
                    help="--impl reference: seconds of oracle work for the whole --steps + --warmup run")
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
