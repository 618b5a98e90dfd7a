"""Summarise one ncu --set full capture of the stream kernel into the JSON kept
under profiles/ (dev tool; bench.py reads `dram_bytes_per_launch` from it for
the roofline's `traffic` field).

    python tools_ncu_summary.py gpurun_out/prof_cfg2.ncu-rep profiles/ncu_cfg2.json \
        --workload "cfg2 ..." --command "ncu ..." --alg-bytes 1689600000
"""
from __future__ import annotations

import argparse
import collections
import csv
import io
import json
import subprocess

METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "launch__grid_size",
    "launch__block_size", "smsp__inst_executed.sum", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_tma.avg.pct_of_peak_sustained_active", "gpc__cycles_elapsed.max",
    "sm__cycles_active.avg", "smsp__cycles_active.avg", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
]
SCALE = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def ncu(rep: str, page: str, extra=()) -> list[list[str]]:
    out = subprocess.run(["ncu", "-i", rep, "--page", page, "--csv", *extra], capture_output=True, text=True,
                         check=True).stdout
    return list(csv.reader(io.StringIO(out)))


def main() -> None:
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("out")
    ap.add_argument("--workload", default="")
    ap.add_argument("--command", default="")
    ap.add_argument("--alg-bytes", type=float, default=0.0)
    ap.add_argument("--units", type=float, default=0.0, help="trace-samples x configs of the launch")
    ap.add_argument("--round", type=int, default=1)
    a = ap.parse_args()
    rows = ncu(a.rep, "raw")
    hdr, units, vals = rows[0], rows[1], rows[2]
    m = {}
    for name in METRICS:
        if name in hdr:
            i = hdr.index(name)
            m[name] = {"value": vals[i], "unit": units[i]}
    kname = vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else ""

    def nbytes(name):
        v = m.get(name)
        return float(v["value"]) * SCALE.get(v["unit"], 1.0) if v else 0.0

    rd, wr = nbytes("dram__bytes_read.sum"), nbytes("dram__bytes_write.sum")
    res = {"round": a.round, "kernel": kname, "workload": a.workload, "command": a.command,
           "dram_bytes_per_launch": rd + wr, "dram_read_bytes": rd, "dram_write_bytes": wr,
           "alg_bytes_per_launch": a.alg_bytes or None, "metrics": m}
    if len(rows) > 3:  # several kernels make one replay (e.g. the walk passes): sum their traffic
        ks = []
        for r in rows[2:]:
            d = dict(zip(hdr, r))
            u = dict(zip(hdr, units))

            def b(name):
                return float(d[name]) * SCALE.get(u[name], 1.0) if name in d and d[name] else 0.0
            ks.append({"kernel": d.get("Kernel Name", ""), "time": d.get("gpu__time_duration.sum"),
                       "time_unit": u.get("gpu__time_duration.sum"),
                       "dram_bytes": b("dram__bytes_read.sum") + b("dram__bytes_write.sum"),
                       "warp_instructions": d.get("smsp__inst_executed.sum"),
                       "issue_active_pct": d.get("smsp__issue_active.avg.pct_of_peak_sustained_active")})
        res["kernels"] = ks
        res["dram_bytes_per_launch"] = sum(k["dram_bytes"] for k in ks)
        res["kernel"] = " + ".join(k["kernel"].split("(")[0] for k in ks)
    # executed-instruction mix and warp-stall reasons from the source page
    try:
        src = ncu(a.rep, "source", ["--print-source", "sass"])
        h = src[1]
        ix = {k: i for i, k in enumerate(h)}
        ops, stalls = collections.Counter(), collections.Counter()
        total = samples = 0
        for r in src[2:]:
            if len(r) < len(h) or not r[ix["Source"]].strip() or r == h:
                continue  # (a multi-kernel report repeats the header per kernel)
            if not r[ix["Instructions Executed"]].strip().isdigit():
                continue
            n = int(r[ix["Instructions Executed"]] or 0)
            total += n
            toks = r[ix["Source"]].split()
            op = (toks[1] if toks[0].startswith("@") else toks[0]).split(".")[0]
            ops[op] += n
            samples += int(r[ix["# Samples"]] or 0)
            for k in h:
                if k.startswith("stall_") and "(Not" not in k:
                    stalls[k] += int(r[ix[k]] or 0)
        res["warp_instructions"] = total
        if a.units:
            res["thread_instructions_per_unit"] = total * 32 / a.units
            res["instruction_mix_per_unit"] = {k: round(v * 32 / a.units, 3) for k, v in ops.most_common(24)}
        res["stall_fraction"] = {k: round(v / max(1, samples), 3) for k, v in stalls.most_common(12)}
    except subprocess.CalledProcessError:
        pass
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps({k: res[k] for k in ("dram_bytes_per_launch", "alg_bytes_per_launch")}))


if __name__ == "__main__":
    main()
