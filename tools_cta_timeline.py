"""Per-CTA timeline of the stream kernel (MAGUS_OPT_TRACE) on a BASELINE
config: where the launch's time goes (ramp, scan spread, look-back wait,
finalisation tail) and how CTAs per SM shape it.  Diagnostics only.

  python tools_cta_timeline.py [--config 2] [--segments S] [--reps 5]
"""
from __future__ import annotations

import argparse
import collections
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)


def main():
    import torch

    import bench
    import paper_conf_sc_zhengspl25_b200 as magus
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--segments", type=int, default=0)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--no-decisions", action="store_true")
    ap.add_argument("--narrow", action="store_true", help="MAGUS_OPT_NARROW: 128-trace CTAs")
    ap.add_argument("--raw", default="", help="save every rep's raw timeline (npy) under this prefix")
    a = ap.parse_args()
    N, T, grid, kind, want_dec, _, _ = bench.WORKLOADS[a.config]
    want_dec = want_dec and not a.no_decisions
    pols = bench.policies_for(grid)
    ctx = magus.Context(device=0)
    if a.segments:
        ctx.set_option(magus.OPT_SEGMENTS, a.segments)
    if a.narrow:
        ctx.set_option(magus.OPT_NARROW, 1)
    x = ctx.gen_traces(bench.SEED_BASE + a.config, N, T, kind=kind)
    out = None
    for _ in range(3):
        out = ctx.replay(x, pols, want_summary=False, want_base=False, want_decisions=want_dec, out=out)
    torch.cuda.synchronize()
    ctx.set_option(magus.OPT_TRACE, 1)
    ctx.set_option(magus.OPT_TIMING, 1)
    res = []
    for _ in range(a.reps):
        ctx.reset_stats()
        out = ctx.replay(x, pols, want_summary=False, want_base=False, want_decisions=want_dec, out=out)
        torch.cuda.synchronize()
        ev_ms = ctx.stats()["main_ms_total"]
        tr = ctx.trace().astype(np.int64)
        if a.raw:
            np.save(f"{a.raw}_{len(res)}.npy", tr)
        t0 = tr[:, 0].min()
        st, scan, look, end = ((tr[:, i] - t0) / 1e3 for i in range(4))   # us
        sm = tr[:, 4]
        per_sm = collections.Counter(sm.tolist())
        ctas_on = np.array([per_sm[v] for v in sm])
        d = {"event_ms": ev_ms, "ctas": len(tr), "sms_used": len(per_sm),
             "ctas_per_sm_hist": dict(collections.Counter(per_sm.values())),
             "start_us": [float(st.min()), float(np.median(st)), float(st.max())],
             "scan_end_us": [float(scan.min()), float(np.median(scan)), float(scan.max())],
             "scan_dur_us_by_ctas_per_sm": {int(k): float(np.median((scan - st)[ctas_on == k]))
                                            for k in sorted(set(ctas_on.tolist()))},
             "lookback_wait_us": [float(np.median(look - scan)), float((look - scan).max())],
             "end_us": [float(end.min()), float(np.median(end)), float(end.max())],
             "finaliser_end_us": float(end[tr[:, 7] == 1].max()) if (tr[:, 7] == 1).any() else None,
             "last_scan_end_us": float(scan.max()),
             "by_segment_scan_end_us": {int(s): float(scan[tr[:, 5] == s].max()) for s in
                                        sorted(set(tr[:, 5].tolist()))[:4]}}
        res.append(d)
    print(json.dumps(res[-1]))
    print(json.dumps({"event_ms_all": [r["event_ms"] for r in res],
                      "end_max_us_all": [r["end_us"][2] for r in res]}))


if __name__ == "__main__":
    main()
