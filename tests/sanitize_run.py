"""Small replay workload for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck) runs of the TMA + mbarrier + look-back kernels.

  compute-sanitizer --tool racecheck python tests/sanitize_run.py

Exercises: several segments (look-back), a ragged trace group and tail word,
bundles (NB = 4, 128-trace CTAs), one config (the 512-trace CTA), bursts, decisions output, the per-sample kernel, the
sequential / speculative / walk kernels (level output), the DP kernels and the
family kernel (a sweep grid's (W, H) group per CTA).
Exits non-zero if the results disagree with the oracle.
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import gen  # noqa: E402
import oracle  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_zhengspl25_b200 as magus  # noqa: E402


def main():
    N, T = 200, 1500
    x = gen.gen_traces(gen.SEEDS[1], N, T)
    xd = torch.zeros((T, 200), dtype=torch.float32, device="cuda:0")
    xd[:, :N] = torch.from_numpy(x).cuda()
    pols = [magus.make_policy(t_hi=th) for th in (0.2, 0.3, 0.4)] + [magus.make_policy(W=7, H=13)]
    plat = magus.platform_preset()
    plat.burst_mbs = 12000.0
    po = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc, tau_dec=p.tau_dec,
                               t_hi=p.t_hi) for p in pols])
    ref = oracle.replay(x, po, oracle.platform(burst=12000.0), want_dec=True)
    ok = True
    with magus.Context(device=0, platform=plat) as ctx:
        # the bundles (128-trace CTAs), one config (the 512-trace CTA, its
        # totals initialised by the launch's first CTA), the per-sample kernel
        for kernel, segs, sub in ((magus.KERNEL_STREAM, 5, [0, 1, 2, 3]), (magus.KERNEL_STREAM, 5, [2]),
                                  (magus.KERNEL_REFERENCE, 0, [0, 1, 2, 3])):
            ctx.set_option(magus.OPT_KERNEL, kernel)
            ctx.set_option(magus.OPT_SEGMENTS, segs)
            r = ctx.replay(xd, [pols[i] for i in sub], n_traces=N, want_decisions=True)
            torch.cuda.synchronize()
            got = r.summary_numpy()
            ok &= bool(np.array_equal(got["energy_j"], ref.summary["energy"][sub]))
            ok &= bool(np.array_equal(got["digest"], ref.summary["digest"][sub]))
            ok &= bool(np.array_equal(r.decisions_numpy().transpose(0, 2, 1), oracle.decision_words(ref.dec[sub], 8)))
            for j, i in enumerate(sub):
                ok &= bool(np.array_equal(r.totals_numpy()[j], oracle.totals(ref.summary[i], ref.base, T,
                                                                             oracle.platform(burst=12000.0))[0]))
        # the sequential (f3), speculative (f3, every guess wrong at warm-up
        # 1) and walk (f4, several segments) kernels, with level output
        vpols = [magus.make_policy(variant=1), magus.make_policy(variant=2, step=2),
                 magus.make_policy(W=5, H=40, variant=2, step=3)]
        vpo = oracle.policies([dict(W=p.window, H=p.history, L=p.deriv_len, tau_inc=p.tau_inc, tau_dec=p.tau_dec,
                                    t_hi=p.t_hi, variant=p.variant, step=p.step) for p in vpols])
        vref = oracle.replay(x, vpo, oracle.platform(burst=12000.0), want_dec=True)
        runs = [(magus.KERNEL_SEQUENTIAL, vpols[:1], [0], 0, 0),        # f3: seq_kernel<closed, binary>
                (magus.KERNEL_SEQUENTIAL, vpols, [0, 1, 2], 0, 0),      # mixed: seq_kernel<closed, multi>
                (magus.KERNEL_SPEC, vpols[:1], [0], 7, 0),
                (magus.KERNEL_WALK, vpols[1:], [1, 2], 6, 0),
                (magus.KERNEL_WALK, vpols[1:], [1, 2], 6, 1)]           # the one-pass walk (OPT_WALK1)
        only = os.environ.get("SANITIZE_ONLY")  # e.g. "0,2,3": a subset of the runs above
        if only:
            runs = [runs[int(i)] for i in only.split(",")]
        for kernel, pp, idx, segs, walk1 in runs:
            ctx.set_option(magus.OPT_KERNEL, kernel)
            ctx.set_option(magus.OPT_WALK1, walk1)
            ctx.set_option(magus.OPT_SEGMENTS, segs)
            ctx.set_option(magus.OPT_SPEC_WARM, 1)
            lv, rr = ctx.replay_levels(xd, pp, n_traces=N)
            torch.cuda.synchronize()
            ok &= bool(np.array_equal(lv.cpu().numpy().transpose(0, 2, 1), vref.dec[idx].astype(np.uint8)))
            ok &= bool(np.array_equal(rr.summary_numpy()["energy_j"], vref.summary["energy"][idx]))
        ctx.set_option(magus.OPT_KERNEL, magus.KERNEL_AUTO)
        ctx.set_option(magus.OPT_SEGMENTS, 0)
        ctx.set_option(magus.OPT_WALK1, 0)
        for full in (False, True):  # f2: the scalar-path binary kernel, the two-lane grid kernel
            out = ctx.offline_bound(xd[:200, :8], [0.0, 100.0], full_grid=full)
            torch.cuda.synchronize()
            ok &= bool(np.array_equal(out.cpu().numpy()[3, 1],
                                      oracle.offline_bound(x[:200, 3], 100.0, full_grid=full)))
    # the family kernel (a sweep grid's (W, H) group in one CTA: mask warps,
    # bundle warps, TMA issued by a mask warp), several segments, decisions
    fpols = magus.grid_fleet64()
    fpo = oracle.grid_fleet64()  # the oracle's own restatement of the grid
    fref = oracle.replay(x, fpo, want_dec=True)
    with magus.Context(device=0) as ctx:
        ctx.set_option(magus.OPT_SEGMENTS, 3)
        r = ctx.replay(xd, fpols, n_traces=N, want_decisions=True)
        torch.cuda.synchronize()
        ok &= ctx.stats()["last_family"] == 1
        ok &= bool(np.array_equal(r.summary_numpy()["energy_j"], fref.summary["energy"]))
        ok &= bool(np.array_equal(r.summary_numpy()["digest"], fref.summary["digest"]))
        ok &= bool(np.array_equal(r.decisions_numpy().transpose(0, 2, 1), oracle.decision_words(fref.dec, 8)))
    print("sanitize workload parity:", "ok" if ok else "MISMATCH")
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
