"""Developer probe (build with MAGUS_NVCC_FLAGS=-DWALK_STATS): how many 32-step
words of the one-pass walk kernel were carry-dependent (replayed after the
look-back) on the config-2 f4 workload."""
import sys
import torch
sys.path.insert(0, '.')
import paper_conf_sc_zhengspl25_b200 as magus
N, T = 4096, 100000
step = int(sys.argv[1]) if len(sys.argv) > 1 else 2
ctx = magus.Context(device=0)
x = ctx.gen_traces(0x4D41475553000002, N, T)
for segs in (0, 36, 143, 572):
    ctx.set_option(magus.OPT_SEGMENTS, segs)
    r = ctx.replay(x, [magus.make_policy(variant=2, step=step)], want_decisions=False)
    torch.cuda.synchronize()
    s = r.summary_numpy()[0]
    print("segments", ctx.stats()["last_segments"], "deferred words", int(s["n_burst_base"].sum()), "of",
          N * (T // 32), "lanes looking back", int(s["n_burst_magus"].sum()), flush=True)
