"""Developer probe: time the f2 full-grid / binary DP on synthetic inputs of
controlled stretch density (all below the r_min capacity, the mix traces,
all above it)."""
import sys
import torch
import paper_conf_sc_zhengspl25_b200 as magus

full = "--binary" not in sys.argv
N, T = 4096, 20000
lams = [0.0, 10.0, 40.0, 160.0] if full else [0.0, 10.0, 40.0, 160.0, 640.0, 2560.0, 10240.0, 40960.0]
with magus.Context(device=0) as ctx:
    mix = ctx.gen_traces(seed=7, n_traces=N, n_steps=T)
    cases = {"zero": torch.zeros_like(mix), "mix": mix, "high": torch.full_like(mix, 30000.0)}
    for name, x in cases.items():
        for _ in range(2):
            ctx.offline_bound(x, lams, full_grid=full)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3):
            ctx.offline_bound(x, lams, full_grid=full)
        e1.record()
        torch.cuda.synchronize()
        print(name, "ms per 1e5 steps:", round(e0.elapsed_time(e1) / 3 * (100000 / T), 2))
