"""configs[0] (20x30x10) step anatomy: host-measured waxpby / solve / maxabsdiff times with L2 flushed before each step, for 1, 2 and 150 CG iterations (on-chip cluster kernel)."""
import os, sys, time
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
ctx = H.Context(0)
p = H.Problem(ctx, 20, 30, 10)
p.set_option(H.HPCCG_OPT_GRAPH, 1)
xp = p.vec_ptr(H.HPCCG_VEC_X)
n = p.n
flush = torch.empty(64 << 20, dtype=torch.float64, device="cuda")
for variant in (0, 1):
    p.set_option(H.HPCCG_OPT_CG_VARIANT, variant)
    for it in (1, 2, 150):
        ts, tw, tm, tall = [], [], [], []
        for rep in range(8):
            flush.zero_(); torch.cuda.synchronize()
            t0 = time.perf_counter()
            ctx.waxpby(n, 0.0, xp, 0.0, xp, xp)
            t1 = time.perf_counter()
            r = p.solve(it, 0.0)
            t2 = time.perf_counter()
            e = p.maxabsdiff()
            t3 = time.perf_counter()
            tw.append(t1 - t0); ts.append(t2 - t1); tm.append(t3 - t2)
        print({"variant": variant, "iters": it, "waxpby_us": round(min(tw) * 1e6, 1), "solve_us": round(min(ts) * 1e6, 1),
               "maxabs_us": round(min(tm) * 1e6, 1), "mode": p.stats()["graph_mode"], "niters": r["niters"]}, flush=True)
