"""On-chip solve (configs[0]-sized problems): per-iteration device time with
the gathered vector halo'd in every CTA's shared memory (HPCCG_OPT_SMEM_HALO
1: local gathers) against distributed-shared-memory gathers (0), alternating,
from stats total_ms of 150- and 2-iteration solves (tol 0), both CG variants."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
ctx = H.Context(0)
for dims in [(20, 30, 10), (24, 24, 24), (30, 20, 20), (12, 12, 12)]:
    p = H.Problem(ctx, *dims)
    p.set_option(H.HPCCG_OPT_PERSISTENT, 2)
    xp = p.vec_ptr(H.HPCCG_VEC_X)
    for variant in (0, 1):
        p.set_option(H.HPCCG_OPT_CG_VARIANT, variant)
        res = {}
        for rep in range(3):
            for halo in (0, 1):
                p.set_option(H.HPCCG_OPT_SMEM_HALO, halo)
                t = {}
                for it in (2, 40):
                    best = 1e9
                    for _ in range(5):
                        ctx.waxpby(p.n, 0.0, xp, 0.0, xp, xp)  # x0 = 0 (on the device)
                        p.solve(it, 0.0)
                        best = min(best, p.stats()["total_ms"])
                    t[it] = best
                res.setdefault(halo, []).append(round((t[40] - t[2]) * 1e3 / 38, 3))
        print(json.dumps({"dims": dims, "variant": variant, "mode": p.stats()["graph_mode"],
                          "us_per_iter": res}), flush=True)
    p.free()
