"""GPU tuning probe: SpMV register-budget variants and solve modes at 128^3.
Prints one JSON line per configuration (timing mode gives per-phase events)."""
import json
import sys
import os

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H

dims = tuple(int(v) for v in (sys.argv[1:4] if len(sys.argv) > 3 else (128, 128, 128)))
iters = int(sys.argv[4]) if len(sys.argv) > 4 else 200
torch.cuda.set_device(0)
ctx = H.Context(0)
p = H.Problem(ctx, *dims)
n, nnz = p.n, p.info["nnz_local"]
xptr = p.vec_ptr(H.HPCCG_VEC_X)
spmv_bytes = 12.0 * nnz + 16.0 * n


def run(minb, graph, timing, wh, reps=3, l2=1):
    p.set_option(H.HPCCG_OPT_L2_PERSIST, l2)
    p.set_option(H.HPCCG_OPT_SPMV_MINB, minb)
    p.set_option(H.HPCCG_OPT_GRAPH, graph)
    p.set_option(H.HPCCG_OPT_TIMING, timing)
    p.set_option(H.HPCCG_OPT_WHILE, wh)
    best = None
    for _ in range(reps + 1):
        ctx.waxpby(n, 0.0, xptr, 0.0, xptr, xptr)
        r = p.solve(iters + 1, 0.0)
        st = p.stats()
        if best is None or st["total_ms"] < best["total_ms"]:
            best = st
    out = {"dims": dims, "minb": minb, "graph": graph, "timing": timing, "while": wh, "l2": l2,
           "t_iter_us": best["total_ms"] * 1e3 / iters}
    if timing:
        sp = best["spmv_ms"] / best["spmv_launches"]
        out.update(spmv_us=sp * 1e3, spmv_gbs=spmv_bytes / (sp * 1e-3) / 1e9,
                   upd_us=best["update_ms"] * 1e3 / iters, pupd_us=best["pupdate_ms"] * 1e3 / iters)
    print(json.dumps(out), flush=True)


for l2 in (1, 0):
    for minb in (1, 2, 3, 4):
        run(minb, 0, 1, 0, l2=l2)
    for minb in (1, 2, 3, 4):
        run(minb, 1, 0, 1, l2=l2)
run(0, 1, 0, 0)
run(0, 0, 0, 0)
