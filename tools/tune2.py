"""Quick probe: L2 persistence on/off, timing vs while-graph at one size."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
dims = tuple(int(v) for v in (sys.argv[1:4] if len(sys.argv) > 3 else (128, 128, 128)))
iters = int(sys.argv[4]) if len(sys.argv) > 4 else 200
ctx = H.Context(0)
p = H.Problem(ctx, *dims)
n, nnz = p.n, p.info["nnz_local"]
xptr = p.vec_ptr(H.HPCCG_VEC_X)
dev = torch.cuda.get_device_properties(0)
print(json.dumps({"l2": getattr(dev, "L2_cache_size", None)}))
for l2 in (1, 0):
    for timing in (1, 0):
        p.set_option(H.HPCCG_OPT_L2_PERSIST, l2)
        p.set_option(H.HPCCG_OPT_TIMING, timing)
        best = None
        for _ in range(4):
            ctx.waxpby(n, 0.0, xptr, 0.0, xptr, xptr)
            p.solve(iters + 1, 0.0)
            st = p.stats()
            if best is None or st["total_ms"] < best["total_ms"]:
                best = st
        out = {"dims": dims, "l2": l2, "timing": timing, "t_iter_us": best["total_ms"] * 1e3 / iters,
               "l2_persist_bytes": best["l2_persist_bytes"], "graph_mode": best["graph_mode"]}
        if timing:
            out.update(spmv_us=best["spmv_ms"] * 1e3 / best["spmv_launches"],
                       upd_us=best["update_ms"] * 1e3 / iters, pupd_us=best["pupdate_ms"] * 1e3 / iters)
        print(json.dumps(out), flush=True)
