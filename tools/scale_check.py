"""Correctness + timing at the big configs on one GPU: 256^3 and 512^3 to
tol 1e-12 (SURVEY 8(c) expects niters 112 and 115), max|x-1|."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
for dims, expect in [((256, 256, 256), 112), ((512, 512, 512), 115)]:
    ctx = H.Context(0)
    p = H.Problem(ctx, *dims)
    r = p.solve(150, 1e-12)
    st = p.stats()
    print(json.dumps({"dims": dims, "niters": r["niters"], "expect_scratch": expect,
                      "normr": r["normr"], "maxabsdiff": p.maxabsdiff(),
                      "t_iter_us": st["total_ms"] * 1e3 / max(1, r["niters"]),
                      "nnz": p.info["nnz_global"]}), flush=True)
    p.free()
    ctx.close()
