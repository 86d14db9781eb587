"""Per-kernel timeline of the CG iteration from the device trace
(HPCCG_OPT_TRACE): kernel durations (first-block start -> last-block end) and
the gaps between consecutive kernels, in the product configuration.
usage: trace.py NX NY NZ ITERS ['opt=val,...' ...]  (probe.py option names)"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
sys.argv += [] if len(sys.argv) > 5 else [""]
nx, ny, nz, iters = (int(v) for v in sys.argv[1:5])
KEYS = {"graph": H.HPCCG_OPT_GRAPH, "timing": H.HPCCG_OPT_TIMING, "while": H.HPCCG_OPT_WHILE,
        "pdl": H.HPCCG_OPT_PDL, "waves": H.HPCCG_OPT_VEC_WAVES, "unroll": H.HPCCG_OPT_VEC_UNROLL,
        "rows": H.HPCCG_OPT_SPMV_ROWS, "l2": H.HPCCG_OPT_L2_PERSIST,
        "wu": H.HPCCG_OPT_WHILE_UNROLL, "ff": H.HPCCG_OPT_FINISHER_FREE,
        "peer": H.HPCCG_OPT_HALO_PEER, "serp": H.HPCCG_OPT_SERPENTINE,
        "defer": H.HPCCG_OPT_DEFER_X}
if os.environ.get("PROBE_NCCL"):  # 1-rank NCCL communicator: the multi-GPU code path
    ctx = H.Context(0, rank=0, nranks=1, unique_id=H.hpccg_unique_id())
else:
    ctx = H.Context(0)
p = H.Problem(ctx, nx, ny, nz)
p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
xptr = p.vec_ptr(H.HPCCG_VEC_X)
for spec in sys.argv[5:]:
    opts = dict(kv.split("=") for kv in spec.split(",") if kv)
    for k, v in opts.items():
        p.set_option(KEYS[k], int(v))
    p.set_option(H.HPCCG_OPT_TRACE, iters)
    for _ in range(3):
        ctx.waxpby(p.n, 0.0, xptr, 0.0, xptr, xptr)
        r = p.solve(iters + 1, 0.0)
    st = p.stats()
    tr = p.trace(iters).astype(np.float64)[5:]   # skip the first iterations
    dur = (tr[:, :, 1] - tr[:, :, 0]) / 1e3       # us
    gap_pu_spmv = (tr[:, 1, 0] - tr[:, 0, 1]) / 1e3
    gap_spmv_upd = (tr[:, 2, 0] - tr[:, 1, 1]) / 1e3
    gap_upd_next = (tr[1:, 0, 0] - tr[:-1, 2, 1]) / 1e3
    period = (tr[1:, 0, 0] - tr[:-1, 0, 0]) / 1e3
    out = {"dims": [nx, ny, nz], "opts": opts, "t_iter_us_events": st["total_ms"] * 1e3 / iters,
           "period_us": round(float(np.median(period)), 2),
           "pupdate_us": round(float(np.median(dur[:, 0])), 2),
           "spmv_us": round(float(np.median(dur[:, 1])), 2),
           "update_us": round(float(np.median(dur[:, 2])), 2),
           "gap_pupdate_spmv": round(float(np.median(gap_pu_spmv)), 2),
           "gap_spmv_update": round(float(np.median(gap_spmv_upd)), 2),
           "gap_update_next": round(float(np.median(gap_upd_next)), 2),
           "mode": st["graph_mode"]}
    print(json.dumps(out), flush=True)
    p.set_option(H.HPCCG_OPT_TRACE, 0)
    for k in opts:
        p.set_option(KEYS[k], {"graph": 1, "while": 1, "pdl": 1, "waves": 1, "unroll": 4, "rows": 2,
                               "l2": 1, "wu": 4, "serp": -1}.get(k, 0))
