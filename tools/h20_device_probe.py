import sys, time
sys.path.insert(0, ".")
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
ctx = H.Context(0)
p = H.Problem(ctx, 20, 30, 10)
xp = p.vec_ptr(H.HPCCG_VEC_X)
for it in (1, 2, 3, 11, 51, 150):
    best = None; bt = None
    for rep in range(10):
        ctx.waxpby(p.n, 0.0, xp, 0.0, xp, xp)
        t0 = time.perf_counter(); r = p.solve(it, 0.0); t1 = time.perf_counter()
        st = p.stats()
        best = st["total_ms"] * 1e3 if best is None else min(best, st["total_ms"] * 1e3)
        bt = (t1 - t0) * 1e6 if bt is None else min(bt, (t1 - t0) * 1e6)
    print({"max_iter": it, "niters": r["niters"], "device_us": round(best, 2), "host_us": round(bt, 1)})
