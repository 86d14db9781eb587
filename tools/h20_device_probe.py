"""configs[0] (20x30x10) solve anatomy on the on-chip cluster kernel: device
time (stats total_ms) and host time of tol-0 solves of 1..150 iterations, x0
reset on the device; argv[1] (optional) = HPCCG_OPT_SMEM_HALO."""
import sys, time
sys.path.insert(0, ".")
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
ctx = H.Context(0)
p = H.Problem(ctx, 20, 30, 10)
if len(sys.argv) > 1:
    p.set_option(H.HPCCG_OPT_SMEM_HALO, int(sys.argv[1]))
xp = p.vec_ptr(H.HPCCG_VEC_X)
for it in (1, 2, 3, 11, 51, 150):
    best = None; bt = None
    for rep in range(10):
        ctx.waxpby(p.n, 0.0, xp, 0.0, xp, xp)
        t0 = time.perf_counter(); r = p.solve(it, 0.0); t1 = time.perf_counter()
        st = p.stats()
        best = st["total_ms"] * 1e3 if best is None else min(best, st["total_ms"] * 1e3)
        bt = (t1 - t0) * 1e6 if bt is None else min(bt, (t1 - t0) * 1e6)
    print({"halo": sys.argv[1:], "max_iter": it, "niters": r["niters"], "device_us": round(best, 2),
           "host_us": round(bt, 1), "mode": st["graph_mode"]}, flush=True)
