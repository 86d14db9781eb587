"""configs[0] bench step anatomy (20x30x10, tol 1e-12 / 150, L2 flushed
before each step as bench.py does): CUDA-event time of the whole step and of
its three calls (x0 reset, hpccg_solve, hpccg_maxabsdiff), plus the solve's
own device time (stats total_ms)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
torch.cuda.set_device(0)
st = torch.cuda.Stream()
ctx = H.Context(0, stream=st.cuda_stream)
p = H.Problem(ctx, 20, 30, 10)
xp = p.vec_ptr(H.HPCCG_VEC_X)
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size // 8, dtype=torch.float64, device="cuda")
ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
rows = []
for rep in range(30):
    with torch.cuda.stream(st):
        flush.zero_()
    ev[0].record(st)
    ctx.waxpby(p.n, 0.0, xp, 0.0, xp, xp)
    ev[1].record(st)
    r = p.solve(150, 1e-12)
    ev[2].record(st)
    e = p.maxabsdiff()
    ev[3].record(st)
    ev[3].synchronize()
    rows.append([ev[0].elapsed_time(ev[1]) * 1e3, ev[1].elapsed_time(ev[2]) * 1e3, ev[2].elapsed_time(ev[3]) * 1e3,
                 ev[0].elapsed_time(ev[3]) * 1e3, p.stats()["total_ms"] * 1e3])
import numpy as np
a = np.median(np.array(rows[5:]), axis=0)
print({"x0_us": round(a[0], 1), "solve_us": round(a[1], 1), "maxabs_us": round(a[2], 1), "step_us": round(a[3], 1),
       "solve_device_us": round(a[4], 1), "niters": r["niters"]})
