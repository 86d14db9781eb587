"""Host-synchronous call latency at small n: our C-ABI AXPY / DOT vs the
ctypes floor and torch's own kernels + synchronize (reference points)."""
import os, sys, time, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
ctx = H.Context(0)
n = 1000
x = torch.rand(n, dtype=torch.float64, device="cuda")
y = torch.rand(n, dtype=torch.float64, device="cuda")
xp, yp = x.data_ptr(), y.data_ptr()
lib = H.lib()
def t(f, reps=2000):
    for _ in range(100): f()
    t0 = time.perf_counter()
    for _ in range(reps): f()
    return round((time.perf_counter() - t0) / reps * 1e6, 2)
out = {
 "ctypes_noop_us": t(lambda: lib.hpccg_version()),
 "axpy_us": t(lambda: ctx.waxpby(n, 1.0, xp, 2.5, yp, xp)),
 "dot_us": t(lambda: ctx.ddot(n, xp, yp)),
 "torch_axpy_sync_us": t(lambda: (x.add_(y, alpha=2.5), torch.cuda.synchronize())),
 "torch_dot_item_us": t(lambda: torch.dot(x, y).item()),
 "torch_sync_only_us": t(lambda: torch.cuda.synchronize()),
}
print(out)
