"""BLAS-1 probe: host-synchronous hpccg_waxpby (JACC AXPY x += a y) and
hpccg_ddot at large n, median of R calls, algorithmic GB/s.
usage: [HPCCG_AXPY_UNROLL=2|4] [HPCCG_DOT_UNROLL=2|4] blas1_probe.py N [N ...]"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H

ctx = H.Context(0)
for n in (int(float(v)) for v in sys.argv[1:]):
    x = torch.rand(n, dtype=torch.float64, device="cuda")
    y = torch.rand(n, dtype=torch.float64, device="cuda")
    torch.cuda.synchronize()
    res = {}
    for name, call, nbytes in (("axpy", lambda: ctx.waxpby(n, 1.0, x.data_ptr(), 2.5, y.data_ptr(), x.data_ptr()), 24 * n),
                               ("dot", lambda: ctx.ddot(n, x.data_ptr(), y.data_ptr()), 16 * n)):
        for _ in range(3):
            call()
        ts = []
        for _ in range(15):
            t0 = time.perf_counter()
            call()
            ts.append(time.perf_counter() - t0)
        ts.sort()
        t = ts[len(ts) // 2]
        res[name + "_us"] = round(t * 1e6, 2)
        res[name + "_GBs"] = round(nbytes / t / 1e9, 1)
    print(json.dumps({"n": n, "unroll": [os.environ.get("HPCCG_AXPY_UNROLL", "-"), os.environ.get("HPCCG_DOT_UNROLL", "-")], **res}), flush=True)
    del x, y
