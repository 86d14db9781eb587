"""LBM (f4) probe: us/step at SIZE for the one-step kernel's cache policies and
the two-step kernel's rows per CTA (state reset before every measurement).
usage: lbm_probe.py SIZE STEPS"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
S, steps = int(sys.argv[1]), int(sys.argv[2])
ctx = H.Context(0)
l = H.Lbm(ctx, S)
f0 = synth.lbm_state(S, 21)
# bits: 1-2 policy (0 -> default 1 = stores cached, 2 = all cached, 3 = all streaming), 3 no PDL,
# 4 two steps per kernel, 8-15 rows per CTA of the two-step kernel, 16-18 its min CTAs/SM
cases = [("single pol=default", 0), ("single all-stream", 6), ("single no-PDL", 8)]
cases += [("pairs rows=%d minB=%d" % (r, mb), 16 | r << 8 | mb << 16)
          for mb, rr in ((4, (14, 16)), (5, (11, 12, 14)), (6, (9, 10, 12)), (8, (7, 8, 10)))
          for r in rr]
for name, bits in cases + cases[:1] + cases[3:]:
    ts = []
    for _ in range(3):
        l.set(0, f0)
        l.set(1, f0)
        ts.append(l.run(steps, 0.8, bits))
    fin = l.get(0)
    us = min(ts) * 1e3 / steps
    print({"S": S, "case": name, "us_per_step": round(us, 2),
           "all_us": [round(t * 1e3 / steps, 2) for t in ts],
           "GBs_alg": round(144.0 * (S - 2) ** 2 / (us * 1e-6) / 1e9, 1),
           "finite": bool(np.isfinite(fin).all()), "max": float(np.nanmax(np.abs(fin)))}, flush=True)
