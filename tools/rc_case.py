"""compute-sanitizer probe: one small solve in a chosen mode.
usage: rc_case.py HALO_PEER WHILE TIMING P SERP  (env PDL=0|1)"""
import sys, numpy as np
sys.path.insert(0, '.')
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
mode, wh, timing, P, serp = (int(v) for v in sys.argv[1:6])
if P == 1:
    c = H.Context(0)
else:
    c = H.Context(0, nranks=P, loopback=True)
p = H.Problem(c, 16, 12, 6)
if P > 1:
    p.set_option(H.HPCCG_OPT_HALO_PEER, mode)
p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
p.set_option(H.HPCCG_OPT_WHILE, wh)
p.set_option(H.HPCCG_OPT_TIMING, timing)
import os
p.set_option(H.HPCCG_OPT_PDL, int(os.environ.get("PDL", "1")))
p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n * P))
r = p.solve(20, 0.0)
print(sys.argv[1:], r["niters"])
