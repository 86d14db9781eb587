"""compute-sanitizer probe of the round-2 kernels OUTSIDE the WHILE node:
fused p update + SpMV, deferred x (cg_xfix), multi-trip SpMV, cluster finisher.
usage: rc_fused.py WHILE  (0: per-iteration graph + plain timed launches)"""
import sys
import numpy as np
sys.path.insert(0, '.')
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
wh = int(sys.argv[1]) if len(sys.argv) > 1 else 0
with H.Context(0) as c, H.Problem(c, 32, 32, 40) as p:
    p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
    p.set_option(H.HPCCG_OPT_WHILE, wh)
    p.set_option(H.HPCCG_OPT_DEFER_X, 1)
    for opts in ((H.HPCCG_OPT_FUSE_PSPMV, 1), (H.HPCCG_OPT_SPMV_TRIPS, 3)):
        p.set_option(*opts)
        for tm in (0, 1):
            p.set_option(H.HPCCG_OPT_TIMING, tm)
            p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
            print(opts, tm, p.solve(20, 0.0)["niters"], flush=True)
        p.set_option(opts[0], 0 if opts[0] == H.HPCCG_OPT_FUSE_PSPMV else 1)
with H.Context(0) as c, H.Problem(c, 128, 128, 160) as p:   # > 4096 SpMV blocks: the finisher
    p.set_option(H.HPCCG_OPT_WHILE, wh)
    p.set_option(H.HPCCG_OPT_PAP_CLUSTER, 1)
    p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
    print("papcl", p.solve(4, 0.0)["niters"], flush=True)
