"""Stress probe of HPCCG_OPT_FUSE_PSPMV: repeated solve(MAXIT, 0) of one grid in
each launch mode, every result compared bitwise with the unfused plain run.
usage: fz_probe.py NX NY NZ [reps] [maxit] [defer]"""
import sys
import numpy as np
sys.path.insert(0, '.')
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
nx, ny, nz = (int(v) for v in sys.argv[1:4])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 5
maxit = int(sys.argv[5]) if len(sys.argv) > 5 else 30
defer = int(sys.argv[6]) if len(sys.argv) > 6 else -1
with H.Context(0) as c, H.Problem(c, nx, ny, nz) as p:
    p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
    p.set_option(H.HPCCG_OPT_DEFER_X, defer)

    def run(fuse, wh, tm, gr):
        p.set_option(H.HPCCG_OPT_FUSE_PSPMV, fuse)
        p.set_option(H.HPCCG_OPT_WHILE, wh)
        p.set_option(H.HPCCG_OPT_TIMING, tm)
        p.set_option(H.HPCCG_OPT_GRAPH, gr)
        p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
        try:
            r = p.solve(maxit, 0.0)
            return (r["niters"], r["normr"], p.get_vec(H.HPCCG_VEC_X).tobytes())
        except H.HpccgError as e:
            return ("ERR", str(e)[:80], b"")
    ref = run(0, 0, 1, 1)
    bad = {}
    for rep in range(reps):
        for mode in ((1, 0, 1, 1), (1, 0, 0, 0), (1, 0, 0, 1), (1, 1, 0, 1)):
            o = run(*mode)
            if o != ref:
                bad[mode] = bad.get(mode, 0) + 1
                if bad[mode] == 1:
                    print("MISMATCH", mode, o[:2], "ref", ref[:2], flush=True)
    print(f"{nx}x{ny}x{nz} reps={reps} maxit={maxit} defer={defer} bad={bad}", flush=True)
