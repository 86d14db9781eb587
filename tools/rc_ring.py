"""compute-sanitizer probe for the late round-2 kernels, outside WHILE bodies
(plain launches = TIMING 1, and the per-iteration graph = WHILE 0): the
ring-deferred x update (cg_pupdate_ring_kernel, its flush, cg_xfix_ring_kernel;
ring SpMV) on one slab and on loopback z-slabs with HALO_PEER 2, the clustered
SpMV, and the on-chip solve with the halo'd gathered vector (one cluster
kernel).  Checks the result against the unringed run (bitwise).
usage: rc_ring.py"""
import sys
import numpy as np
sys.path.insert(0, ".")
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H


def run(p, n, **opts):
    for k, v in opts.items():
        p.set_option(getattr(H, "HPCCG_OPT_" + k), v)
    p.set_vec(H.HPCCG_VEC_X, np.zeros(n))
    r = p.solve(20, 0.0)
    return r["niters"], r["normr"], p.get_vec(H.HPCCG_VEC_X)


with H.Context(0) as c, H.Problem(c, 16, 12, 6) as p:
    p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
    base = run(p, p.n, DEFER_X=1, TIMING=1)
    for timing, wh in ((1, 0), (0, 0)):
        for extra in ({}, {"SPMV_CLUSTER": 1}, {"SERPENTINE": 3}):
            o = run(p, p.n, DEFER_X=3, TIMING=timing, WHILE=wh, **extra)
            assert o[:2] == base[:2] and np.array_equal(o[2], base[2]), (timing, wh, extra)
            p.set_option(H.HPCCG_OPT_SPMV_CLUSTER, 0)
            p.set_option(H.HPCCG_OPT_SERPENTINE, -1)
    print("single slab ring ok")
with H.Context(0, nranks=2, loopback=True) as c, H.Problem(c, 16, 12, 6) as p:
    p.set_option(H.HPCCG_OPT_HALO_PEER, 2)
    base = run(p, 2 * p.n, DEFER_X=1, TIMING=1)
    for timing, wh in ((1, 0), (0, 0)):
        o = run(p, 2 * p.n, DEFER_X=3, TIMING=timing, WHILE=wh)
        assert o[:2] == base[:2] and np.array_equal(o[2], base[2]), (timing, wh)
    print("z-slab ring ok")
with H.Context(0) as c, H.Problem(c, 20, 30, 10) as p:
    p.set_option(H.HPCCG_OPT_PERSISTENT, 2)
    a = run(p, p.n, SMEM_HALO=0)
    b = run(p, p.n, SMEM_HALO=1)
    assert a[:2] == b[:2] and np.array_equal(a[2], b[2])
    print("on-chip halo ok")
