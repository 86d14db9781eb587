import numpy as np, sys
sys.path.insert(0, '.')
import oracle
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
P, dims = 2, (16, 12, 6)
ref = oracle.generate(16, 12, 12)
print("oracle sr", oracle.cg_sr(ref, 150, 1e-12)["niters"], "hpccg", oracle.cg(ref, 150, 1e-12)["niters"])
for variant in (0, 1):
    for seq in ([1], [0], [0, 1], [1, 1], [1, 0]):
        with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
            p.set_option(H.HPCCG_OPT_CG_VARIANT, variant)
            out = []
            for peer in seq:
                p.set_option(H.HPCCG_OPT_HALO_PEER, peer)
                p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n * P))
                r = p.solve(150, 1e-12)
                out.append((peer, r["niters"], r["normr"]))
            print(variant, out, flush=True)
for wh in (0, 1):
  for timing in (0, 1):
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
        p.set_option(H.HPCCG_OPT_CG_VARIANT, 1)
        p.set_option(H.HPCCG_OPT_WHILE, wh)
        p.set_option(H.HPCCG_OPT_TIMING, timing)
        p.set_option(H.HPCCG_OPT_HALO_PEER, 1)
        r = p.solve(150, 1e-12)
        print("sr fresh peer wh", wh, "timing", timing, r["niters"], r["normr"], flush=True)
