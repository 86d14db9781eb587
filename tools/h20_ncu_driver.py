import sys
sys.path.insert(0, ".")
import numpy as np
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
ctx = H.Context(0)
p = H.Problem(ctx, 20, 30, 10)
for _ in range(3):
    p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
    r = p.solve(150, 1e-12)
print(r["niters"], p.stats()["graph_mode"])
