import sys, os, json
sys.path.insert(0, "/root/repo")
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
order = [tuple(int(v) for v in a.split("x")) for a in sys.argv[1:]]
for dims in order:
    ctx = H.Context(0)
    p = H.Problem(ctx, *dims)
    print(dims, p.info, H.lib().hpccg_last_error(), flush=True)
    b = p.get_vec(H.HPCCG_VEC_B)
    print("b sum", b[:5], float(b.sum()), flush=True)
    p.free(); ctx.close()
