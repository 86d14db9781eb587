import os, sys
sys.path.insert(0, '.')
import synth
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
S = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
ctx = H.Context(0)
l = H.Lbm(ctx, S)
f0 = synth.lbm_state(S, 21)
l.set(0, f0); l.set(1, f0)
print(l.run(8, 0.8))
