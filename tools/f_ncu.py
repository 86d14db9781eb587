"""Driver for the ncu captures of the f1 / f4 hot paths (run under ncu with
--graph-profiling graph: the tridiagonal CG solve is a graph with a WHILE
node, whose kernel nodes ncu cannot profile one by one): the fused
tridiagonal CG (variant 1) at SIZE 1e8 -- a 1-iteration solve (init only) and
a 5-iteration one, so DRAM bytes per iteration = the difference / 4 -- then
the D2Q9 pull step at 1000^2 (plain launches)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
ctx = H.Context(0)
t = H.Tri(ctx, 100_000_000)
t.solve(1, 0.0, 1)
t.solve(5, 0.0, 1)
t.free()
l = H.Lbm(ctx, 1000)
f0 = synth.lbm_state(1000, 21)
l.set(0, f0)
l.set(1, f0)
l.run(4, 0.8)
l.free()
ctx.close()
