import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
from synth import graphs as G
import paper_conf_sc_fallingsb23_b200 as m
from tests import refs

n_, m_, wk = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3]
g = G.random_small(n_, m_, seed=n_ + m_, weights=wk, multi=True, self_loops=True)
n, nindex, nlist, ew = g.numpy()
u, v, w, ids = refs.canonical_edges(n, nindex, nlist, ew)
omask, ot, oc = oracle.kruskal_graph(g)
print("n", n, "M", g.M, "canonical", len(u), "weights", np.unique(w, return_counts=True))
gd = g.to("cuda:0")
for opts in [dict(), dict(), dict(filter=0), dict(flatten=0), dict(atomic_guards=0), dict(max_ctas=1)]:
    o = m.default_options(**opts)
    mask, tot, ws = m.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight, options=o)
    st = m.ecl_mst_read_stats(ws)
    T = st["threshold"]
    light = int((w < T).sum()) if st["filtered"] else len(u)
    mk = mask.cpu().numpy()
    print(opts, "status", st["status"], "tot ok", int(tot.item()) == ot, "mask diff", int((mk != omask).sum()),
          "canon", st["canonical_edges"], "heavy", st["heavy_edges"], "light py", light, "p2", st["phase2_round"], "T", T, "grid", st["grid"], "rounds", st["rounds"])
    print("   live", st["live"][:40])
    print("   win ", st["winners"][:40])
