import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
from synth import graphs as G
import paper_conf_sc_fallingsb23_b200 as m
cases = [("road-small", synth.make_config("road", "small")), ("grid-full", synth.make_config("grid", "full")),
         ("path", G.path_graph(100000)), ("rand", G.random_small(50000, 70000, seed=3, weights="uniform"))]
for name, g in cases:
    omask, ot, oc = oracle.kruskal_graph(g)
    gd = g.to("cuda:0")
    for order, mc in ((1, 0), (2, 0), (2, 1), (2, 2), (2, 3)):
        o = m.default_options(populate_order=order, max_ctas=mc)
        mask, tot, ws = m.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight, options=o)
        st = m.ecl_mst_read_stats(ws)
        print(name, "M", g.M, "order", order, "maxctas", mc, "grid", st["grid"], "status", st["status"], "ok", int(tot.item()) == ot, "live0", st["live"][:1], "canon", st["canonical_edges"])
