"""One small forced-relabel MSF run, for compute-sanitizer (synccheck, memcheck, initcheck):

  compute-sanitizer --tool synccheck python tools/sanitize_run.py ties 1
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sc_fallingsb23_b200 as m  # noqa: E402
from synth import graphs as G  # noqa: E402

g = G.random_small(1000, 6000, seed=7000, weights=sys.argv[1] if len(sys.argv) > 1 else "ties", multi=True, self_loops=True)
omask, ototal, _ = oracle.kruskal_graph(g)
gd = g.to("cuda:0")
for it in range(int(sys.argv[2]) if len(sys.argv) > 2 else 3):
    mask, total, ws = m.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight, options=m.default_options(relabel=1, filter=0))
    st = m.ecl_mst_read_stats(ws)
    print(it, "ok" if int(total.item()) == ototal and np.array_equal(mask.cpu().numpy(), omask) else "BAD",
          st["relabels"], st["winners"], flush=True)
