"""Generate full-size C5 (uniform 2^26, 1e9 draws) on cuda:0 and run the hot path."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_sc_fallingsb23_b200 as ecl
t = time.time()
g = synth.make_config("uniform", "full", device="cuda:0")
torch.cuda.synchronize()
print("gen s", round(time.time() - t, 1), g.stats(), "peak GB", torch.cuda.max_memory_allocated() / 1e9, flush=True)
ws = torch.empty(ecl.ecl_mst_workspace_bytes(g.n, g.M), dtype=torch.uint8, device="cuda:0")
print("ws GB", ws.numel() / 1e9, flush=True)
o = ecl.default_options(trace=2)
for i in range(3):
    mask, total, ws = ecl.ecl_mst_device(g.n, g.nindex, g.nlist, g.eweight, workspace=ws, options=o)
    kt = ecl.ecl_mst_kernel_times()
    st = ecl.ecl_mst_read_stats(ws)
    print("run", i, "ms", round(sum(kt.values()), 3), {k: round(v, 3) for k, v in kt.items()}, flush=True)
print("status", st["status"], "msf_edges", st["msf_edges"], "n", g.n, "total", int(total.item()), "rounds", st["rounds"],
      "p2", st["phase2_round"], "live", st["live"], "win", st["winners"])
