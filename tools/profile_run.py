"""Minimal driver for ncu: build a config graph on cuda:0, run the hot path a few times.

  ncu ... python tools/profile_run.py --config road --runs 2
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_fallingsb23_b200 as eclmst  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="road")
    ap.add_argument("--size", default="full")
    ap.add_argument("--runs", type=int, default=2)
    ap.add_argument("--opt", action="append", default=[], help="option=value for ecl_mst_options")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    g = synth.make_config(args.config, args.size, device=dev)
    kw = {k: int(v) for k, v in (o.split("=") for o in args.opt)}
    opts = eclmst.default_options(**kw)
    ws = torch.empty(eclmst.ecl_mst_workspace_bytes(g.n, g.M), dtype=torch.uint8, device=dev)
    for _ in range(args.runs):
        mask, total, ws = eclmst.ecl_mst_device(g.n, g.nindex, g.nlist, g.eweight, workspace=ws, options=opts)
    torch.cuda.synchronize()
    st = eclmst.ecl_mst_read_stats(ws)
    print(f"{g.name}: n={g.n} M={g.M} total={int(total.item())} rounds={st['rounds']} "
          f"live={st['live']} t_ns={[t - st['t_ns'][0] for t in st['t_ns']]}")


if __name__ == "__main__":
    main()
