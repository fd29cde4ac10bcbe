"""Per-CTA end times of one stage (imbalance diagnostics).

  python tools/trace_cta.py --config uniform --slot 5   (slot numbering as stats.t_ns: 4+2g pass A/populate, 5+2g pass B)
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
    ap.add_argument("--config", default="uniform")
    ap.add_argument("--slot", type=int, action="append", default=[])
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    g = synth.make_config(args.config, "full", device=dev)
    opts = eclmst.default_options(trace=1)
    ws = torch.empty(eclmst.ecl_mst_workspace_bytes(g.n, g.M), dtype=torch.uint8, device=dev)
    for _ in range(2):
        eclmst.ecl_mst_device(g.n, g.nindex, g.nlist, g.eweight, workspace=ws, options=opts)
    st = eclmst.ecl_mst_read_stats(ws)
    tr = eclmst.ecl_mst_read_trace(ws, st).double()
    G = st["grid"]
    for slot in args.slot or [5]:
        prev = st["t_ns"][slot - 1]
        row = (tr[slot][:G] - prev) / 1e3
        print(f"slot {slot}: min {row.min():.1f} med {row.median():.1f} max {row.max():.1f} us")
        print("  by CTA index (groups of 16):", [round(float(x), 0) for x in row.view(-1, 16).mean(1)] if G % 16 == 0 else "")
        print("  even/odd CTA mean:", float(row[0::2].mean()), float(row[1::2].mean()))
        print("  first/second half:", float(row[: G // 2].mean()), float(row[G // 2:].mean()))


if __name__ == "__main__":
    main()
