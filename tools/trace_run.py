"""Per-CTA stage timing of the persistent kernel (load imbalance diagnostics).

  python tools/trace_run.py --config rmat [--opt atomic_guards=0 ...]

For every stage (populate / pass A / pass B of each global round) prints the
stage duration (last CTA done - previous barrier) and how early the typical
and the first CTA finished: a large gap means CTAs wait at the grid barrier.
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
    ap.add_argument("--opt", action="append", default=[])
    ap.add_argument("--runs", type=int, default=3)
    ap.add_argument("--ov", action="append", default=[], help="generator override k=v (e.g. width=3000)")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    ov = {k: (float(v) if "." in v else int(v)) for k, v in (o.split("=") for o in args.ov)}
    g = synth.make_config(args.config, args.size, device=dev, **ov)
    kw = {k: int(v) for k, v in (o.split("=") for o in args.opt)}
    kw["trace"] = 1
    opts = eclmst.default_options(**kw)
    ws = torch.zeros(eclmst.ecl_mst_workspace_bytes(g.n, g.M), dtype=torch.uint8, device=dev)
    for _ in range(args.runs):
        eclmst.ecl_mst_device(g.n, g.nindex, g.nlist, g.eweight, workspace=ws, options=opts)
    st = eclmst.ecl_mst_read_stats(ws)
    tr = eclmst.ecl_mst_read_trace(ws, st).double()
    t = st["t_ns"]
    print(f"{g.name} opts={kw} total {(t[2] - t[0]) / 1e3:.1f} us  rounds {st['rounds']} grid {st['grid']}")
    prev = t[1]
    R, p2 = st["rounds"], st["phase2_round"]
    seq = []
    for r in range(R):
        if r == p2 and t[3]:
            seq.append(("flatten", 3))
        seq.append(("populate" if r in (0, p2) else "passA", 4 + 2 * r, r))
        if r < R - 1 and t[5 + 2 * r]:
            seq.append(("passB", 5 + 2 * r, r))
    tot_wait = 0.0
    for item in seq:
        name, slot = item[0], item[1]
        r = item[2] if len(item) > 2 else -1
        row = tr[slot]
        valid = row[row > 0]
        if valid.numel() == 0:
            continue
        end = t[slot] if t[slot] else float(valid.max())
        dur = (float(valid.max()) - prev) / 1e3
        med = (float(valid.median()) - prev) / 1e3
        mn = (float(valid.min()) - prev) / 1e3
        wait = float((valid.max() - valid).mean()) / 1e3
        tot_wait += wait
        live = st["live"][r] if r >= 0 else 0
        print(f"  r{r:<3d} {name:9s} live {live:>11d}  last {dur:8.1f} us  median {med:8.1f}  first {mn:8.1f}  "
              f"mean wait {wait:7.1f}")
        prev = end
    print(f"  sum of mean CTA wait at barriers: {tot_wait:.1f} us")
    # populate: per-CTA end (its last warp) and SM
    trf = eclmst.ecl_mst_read_trace(ws, dict(st, grid=4096)).double()
    KG = trf.shape[1]
    for ph, slot, t0 in ((1, 2, t[1]), (2, 3, t[3])):
        row, sms = trf[slot][: KG // 2], trf[slot][KG // 2:]
        ok = row > t0 if t0 else row > 0
        if not t0 or int(ok.sum()) == 0:
            continue
        end = (row[ok] - t0) / 1e3
        sm_ok = sms[ok]
        per = {}
        for e, s_ in zip(end.tolist(), sm_ok.tolist()):
            per.setdefault(int(s_), []).append(e)
        sl = sorted(per)
        mx = torch.tensor([max(per[s_]) for s_ in sl])
        print(f"  populate{ph}: {int(ok.sum())} CTAs, end min {float(end.min()):.1f} med {float(end.median()):.1f} "
              f"max {float(end.max()):.1f} us; per-SM last end min {float(mx.min()):.1f} max {float(mx.max()):.1f}; "
              f"slowest SMs {[sl[i] for i in torch.argsort(mx)[-8:].tolist()]} fastest {[sl[i] for i in torch.argsort(mx)[:8].tolist()]}")
        ne = end.numel() // 16 * 16
        print(f"    by CTA index in 16 groups: {[round(float(x)) for x in end[:ne].view(16, -1).mean(1)]}")
        print(f"    by CTA index mod 4: {[round(float(end[i::4].mean())) for i in range(4)]}; deciles "
              f"{[round(float(x)) for x in torch.quantile(end, torch.linspace(0, 1, 11, dtype=end.dtype))]}")
    # what the slow CTAs of the first passes have in common: their SM, their work
    G = st["grid"]
    sm, nloc = tr[0][:G], tr[1][:G]
    if float(sm.max()) > 0:
        for slot in (5, 6, 7):
            if not t[slot - 1] or not t[slot]:
                continue
            end = (tr[slot][:G] - t[slot - 1]) / 1e3
            order = torch.argsort(end)
            slow, fast = order[-G // 8:], order[: G // 8]
            c = torch.corrcoef(torch.stack([end, nloc]))[0, 1]
            print(f"  slot {slot}: end min {float(end.min()):.1f} med {float(end.median()):.1f} max {float(end.max()):.1f} us;"
                  f" corr(end, first-pass chunks) {float(c):.2f}; slowest 1/8 chunks {float(nloc[slow].mean()):.0f}"
                  f" vs fastest {float(nloc[fast].mean()):.0f}")
            per_sm = {}
            for b in range(G):
                per_sm.setdefault(int(sm[b]), []).append(float(end[b]))
            sms = sorted(per_sm)
            means = torch.tensor([sum(per_sm[s]) / len(per_sm[s]) for s in sms])
            print(f"    per-SM mean end: min {float(means.min()):.1f} max {float(means.max()):.1f}; slowest SMs "
                  f"{[sms[i] for i in torch.argsort(means)[-8:].tolist()]}, fastest {[sms[i] for i in torch.argsort(means)[:8].tolist()]}")
            half = len(sms) // 2
            print(f"    SM ids < {sms[half]}: {float(means[:half].mean()):.1f} us, >=: {float(means[half:].mean()):.1f} us; "
                  f"by SM id in 8 groups {[round(float(x), 0) for x in means[: len(means) // 8 * 8].view(8, -1).mean(1)]}")


if __name__ == "__main__":
    main()
