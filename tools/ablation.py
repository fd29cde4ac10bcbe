"""De-optimisation ablation and filter-seed study on B200.

  python tools/ablation.py --configs road rmat rgg --out profiles/r01_ablation.json
  python tools/ablation.py --seeds 99 --configs rmat rgg --out profiles/r01_seeds.json

Ablation: every option knob of ecl_mst_options that the paper evaluates as an
optimisation (Table 5 semantics): atomic guards, thread-
based populate, the filter, path halving / flatten,
both edge directions, no tuples, topology-driven and
vertex-centric -- alone and cumulatively -- plus this build's own
knobs (populate chunk order, crowded-round split, c, contraction).  Each variant's mask and
total must equal the default run's bit for bit (the default is itself checked
against the oracle by tests/ and bench.py); the JSON keeps the median time of
`--runs` timed runs (CUDA events, L2 flushed before each).

Seed study: the paper's 20-sample threshold under 99 seeds (P:398,
Fig. 6): time per seed, and how far the light-edge count lands from its
target c|V| CSR entries (Fig. 7's "relative distance from the target").
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_fallingsb23_b200 as eclmst  # noqa: E402
import synth  # noqa: E402

VARIANTS = [
    ("default", {}),
    ("guards off", {"atomic_guards": 0}),
    ("guards everywhere", {"atomic_guards": 1}),
    ("filter off", {"filter": 0}),
    ("filter on", {"filter": 1}),
    ("no path halving", {"path_halving": 0}),
    ("no flatten", {"flatten": 0}),
    ("no halving, no flatten", {"path_halving": 0, "flatten": 0}),
    ("populate interleaved", {"populate_order": 1}),
    ("populate contiguous", {"populate_order": 2}),
    ("no crowded-round split", {"refilter": 0}),
    ("filter c=2", {"filter_c": 2}),
    ("filter c=3", {"filter_c": 3}),
    ("paper: 20 samples", {"threshold_samples": 20}),
    ("paper-like: 20 samples, no split", {"threshold_samples": 20, "refilter": 0}),
    ("exact-quantile threshold", {"threshold_mode": 2}),
    ("no contraction (relabel off)", {"relabel": 0}),
    # Table 5: each de-optimisation alone ...
    ("thread-based populate (P:372)", {"populate_mode": 1}),
    ("both edge directions (P:375)", {"both_directions": 1}),
    ("no tuples / SoA (P:376)", {"tuple_layout": 1}),
    ("topology-driven (P:377)", {"drive": 1}),
    ("vertex-centric (P:378)", {"drive": 2}),
    # ... and cumulatively, in the paper's order.  Step (4), "no
    # implicit path compression", has no knob of its own: pass B's hook needs
    # the round's representatives in the tuples; the topology-
    # driven step finds from the original endpoints in every round instead.
    ("cum: no guards", {"atomic_guards": 0}),
    ("cum: + thread-based", {"atomic_guards": 0, "populate_mode": 1}),
    ("cum: + no filter", {"atomic_guards": 0, "populate_mode": 1, "filter": 0}),
    ("cum: + both directions", {"atomic_guards": 0, "populate_mode": 1, "filter": 0, "both_directions": 1}),
    ("cum: + no tuples", {"atomic_guards": 0, "populate_mode": 1, "filter": 0, "both_directions": 1,
                          "tuple_layout": 1}),
    ("cum: + topology-driven", {"atomic_guards": 0, "populate_mode": 1, "filter": 0, "both_directions": 1,
                                "tuple_layout": 1, "drive": 1}),
    ("cum: + vertex-centric", {"atomic_guards": 0, "populate_mode": 1, "filter": 0, "both_directions": 1,
                               "tuple_layout": 1, "drive": 2}),
]


def timed(g, opts, runs, ws, flush):
    dev = g.nlist.device
    mask = torch.empty(g.M, dtype=torch.uint8, device=dev)
    total = torch.empty(1, dtype=torch.int64, device=dev)
    ts = []
    for i in range(runs + 1):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        eclmst.ecl_mst_device(g.n, g.nindex, g.nlist, g.eweight, in_mst_out=mask, total_weight_out=total,
                              workspace=ws, options=opts)
        b.record()
        torch.cuda.synchronize()
        if i:
            ts.append(a.elapsed_time(b))
    return statistics.median(ts), mask, int(total.item()), eclmst.ecl_mst_read_stats(ws)


def ablation(cfgs, runs, path=None):
    out = {}
    dev = torch.device("cuda:0")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    for c in cfgs:
        g = synth.make_config(c, "full", device=dev)
        ws = torch.empty(eclmst.ecl_mst_workspace_bytes(g.n, g.M, eclmst.default_options(both_directions=1)),
                         dtype=torch.uint8, device=dev)
        rows = []
        ref_mask = ref_total = None
        for name, kw in VARIANTS:
            try:
                ms, mask, total, st = timed(g, eclmst.default_options(**kw), runs, ws, flush)
            except Exception as e:   # (recorded, not fatal: e.g. a de-optimisation too slow or too large)
                rows.append({"variant": name, "options": kw, "error": str(e)[:200]})
                print(f"{c:8s} {name:34s} ERROR {e}", flush=True)
                continue
            if ref_mask is None:
                ref_mask, ref_total = mask.clone(), total
                same = True
            else:
                same = bool(total == ref_total and torch.equal(mask, ref_mask))
            rows.append({"variant": name, "options": kw, "ms": ms, "identical_msf": same,
                         "rounds": st["rounds"], "refilters": st["refilters"], "filtered": st["filtered"],
                         "sum_live": int(sum(st["live"]))})
            print(f"{c:8s} {name:34s} {ms:9.3f} ms  same={same} rounds={st['rounds']}", flush=True)
        out[c] = {"graph": g.name, "n": g.n, "M": g.M, "rows": rows}
        if path:
            with open(path, "w") as f:
                json.dump(out, f, indent=1)
        del ws, g
        torch.cuda.empty_cache()
    return out


THRESHOLD_MODES = [
    ("paper: S=20", {"threshold_samples": 20}),
    ("default: S=1024", {"threshold_samples": 1024}),
    ("exact quantile", {"threshold_mode": 2}),        # NEXT-3: radix select over all M weights
]


def seed_study(cfgs, seeds, runs):
    """Threshold study (Fig. 6/7 semantics): per mode, time and
    light-entry count vs the target c|V| over `seeds` seeds (one run for the
    exact quantile, which does not depend on the seed)."""
    out = {}
    dev = torch.device("cuda:0")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    for c in cfgs:
        g = synth.make_config(c, "full", device=dev)
        ws = torch.empty(eclmst.ecl_mst_workspace_bytes(g.n, g.M), dtype=torch.uint8, device=dev)
        w = g.eweight
        cc = 3 if g.M >= 16 * g.n else 4      # the default c (DESIGN reading Q5b)
        target = cc * g.n                      # c|V| lightest CSR entries
        ref = None
        modes = {}
        for mname, kw in THRESHOLD_MODES:
            rows = []
            for seed in range(seeds if "threshold_mode" not in kw else 1):
                ms, mask, total, st = timed(g, eclmst.default_options(seed=seed, **kw), runs, ws, flush)
                if ref is None:
                    ref = (mask.clone(), total)
                same = bool(total == ref[1] and torch.equal(mask, ref[0]))
                light = int((w < st["threshold"]).sum().item()) if st["filtered"] else g.M
                rows.append({"seed": seed, "ms": ms, "threshold": st["threshold"], "light_entries": light,
                             "rel_to_target": light / target - 1.0, "identical_msf": same,
                             "refilters": st["refilters"]})
            ms_all = sorted(r["ms"] for r in rows)
            rel = sorted(r["rel_to_target"] for r in rows)
            summ = {"runs": len(rows), "min_ms": ms_all[0], "q1_ms": ms_all[len(ms_all) // 4],
                    "median_ms": statistics.median(ms_all), "q3_ms": ms_all[3 * len(ms_all) // 4],
                    "max_ms": ms_all[-1], "rel_to_target_median": statistics.median(rel),
                    "rel_to_target_min": rel[0], "rel_to_target_max": rel[-1],
                    "all_identical": all(r["identical_msf"] for r in rows)}
            print(c, mname, json.dumps(summ), flush=True)
            modes[mname] = {"options": kw, "summary": summ, "rows": rows}
        out[c] = {"graph": g.name, "n": g.n, "M": g.M, "c": cc, "target_light_entries": target, "modes": modes}
        del ws, g
        torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", nargs="+", default=["road", "rgg", "rmat"])
    ap.add_argument("--runs", type=int, default=5)
    ap.add_argument("--seeds", type=int, default=0, help="run the seed study with this many seeds instead")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    res = (seed_study(args.configs, args.seeds, max(1, args.runs)) if args.seeds
           else ablation(args.configs, args.runs, args.out))
    res["gpu"] = torch.cuda.get_device_name(0)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
