"""Summarise ncu outputs into profiles/ (JSON + markdown-ready numbers).

  python tools/ncu_summary.py full  <report.ncu-rep> <out.json> [workload-name]
  python tools/ncu_summary.py launches <launches.csv> <out.json>
"""
import csv
import io
import json
import subprocess
import sys

FULL_METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "lts__t_sectors_op_red.sum", "lts__t_sectors_op_atom.sum", "lts__t_requests_op_red.sum",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
    "l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "launch__occupancy_limit_registers", "sm__maximum_warps_per_active_cycle_pct",
]

UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
              "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "s": 1, "second": 1,
              "nsecond": 1e-9}


def stage_of(kernel_name):
    k = kernel_name.replace("(int)", "")
    for pat, st in (("k_init", "init"), ("k_populate<1", "populate1"), ("k_populate<2", "populate2"),
                    ("k_rounds<1", "rounds1"), ("k_rounds<2", "rounds2"), ("k_qhist", "init"), ("k_qselect", "init"),
                    ("k_flatten", "flatten"), ("k_giant", "flatten"), ("k_finalize", "finalize")):
        if pat in k:
            return st
    return k


def full(rep, out, workload=None):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = [r for r in csv.reader(io.StringIO(raw))]
    hdr, units = rows[0], rows[1]
    per_stage = {}
    for vals in rows[2:]:
        d = {}
        for h, u, v in zip(hdr, units, vals):
            if h in FULL_METRICS or h == "Kernel Name":
                try:
                    d[h] = {"value": float(v.replace(",", "")), "unit": u}
                except ValueError:
                    d[h] = v

        def si(name):
            e = d.get(name)
            if not isinstance(e, dict):
                return 0.0
            return e["value"] * UNIT_SCALE.get(e["unit"], 1)
        st = stage_of(d.get("Kernel Name", "?"))
        e = per_stage.setdefault(st, {"kernel": d.get("Kernel Name"), "launches": 0, "duration_s": 0.0,
                                      "dram_read_bytes": 0.0, "dram_write_bytes": 0.0, "metrics": []})
        e["launches"] += 1
        e["duration_s"] += si("gpu__time_duration.sum")
        e["dram_read_bytes"] += si("dram__bytes_read.sum")
        e["dram_write_bytes"] += si("dram__bytes_write.sum")
        e["metrics"].append({h: d[h] for h in FULL_METRICS if h in d})
    for e in per_stage.values():
        e["dram_bytes"] = e["dram_read_bytes"] + e["dram_write_bytes"]
        e["dram_gbs"] = e["dram_bytes"] / e["duration_s"] / 1e9 if e["duration_s"] else None
    summary = {"report": rep, "workload": workload,
               "note": "ncu --set full, one launch of every kernel of one MSF (cold L2, serialised replays)",
               "dram_bytes_per_launch": {k: v["dram_bytes"] for k, v in per_stage.items()},
               "stages": per_stage}
    json.dump(summary, open(out, "w"), indent=1)
    for k, v in per_stage.items():
        print(f"{k:10s} {v['duration_s']*1e3:8.3f} ms  dram {v['dram_bytes']/1e9:7.3f} GB  "
              f"{(v['dram_gbs'] or 0):7.1f} GB/s")


def launches(path, out):
    text = open(path).read()
    start = text.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(text[start:])))
    per = {}
    seq = []
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"]
        short = name.split("(")[0][-80:]
        v = float(r["Metric Value"].replace(",", ""))
        scale = UNIT_SCALE.get(r["Metric Unit"], 1e-9)
        seq.append({"id": int(r["ID"]), "kernel": short, "s": v * scale})
        per.setdefault(short, []).append(v * scale)
    tot = sum(x["s"] for x in seq)
    summary = {"launches": len(seq), "total_s": tot,
               "by_kernel": sorted([{"kernel": k, "count": len(v), "total_s": sum(v), "share": sum(v) / tot}
                                    for k, v in per.items()], key=lambda d: -d["total_s"])}
    json.dump(summary, open(out, "w"), indent=1)
    for d in summary["by_kernel"][:8]:
        print(f'{d["share"]*100:6.2f}%  {d["count"]:4d}  {d["total_s"]*1e3:9.3f} ms  {d["kernel"]}')


if __name__ == "__main__":
    if sys.argv[1] == "full":
        full(sys.argv[2], sys.argv[3], sys.argv[4] if len(sys.argv) > 4 else None)
    else:
        launches(sys.argv[2], sys.argv[3])
