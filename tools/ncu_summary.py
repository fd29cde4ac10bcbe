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


def full(rep, out, workload=None):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = [r for r in csv.reader(io.StringIO(raw))]
    hdr, units = rows[0], rows[1]
    kernels = []
    for vals in rows[2:]:
        d = {}
        for h, u, v in zip(hdr, units, vals):
            if h in FULL_METRICS or h == "Kernel Name":
                try:
                    x = float(v.replace(",", ""))
                    d[h] = {"value": x, "unit": u}
                except ValueError:
                    d[h] = v
        kernels.append(d)
    k = kernels[0]

    def si(name):
        e = k.get(name)
        if not isinstance(e, dict):
            return None
        return e["value"] * UNIT_SCALE.get(e["unit"], 1)
    rd, wr, t = si("dram__bytes_read.sum"), si("dram__bytes_write.sum"), si("gpu__time_duration.sum")
    summary = {
        "report": rep, "workload": workload, "kernel": k.get("Kernel Name"),
        "duration_s": t, "dram_read_bytes": rd, "dram_write_bytes": wr,
        "dram_bytes_per_launch": (rd or 0) + (wr or 0),
        "dram_gbs": ((rd or 0) + (wr or 0)) / t / 1e9 if t else None,
        "metrics": {h: k[h] for h in FULL_METRICS if h in k},
    }
    json.dump(summary, open(out, "w"), indent=1)
    print(json.dumps({x: summary[x] for x in ("kernel", "duration_s", "dram_bytes_per_launch", "dram_gbs")}))


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
