"""Per-source-line warp-stall summary of an ncu report (needs -lineinfo).

  python tools/ncu_lines.py report.ncu-rep [top_n]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"]
    if len(sys.argv) > 3:
        cmd += ["--kernel-name", sys.argv[3]]
    if len(sys.argv) > 4:
        cmd += ["--launch-skip", sys.argv[4], "--launch-count", "1"]
    out = subprocess.run(cmd, capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    cur_file = "?"
    hdr = None
    lines = []
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            cur_file = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or not r[0] or r[0] == "":
            continue
        try:
            ln = int(r[0])
        except ValueError:
            continue
        d = dict(zip(hdr[2:], r[2:]))
        try:
            samples = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
        except ValueError:
            samples = 0
        stalls = {}
        for k, v in d.items():
            if k.startswith("stall_") and "Not Issued" not in k:
                try:
                    stalls[k[6:]] = int(v)
                except ValueError:
                    pass
        lines.append((samples, cur_file, ln, r[1].strip(), stalls))
    tot = sum(x[0] for x in lines) or 1
    print(f"total samples {tot}")
    for s, f, ln, src, st in sorted(lines, key=lambda x: -x[0])[:top]:
        tops = ", ".join(f"{k}:{100 * v / max(s, 1):.0f}%" for k, v in sorted(st.items(), key=lambda x: -x[1])[:3] if v)
        print(f"{100 * s / tot:5.1f}%  {f}:{ln:<4d} {src[:70]:70s} [{tops}]")


if __name__ == "__main__":
    main()
