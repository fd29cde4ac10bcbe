"""Warp instructions executed per CUDA source line of one kernel in an ncu report.

  python tools/ncu_inst.py report.ncu-rep <kernel-regex> [launch-skip] [top]
"""
import csv
import io
import subprocess
import sys

rep, krx = sys.argv[1], sys.argv[2]
skip = sys.argv[3] if len(sys.argv) > 3 else "0"
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass", "--kernel-name",
                      f"regex:{krx}", "--launch-skip", skip, "--launch-count", "1"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = None
f = "?"
acc = []
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr and r[0].isdigit():
        d = dict(zip(hdr, r))
        try:
            n = int(float(d.get("Instructions Executed", "0") or 0))
        except ValueError:
            continue
        if n:
            acc.append((n, f"{f}:{r[0]}", r[1][:90]))
tot = sum(a[0] for a in acc)
print(f"total warp instructions {tot:.4g}")
for n, where, src in sorted(acc, reverse=True)[:top]:
    print(f"{100 * n / tot:5.1f}%  {where:18s} {src}")
