"""One-line summary of a bench.py JSON line (for gpurun logs)."""
import json
import sys

for path in sys.argv[1:]:
    try:
        d = json.loads(open(path).read().strip().splitlines()[-1])
    except (OSError, ValueError, IndexError) as e:
        print(path, "unreadable:", e)
        continue
    r = d.get("roofline") or {}
    st = (r.get("stage_ms") or {})
    print(path, f"ms={d.get('ms_per_step'):.3f}", f"value={d.get('value'):.4g}", "stage", r.get("stage"),
          f"frac={r.get('frac', 0):.3f}", "parity", d.get("parity_vs_oracle"),
          "e2e_ms", (d.get("e2e") or {}).get("ms_per_step"), "cpu", (d.get("cpu_baseline") or {}).get("ms"),
          "clocks", d.get("clocks"), "stages", {k: round(v, 3) for k, v in st.items()})
