"""Summarise an ncu SASS source page CSV: hottest instructions and stall reasons."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = rows[2:]
idx = {h: i for i, h in enumerate(hdr)}
S = idx["Warp Stall Sampling (All Samples)"]
tot = sum(int(r[S] or 0) for r in data if len(r) > S)
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
agg = {h: 0 for h in stalls}
for r in data:
    for h in stalls:
        try: agg[h] += int(r[idx[h]] or 0)
        except (ValueError, IndexError): pass
print("total samples", tot)
for h, v in sorted(agg.items(), key=lambda x: -x[1])[:10]:
    print(f"  {h:28s} {v:8d} {100*v/max(tot,1):5.1f}%")
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
order = sorted(range(len(data)), key=lambda i: -int(data[i][S] or 0))[:N]
for i in sorted(order):
    r = data[i]
    top = sorted(((int(r[idx[h]] or 0), h) for h in stalls), reverse=True)[:2]
    print(f"{i:5d} {int(r[S]):7d} {100*int(r[S])/tot:5.1f}%  {r[1].strip()[:60]:60s} {top}")
