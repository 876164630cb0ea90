"""Summarise an ncu source-page CSV (SASS level): total stall reasons and the hottest instructions.
usage: ncu -i X.ncu-rep --page source --csv > x.csv; python tools/ncu_hot.py x.csv [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
hdr = rows[1]
data = [r for r in rows[2:] if len(r) == len(hdr)]
S = hdr.index("Warp Stall Sampling (All Samples)")
tot = sum(float(r[S] or 0) for r in data) or 1.0
stalls = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
agg = {hdr[i]: sum(float(r[i] or 0) for r in data) for i in stalls}
print("samples", tot)
for k, v in sorted(agg.items(), key=lambda x: -x[1])[:10]:
    print(f"  {k:28s} {v / tot * 100:5.1f}%")
for r in sorted(data, key=lambda r: -float(r[S] or 0))[:top]:
    why = max(stalls, key=lambda i: float(r[i] or 0))
    print(f"{r[0]:>6s} {float(r[S] or 0) / tot * 100:5.1f}% {hdr[why]:22s} {r[1][:90]}")
