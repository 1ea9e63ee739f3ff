"""Per-instruction warp-stall samples from an ncu source page (sass), grouped
into contiguous regions, for reading where a kernel's warps wait.

    ncu -i X.ncu-rep --page source --csv --print-source sass > X.csv
    python tools/sass_hot.py X.csv [top]
"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr = rows[1]
body = [r for r in rows[2:] if len(r) == len(hdr)]
ci = {h: i for i, h in enumerate(hdr)}
stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
tot = sum(int(r[ci["Warp Stall Sampling (All Samples)"]] or 0) for r in body)
print("total samples", tot)
agg = {h: 0 for h in stall_cols}
for r in body:
    for h in stall_cols:
        agg[h] += int(r[ci[h]] or 0)
print("stall reasons:", ", ".join(f"{h[6:]} {100*v/tot:.1f}%" for h, v in sorted(agg.items(), key=lambda x: -x[1]) if v))
idx = sorted(range(len(body)), key=lambda i: -int(body[i][ci["Warp Stall Sampling (All Samples)"]] or 0))[:top]
for i in sorted(idx):
    r = body[i]
    s = int(r[ci["Warp Stall Sampling (All Samples)"]] or 0)
    reasons = sorted(((int(r[ci[h]] or 0), h[6:]) for h in stall_cols), reverse=True)[:3]
    print(f"{i:5d} {100*s/tot:5.1f}%  {r[1].strip()[:60]:60s} " + " ".join(f"{n}:{v}" for v, n in reasons if v))
