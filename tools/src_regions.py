"""Stall samples / executed instructions of one kernel of an ncu source CSV
(`ncu -i X --page source --csv --print-source sass`), grouped by the CUDA
source line (needs -lineinfo) -- diagnostics.

    python tools/src_regions.py src.csv <kernel-name-substring> [top]
"""
import csv, re, sys
from collections import defaultdict

path, name = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
cur = None; hdr = None; rows = []
for r in csv.reader(open(path)):
    if r and r[0] == "Kernel Name":
        cur = r[1]; hdr = None; continue
    if r and r[0] == "Address":
        hdr = r; continue
    if cur and name in cur and hdr and len(r) > 5:
        rows.append(dict(zip(hdr, r)))
src_col = next(k for k in hdr if k.startswith("Source")) if hdr else None
iE, iS = "Instructions Executed", "Warp Stall Sampling (All Samples)"
tot_s = sum(float(r[iS] or 0) for r in rows); tot_e = sum(float(r[iE] or 0) for r in rows)
print(f"{len(rows)} SASS lines, {tot_e/1e6:.1f} M warp instructions, {tot_s:.0f} samples")
# stall reason columns
reasons = [k for k in hdr if k.startswith("stall_") or k.startswith("Warp Stall Sampling (All Samples) ")] if hdr else []
agg = defaultdict(lambda: [0.0, 0.0])
for r in rows:
    s = r.get(src_col, "") if src_col else ""
    key = s.strip()[:90]
    agg[key][0] += float(r[iE] or 0); agg[key][1] += float(r[iS] or 0)
for k, (e, s) in sorted(agg.items(), key=lambda t: -t[1][1])[:top]:
    print(f"{s / tot_s * 100:5.1f}% samples {e / tot_e * 100:5.1f}% inst  {k}")
