"""Per-reason warp-stall sample totals of each kernel in an ncu source CSV,
optionally restricted to an address window relative to the kernel start
(diagnostics):  python tools/stall_totals.py src.csv [lo hi]"""
import csv, sys
from collections import defaultdict
path = sys.argv[1]
lo = int(sys.argv[2], 16) if len(sys.argv) > 3 else None
hi = int(sys.argv[3], 16) if len(sys.argv) > 3 else None
cur = None; hdr = None; data = defaultdict(list)
for r in csv.reader(open(path)):
    if r and r[0] == "Kernel Name": cur = r[1]; hdr = None; continue
    if r and r[0] == "Address": hdr = r; continue
    if cur and hdr and len(r) > 5: data[cur].append(dict(zip(hdr, r)))
for k, rows in data.items():
    base = int(rows[0]["Address"], 16)
    if lo is not None:
        rows = [r for r in rows if lo <= int(r["Address"], 16) - base < hi]
    tot = defaultdict(float)
    for r in rows:
        for c, v in r.items():
            if c.startswith("stall_") and "Not Issued" not in c:
                tot[c] += float(v or 0)
        tot["inst"] += float(r["Instructions Executed"] or 0)
    s = sum(v for c, v in tot.items() if c != "inst")
    print(k[:70], f"inst={tot['inst']/1e6:.1f}M samples={s:.0f}")
    print("   " + "  ".join(f"{c[6:]}={v / s * 100:.1f}%" for c, v in sorted(tot.items(), key=lambda t: -t[1]) if c != "inst" and v / s > 0.01))
