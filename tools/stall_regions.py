"""Stall-reason totals per code region from an ncu source CSV (diagnostics).

    python tools/stall_regions.py src.csv kernel_index lo1:hi1[:name] lo2:hi2[:name] ...
(offsets in hex, relative to the kernel's first instruction)
"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
k = int(sys.argv[2])
secs, cur = [], None
for r in rows:
    if r and r[0] == "Kernel Name":
        cur = []; secs.append(cur)
    elif r and r[0] == "Address":
        hdr = r
    elif cur is not None and len(r) > 40 and r[0].startswith("0x"):
        cur.append(r)
rows = secs[k]
base = int(rows[0][0], 16)
cols = [i for i, c in enumerate(hdr) if c.startswith("stall_") and "Not Issued" not in c]
regions = []
for a in sys.argv[3:]:
    p = a.split(":")
    regions.append((int(p[0], 16), int(p[1], 16), p[2] if len(p) > 2 else a))
tot = sum(float(r[2] or 0) for r in rows)
iE = hdr.index("Instructions Executed")
for lo, hi, name in regions:
    sel = [r for r in rows if lo <= int(r[0], 16) - base < hi]
    s = sum(float(r[2] or 0) for r in sel)
    e = sum(float(r[iE] or 0) for r in sel)
    parts = sorted(((sum(float(r[c] or 0) for r in sel), hdr[c]) for c in cols), reverse=True)[:6]
    print(f"{name:10s} samples {s / tot * 100:5.1f}%  inst {e:11.0f}  " + "  ".join(f"{n[6:]}={v / max(s, 1) * 100:.0f}%" for v, n in parts))
