"""Per-instruction execution counts and stall samples from
`ncu -i X.ncu-rep --page source --csv --print-source sass` (diagnostics).

    python tools/sass_prof.py src.csv [kernel_index] [--min N]

Prints offset, warp instructions executed, stall samples and the SASS line
for every instruction executed at least N times (default 1000), plus totals.
"""
import csv, sys

def sections(path):
    cur, hdr, out = None, None, []
    for r in csv.reader(open(path)):
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            out.append(cur)
            hdr = None
        elif r and r[0] == "Address":
            hdr = r
            cur["hdr"] = r
        elif cur is not None and hdr is not None and len(r) > 5:
            cur["rows"].append(r)
    return out

secs = sections(sys.argv[1])
k = int(sys.argv[2]) if len(sys.argv) > 2 and not sys.argv[2].startswith("--") else 0
mn = int(sys.argv[sys.argv.index("--min") + 1]) if "--min" in sys.argv else 1000
s = secs[k]
h = s["hdr"]
iE, iS = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
rows = s["rows"]
base = int(rows[0][0], 16)
tot = sum(float(r[iE] or 0) for r in rows)
tots = sum(float(r[iS] or 0) for r in rows)
print(f"# {s['name']}: {tot:.0f} warp instructions, {tots:.0f} stall samples")
for r in rows:
    e = float(r[iE] or 0)
    if e >= mn:
        print(f"{int(r[0],16)-base:6x} {e:10.0f} {float(r[iS] or 0)/max(tots,1)*100:5.1f}%  {r[1].strip()[:80]}")
