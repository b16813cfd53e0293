"""Top SASS lines by warp-stall samples from `ncu --page source --csv --print-source sass`."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = []
for r in rows[2:]:
    if r and r[0] == "Kernel Name":
        break          # first kernel section only
    if len(r) > 3 and r[0] != "Address":
        data.append(r)
iS = hdr.index("Warp Stall Sampling (All Samples)")
iE = hdr.index("Instructions Executed")
tot = sum(float(r[iS] or 0) for r in data)
tot_e = sum(float(r[iE] or 0) for r in data)
print(f"total samples {tot:.0f}, warp instructions executed {tot_e:.0f}")
top = sorted(range(len(data)), key=lambda i: -float(data[i][iS] or 0))[: int(sys.argv[2]) if len(sys.argv) > 2 else 30]
for i in sorted(top):
    r = data[i]
    print(f"{i:5d} {float(r[iS]) / tot * 100:5.1f}%  exec={r[iE]:>9s}  {r[1].strip()[:90]}")
