"""Summarise the ncu evidence of one round into profiles/ (committed).

    python tools/profile_summary.py <full.ncu-rep> <launches.csv> <round tag> [workload] [n_elements]

Writes profiles/<tag>_ncu_summary.txt (per kernel: duration, DRAM bytes,
throughput, issue/occupancy, top stalls), profiles/<tag>_launches_share.txt
(the launch list's per-kernel share of device time) and
profiles/ncu_summary.json (DRAM bytes per launch, read by bench.py as the
roofline "traffic" field).
"""
from __future__ import annotations

import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "profiles")
KEYS = {"range_kernel": "range", "compress_kernel": "compress", "decompress_kernel": "decompress"}
METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
    "launch__block_size", "launch__shared_mem_per_block_dynamic", "lts__t_bytes.sum",
]


def kname(s: str) -> str | None:
    for k, v in KEYS.items():
        if k in s and not (k == "compress_kernel" and "decompress_kernel" in s):
            return v
    return None


def main():
    rep, launches, tag = sys.argv[1], sys.argv[2], sys.argv[3]
    workload = sys.argv[4] if len(sys.argv) > 4 else None
    n_el = int(sys.argv[5]) if len(sys.argv) > 5 else None
    os.makedirs(OUT, exist_ok=True)
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    lines, js = [], {"dram_bytes_per_launch": {}, "source": os.path.basename(rep), "tag": tag}
    if workload:
        js["workload"] = workload
    for r in rows[2:]:
        k = kname(r[hdr.index("Kernel Name")])
        if k is None:
            continue
        lines.append(f"== {k} ({r[hdr.index('Kernel Name')][:50]})")
        vals = {}
        for m in METRICS:
            if m in hdr:
                i = hdr.index(m)
                lines.append(f"   {m:60s} {r[i]} {units[i]}")
                vals[m] = (r[i], units[i])
        st = [(hdr[i], float(r[i])) for i in range(len(hdr)) if hdr[i].startswith("smsp__average_warps_issue_stalled_")
              and hdr[i].endswith("_per_issue_active.ratio") and r[i] not in ("", "n/a")]
        st.sort(key=lambda t: -t[1])
        for name, v in st[:6]:
            lines.append("   stall %-40s %.3f" % (name.replace("smsp__average_warps_issue_stalled_", "")
                                                  .replace("_per_issue_active.ratio", ""), v))

        def to_bytes(v):
            x, u = float(v[0]), v[1].lower()
            return x * {"byte": 1, "kbyte": 1e3, "mbyte": 1e6, "gbyte": 1e9}.get(u, 1)

        tb = to_bytes(vals["dram__bytes_read.sum"]) + to_bytes(vals["dram__bytes_write.sum"])
        dur = float(vals["gpu__time_duration.sum"][0]) * {"usecond": 1e-6, "msecond": 1e-3, "nsecond": 1e-9}.get(
            vals["gpu__time_duration.sum"][1].lower(), 1e-6)
        lines.append(f"   => DRAM traffic {tb / 1e6:.2f} MB per launch, {tb / dur / 1e9:.1f} GB/s over the launch")
        if n_el and "smsp__inst_executed.sum" in vals:
            ipb = float(vals["smsp__inst_executed.sum"][0]) / ((n_el + 31) // 32)
            lines.append(f"   => {ipb:.1f} warp instructions per 32-element block")
            js.setdefault("warp_inst_per_block", {})[k] = round(ipb, 2)
        js["dram_bytes_per_launch"].setdefault(k, tb)
    with open(os.path.join(OUT, f"{tag}_ncu_summary.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")
    # launch list: share of device time per kernel
    share = defaultdict(float)
    total = 0.0
    with open(launches) as f:
        text = f.read()
    start = text.find('"ID"')
    for r in csv.DictReader(io.StringIO(text[start:])):
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        total += v
        share[kname(r["Kernel Name"]) or r["Kernel Name"][:40]] += v
    with open(os.path.join(OUT, f"{tag}_launches_share.txt"), "w") as f:
        f.write(f"launch list {os.path.basename(launches)} (cold-cache, serialised: compare shares)\n")
        for k, v in sorted(share.items(), key=lambda kv: -kv[1]):
            f.write(f"{k:45s} {v:14.0f} {100 * v / total:6.2f}%\n")
    with open(os.path.join(OUT, "ncu_summary.json"), "w") as f:
        json.dump(js, f, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
