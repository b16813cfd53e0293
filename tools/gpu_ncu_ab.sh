#!/bin/bash
# HW-counter comparison of variants (compress + decompress kernels) on a config
CFG=${CFG:-c3_hacc}; REL=${REL:-1e-3}
M=gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio,smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio,smsp__average_warps_issue_stalled_wait_per_issue_active.ratio,smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio,smsp__average_warps_issue_stalled_sleeping_per_issue_active.ratio,smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio,smsp__average_warps_issue_stalled_membar_per_issue_active.ratio,smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio,smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio
timeout 600 ncu --metrics $M --clock-control none -k regex:"compress_kernel|decompress_kernel" --csv python tools/ncu_ab.py "$@" --config $CFG --rel $REL > gpurun_out/ncu_ab_$TAG.csv 2> gpurun_out/ncu_ab_$TAG.err
python - <<'PY'
import csv, os
rows = list(csv.reader(open(f"gpurun_out/ncu_ab_{os.environ.get('TAG','')}.csv")))
i = next(k for k, r in enumerate(rows) if r and r[0] == "ID")
h = rows[i]
data = {}
for r in rows[i + 1:]:
    if len(r) < len(h): continue
    d = dict(zip(h, r))
    data.setdefault((d["ID"], d["Kernel Name"][:40]), {})[d["Metric Name"]] = d["Metric Value"]
for (kid, kn), m in sorted(data.items(), key=lambda t: int(t[0][0])):
    short = {k.replace("smsp__average_warps_issue_stalled_", "st_").replace("_per_issue_active.ratio", ""): v for k, v in m.items()}
    print(kid, kn, " ".join(f"{k.split('.')[0]}={v}" for k, v in sorted(short.items())))
PY
