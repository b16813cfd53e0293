"""Summarise an ncu report (raw page): key throughput metrics + top stall reasons per kernel."""
import csv, subprocess, sys, io
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units = rows[0], rows[1]
want = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__inst_executed.sum', 'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread', 'launch__grid_size',
        'launch__block_size', 'launch__occupancy_limit_shared_mem', 'launch__occupancy_limit_registers',
        'sm__maximum_warps_per_active_cycle_pct', 'lts__t_bytes.sum', 'smsp__cycles_active.avg']
for r in rows[2:]:
    print("==", r[hdr.index('Kernel Name')][:60])
    for w in want:
        if w in hdr:
            i = hdr.index(w)
            print(f"   {w:60s} {r[i]} {units[i]}")
    st = [(hdr[i], float(r[i])) for i in range(len(hdr)) if hdr[i].startswith('smsp__average_warps_issue_stalled_')
          and hdr[i].endswith('_per_issue_active.ratio') and r[i] not in ('', 'n/a')]
    st.sort(key=lambda t: -t[1])
    for k, v in st[:7]:
        print('   stall %-50s %.3f' % (k.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', ''), v))
