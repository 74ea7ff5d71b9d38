#!/usr/bin/env bash
# Summarise one ncu --set full report (first kernel in it) into the text format of profiles/*_ncu_summary.txt
set -u
rep=$1
ncu -i "$rep" --page raw --csv 2>/dev/null > /tmp/ncu_raw.csv
python - "$rep" <<'PY'
import csv, sys
rows = list(csv.reader(open('/tmp/ncu_raw.csv')))
hdr, units, vals = rows[0], rows[1], rows[2]
d = {h: (u, v) for h, u, v in zip(hdr, units, vals)}
keys = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "smsp__inst_executed.sum", "sm__cycles_elapsed.avg.per_second"]
for k in keys:
    if k in d:
        u, v = d[k]
        print(f"{k:<84}{u:>6} {v}")
st = []
for h, (u, v) in d.items():
    if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
        try: st.append((float(v), h))
        except ValueError: pass
print("top stalls (warps per issue):")
for v, h in sorted(st, reverse=True)[:8]:
    print(f"  {v:8.3f} {h}")
PY
