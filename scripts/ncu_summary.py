"""Summarise an ncu --set full report: headline metrics + top SASS stall sites.
usage: python scripts/ncu_summary.py report.ncu-rep [n_top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
hdr, vals = r[0], r[2]
want = ["gpu__time_duration.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__cycles_elapsed.avg.per_second", "launch__registers_per_thread", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "launch__grid_size", "launch__block_size"]
for h, v in zip(hdr, vals):
    if h in want:
        print(f"{h:70s} {v}")
stalls = [(h, v) for h, v in zip(hdr, vals) if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued")]
tot = sum(float(v or 0) for _, v in stalls)
for h, v in sorted(stalls, key=lambda x: -float(x[1] or 0))[:8]:
    print(f"  stall {h[33:]:28s} {100 * float(v) / max(tot, 1):5.1f}%")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h2 = rows[1]
data = [dict(zip(h2, x)) for x in rows[2:] if len(x) == len(h2)]
k = "Warp Stall Sampling (All Samples)"
tot = sum(int(d[k] or 0) for d in data)
cols = ["stall_long_sb", "stall_membar", "stall_barrier", "stall_wait", "stall_branch_resolving", "stall_short_sb", "stall_mio", "stall_lg"]
for d in sorted(data, key=lambda d: -int(d[k] or 0))[:ntop]:
    s = int(d[k] or 0)
    extra = " ".join(f"{c[6:]}={d[c]}" for c in cols if d.get(c) not in ("0", "", None))
    print(f"{d['Address'][-5:]} {100 * s / max(tot, 1):5.1f}% {d['Source'][:58]:58s} {extra}")
