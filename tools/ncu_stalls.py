"""Top stall reasons (per issue-active, ncu raw page) of the kernels in an ncu
report: python tools/ncu_stalls.py REP.ncu-rep [KERNEL_REGEX] [N]"""
import csv
import subprocess
import sys

rep = sys.argv[1]
kre = sys.argv[2] if len(sys.argv) > 2 else "."
n = int(sys.argv[3]) if len(sys.argv) > 3 else 8
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "-k", f"regex:{kre}"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[0]
keys = {"time_us": "gpu__time_duration.sum",
        "issue_active": "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "warps_active": "smsp__warps_active.avg.pct_of_peak_sustained_active",
        "simt": "smsp__thread_inst_executed_per_inst_executed.ratio",
        "regs": "launch__registers_per_thread", "occ": "sm__warps_active.avg.pct_of_peak_sustained_active",
        "dram_rd": "dram__bytes_read.sum", "dram_wr": "dram__bytes_write.sum",
        "l1_hit": "l1tex__t_sector_hit_rate.pct", "l2_hit": "lts__t_sector_hit_rate.pct"}
idx = [i for i, c in enumerate(h) if c.startswith("smsp__average_warps_issue_stalled_")
       and c.endswith("_per_issue_active.ratio")]
for r in rows[2:]:
    print(r[h.index("Kernel Name")][:70])
    print("   " + ", ".join(f"{k}={r[h.index(v)]}" for k, v in keys.items() if v in h))
    st = sorted(((float(r[i]) if r[i] not in ("", "n/a") else 0.0, h[i]) for i in idx), reverse=True)
    print("   stalls/issue: " + ", ".join(
        f"{c.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', '')}"
        f"={v:.2f}" for v, c in st[:n]))
