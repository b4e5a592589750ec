"""Stall samples and executed warp-instructions per CUDA source line (innermost
inline frame) of one kernel in an ncu report:
python tools/ncu_line_hist.py REP.ncu-rep KERNEL_REGEX [N]"""
import csv
import subprocess
import sys

rep, kre = sys.argv[1], sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "-k", f"regex:{kre}"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
f = lambda x: int(x) if x.strip().isdigit() else 0  # noqa: E731
items, fname = [], ""
for r in rows:
    if r and r[0] in ("File Path", "File Name"):
        fname = r[1].split("/")[-1]
        continue
    if len(r) > 8 and r[0].isdigit() and r[2] == "-":   # a source line aggregate
        items.append((f(r[4]), f(r[7]), f(r[8]), f"{fname}:{r[0]}", r[1].strip()[:80]))
tot = sum(i[0] for i in items)
ti = sum(i[1] for i in items)
print(f"samples {tot}, warp-inst {ti}")
for s_, e_, t_, ln, src in sorted(items, reverse=True)[:n]:
    print(f"{s_:7d} {s_ / max(tot, 1):.3f} inst {e_ / max(ti, 1):.3f} simt {t_ / max(e_, 1) / 32:.2f} {ln:18s} {src}")
