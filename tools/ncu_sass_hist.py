"""Stall samples and executed instructions per SASS opcode of one kernel in an
ncu report (--page source): python tools/ncu_sass_hist.py REP.ncu-rep KERNEL_REGEX"""
import csv
import subprocess
import sys
from collections import Counter

rep, kre = sys.argv[1], sys.argv[2]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", f"regex:{kre}"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = next(r for r in rows if "Source" in r and "Warp Stall Sampling (All Samples)" in r)
iS, iE, iSrc = (hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed"),
                hdr.index("Source"))
f = lambda x: int(x) if x.strip().isdigit() else 0  # noqa: E731
c, e = Counter(), Counter()
for r in rows:
    if len(r) <= max(iS, iE, iSrc) or r is hdr or r[0] == "Kernel Name":
        continue
    t = r[iSrc].split()
    if not t:
        continue
    op = (t[1] if t[0].startswith("@") and len(t) > 1 else t[0]).split(".")[0]
    c[op] += f(r[iS])
    e[op] += f(r[iE])
tot = sum(c.values())
print(f"samples {tot}, warp-inst {sum(e.values())}")
for op, v in c.most_common(int(sys.argv[3]) if len(sys.argv) > 3 else 15):
    print(f"{op:10s} samples {v:7d} ({v / max(tot, 1):.3f})  warp-inst {e[op]}")
