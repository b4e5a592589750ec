"""Per-source-line instruction and stall profile of one kernel in an ncu report
(needs -lineinfo builds and `ncu --import-source on`).

usage: python tools/ncu_lines.py <report.ncu-rep> [top]
Prints lines sorted by warp-level instructions executed, with the mean active
lanes per instruction (the line's SIMT efficiency x 32) and stall share.
"""
import csv
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    kern = ["--kernel-name", f"regex:{sys.argv[3]}"] if len(sys.argv) > 3 else []
    out = subprocess.run(["ncu", "-i", rep, *kern, "--page", "source", "--csv", "--print-source",
                          "cuda,sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    file = "?"
    lines = []
    hdr = None
    for r in rows:
        if r and r[0] == "File Path":
            file = r[1].split("/")[-1]
        elif r and r[0] == "Line No":
            hdr = r
        elif hdr and r and r[0] not in ("", "Function Name"):
            try:
                d = dict(zip(hdr[4:], r[4:]))
                lines.append((float(d["Instructions Executed"]), float(d["Thread Instructions Executed"]),
                              float(d["Warp Stall Sampling (All Samples)"]), f"{file}:{r[0]}", r[1]))
            except (ValueError, KeyError):
                pass
    ti = sum(l[0] for l in lines) or 1
    ts = sum(l[2] for l in lines) or 1
    tt = sum(l[1] for l in lines)
    print(f"total warp-inst {ti:.4g}  thread-inst {tt:.4g}  SIMT {tt / ti / 32:.3f}")
    for l in sorted(lines, reverse=True)[:top]:
        print(f"{l[0] / ti * 100:5.1f}%  lanes {l[1] / max(l[0], 1):5.1f}  stall {l[2] / ts * 100:5.1f}%"
              f"  {l[3]:<16} {l[4][:80]}")


if __name__ == "__main__":
    main()
