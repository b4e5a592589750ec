"""Render tools/sweep.py JSON (soft-barrier threshold sweeps, paper Fig. 9 /
Sec. 5.3) as a markdown table.

usage: python tools/sweep_report.py <sweep.json> [...] > profiles/threshold_sweep_<tag>.md
"""
import json
import sys


def main():
    print("# Soft-barrier threshold sweep (paper Fig. 9, Sec. 5.3 P:1392-1430)\n")
    print("One B200, CUDA events per launch (median), L2 flushed between launches. "
          "`region eff` = active lanes / (32 x executions) of the common code (schedule "
          "counters of the instrumented kernels, SR_F_SCHED). T = 1 reproduces the PDOM "
          "schedule; T = 32 waits for every lane (Fig. 1(b)).\n")
    for path in sys.argv[1:]:
        d = json.load(open(path))
        for wl, rows in d.items():
            unit = {"mcml": "photons_per_s", "divloop": "thread_iters_per_s",
                    "pathtrace": "paths_per_s", "rsbench": "lookups_per_s",
                    "rsfetch": "lookups_per_s"}[wl]
            base = {r["block"]: r["ms"] for r in rows if r["mode"] == "pdom"}
            print(f"## {wl} ({path.split('/')[-1]})\n")
            print("| block | mode | T | ms | speedup vs PDOM | rate | region eff | rounds | "
                  "releases | advances |")
            print("|---|---|---|---|---|---|---|---|---|---|")
            for r in rows:
                sp = base[r["block"]] / r["ms"]
                print(f"| {r['block']} | {r['mode']} | {r['T']} | {r['ms']:.4g} | {sp:.3f} | "
                      f"{r[unit]:.4g} | {r['region_eff']:.3f} | {r['rounds']} | {r['releases']} | "
                      f"{r['advances']} |")
            best = min((r for r in rows if r["mode"] == "spec"), key=lambda r: r["ms"])
            print(f"\nBest threshold: T = {best['T']} (block {best['block']}), "
                  f"{base[best['block']] / best['ms']:.3f}x over PDOM.\n")


if __name__ == "__main__":
    main()
