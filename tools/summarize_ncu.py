"""Summarise the ncu CSVs of tools/gpu_profile.sh into profiles/ (run here, no GPU).

usage: python tools/summarize_ncu.py <tag> [--steps-per-photon X]

Writes
  profiles/simt_<tag>.md            per-kernel SIMT efficiency, issue, pipes, DRAM, time
  profiles/simt_efficiency.json     the same, machine-readable (bench.py embeds it)
  profiles/work_per_unit.json       algorithmic work per unit for the rooflines
  profiles/launches_<tag>.md        the launch list of one bench run and each kernel's share
"""
import csv
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")


def read_ncu_csv(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, {}
    for r in rows:
        if len(r) > 5 and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            name = re.sub(r"\(.*", "", d["Kernel Name"]).replace("void sr::<unnamed>::", "")
            key = (int(d["ID"]), name)
            data.setdefault(key, {})[d["Metric Name"]] = d["Metric Value"].replace(",", "")
    return data


def num(x):
    try:
        return float(x)
    except (TypeError, ValueError):
        return None


def main():
    tag = sys.argv[1]
    os.makedirs(PROF, exist_ok=True)
    simt = read_ncu_csv(os.path.join(OUT, f"simt_{tag}.csv"))
    names = {0: "divloop_pdom", 1: "divloop_spec(T=16)", 2: "commoncall_pdom",
             3: "commoncall_spec", 4: "mcml_pdom", 5: "mcml_spec(T=32)"}
    table, js = [], {}
    for (i, kname), m in sorted(simt.items()):
        label = names.get(i, kname)
        ratio = num(m.get("smsp__thread_inst_executed_per_inst_executed.ratio"))
        eff = ratio / 32 if ratio else None
        row = dict(kernel=kname, simt_efficiency=eff,
                   thread_inst=num(m.get("smsp__thread_inst_executed.sum")),
                   inst=num(m.get("smsp__inst_executed.sum")),
                   issue_active_pct=num(m.get("smsp__issue_active.avg.pct_of_peak_sustained_active")),
                   warps_active_pct=num(m.get("smsp__warps_active.avg.pct_of_peak_sustained_active")),
                   time_ns=num(m.get("gpu__time_duration.sum")),
                   sm_hz=num(m.get("sm__cycles_elapsed.avg.per_second")),
                   dram_bytes=(num(m.get("dram__bytes_read.sum")) or 0) + (num(m.get("dram__bytes_write.sum")) or 0),
                   regs=num(m.get("launch__registers_per_thread")),
                   grid=num(m.get("launch__grid_size")), block=num(m.get("launch__block_size")))
        js[label] = row
        table.append(f"| {label} | {eff:.3f} | {row['thread_inst']:.4g} | {row['inst']:.4g} | "
                     f"{row['issue_active_pct']:.1f} | {row['warps_active_pct']:.1f} | "
                     f"{row['time_ns'] / 1e3:.1f} | {row['dram_bytes']:.3g} | {row['regs']:.0f} | "
                     f"{row['grid']:.0f}x{row['block']:.0f} |")
    js["_source"] = f"ncu --metrics ... --clock-control none, tools/one_launch.py, round tag {tag}"
    json.dump(js, open(os.path.join(PROF, "simt_efficiency.json"), "w"), indent=1)
    md = [f"# ncu per-kernel summary ({tag})", "",
          "One launch of each kernel at its BASELINE.json config (tools/one_launch.py), "
          "`ncu --clock-control none`. SIMT efficiency = "
          "`smsp__thread_inst_executed_per_inst_executed.ratio / 32` (P:234-236).", "",
          "| kernel | SIMT eff | thread-inst | warp-inst | issue active % | warps active % | "
          "time us | DRAM bytes | regs | grid |", "|---|---|---|---|---|---|---|---|---|---|",
          *table]
    open(os.path.join(PROF, f"simt_{tag}.md"), "w").write("\n".join(md) + "\n")

    # algorithmic work per unit
    spp = None
    for a in sys.argv[2:]:
        if a.startswith("--steps-per-photon="):
            spp = float(a.split("=")[1])
    wpu = {}
    if spp and "mcml_pdom" in js:
        photons = 1e7
        wpu["mcml_thread_inst_per_step"] = js["mcml_pdom"]["thread_inst"] / (photons * spp)
        wpu["mcml_steps_per_photon"] = spp
        wpu["mcml_spec_dram_bytes_per_launch"] = js.get("mcml_spec(T=32)", {}).get("dram_bytes")
        wpu["basis"] = ("PDOM kernel smsp__thread_inst_executed.sum (active lanes only = the work "
                        "every lane must do) / (10^7 photons x steps per photon); ncu " + tag)
        json.dump(wpu, open(os.path.join(PROF, "work_per_unit.json"), "w"), indent=1)

    lpath = os.path.join(OUT, f"launches_{tag}.csv")
    if os.path.exists(lpath):
        L = read_ncu_csv(lpath)
        tot = sum(num(m.get("gpu__time_duration.sum")) or 0 for m in L.values())
        lines = [f"# launch list of `bench.py --steps 2 --warmup 1` under ncu ({tag})", "",
                 "ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, "
                 "serialised: compare shares, not absolutes).", "",
                 "| id | kernel | time us | share |", "|---|---|---|---|"]
        for (i, k), m in sorted(L.items()):
            t = num(m.get("gpu__time_duration.sum")) or 0
            lines.append(f"| {i} | {k[:60]} | {t / 1e3:.1f} | {t / tot:.3f} |")
        open(os.path.join(PROF, f"launches_{tag}.md"), "w").write("\n".join(lines) + "\n")
    print(json.dumps(wpu, indent=1))


if __name__ == "__main__":
    main()
