"""Summarise the ncu CSVs of tools/gpu_profile.sh into profiles/ (run here, no GPU).

usage: python tools/summarize_ncu.py <tag>

Writes
  profiles/simt_<tag>.md            per-kernel SIMT efficiency, issue, warps, time
  profiles/simt_efficiency.json     the same, machine-readable (bench.py embeds it;
                                    tools/simt_predict.py compares against it)
  profiles/work_per_unit.json       algorithmic work per unit for the rooflines
  profiles/launches_<tag>.md        launch list of one bench run, each kernel's share
"""
import csv
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

# launch order of tools/one_launch.py (default: every family, pdom then spec)
sys.path.insert(0, ROOT)
from paper_conf_cgo_damanijskymg20_b200 import inputs as _I  # noqa: E402

_TRS = _I.NEXT1.threshold
LABELS_ALL = ["divloop_pdom", "divloop_spec(T=16)", "commoncall_pdom", "commoncall_spec",
              "mcml_pdom", "mcml_spec(T=32)", "rs_pdom", f"rs_spec(T={_TRS})", "pt_pdom",
              f"pt_spec(T={_I.C4.threshold})"]
LABELS_DLBATCH = ["divloop_pdom_batch", "divloop_spec_batch(T=16)"]
LABELS_RSSTATIC = [f"rs_spec_static(T={_TRS})"]
LABELS_DLPOOL = ["divloop_pool(T=16)"]
LABELS_DLPOOL4 = ["divloop_pool_split4(T=16)"]
LABELS_PTPOOL = [f"pt_spec_pool(T={_I.C4.threshold})"]
LABELS_MCSTATIC = ["mcml_pdom_static", "mcml_spec_static(T=32)"]
LABELS_MCSTATIC8 = ["mcml_spec_static(T=8)"]
LABELS_MCSTATICU4 = ["mcml_spec_static(T=32,U=4)"]


def gbs(r, hbm):
    """achieved DRAM GB/s of one launch and its share of the measured HBM peak"""
    if not r.get("dram_bytes") or not r.get("time_ns"):
        return "-"
    g = r["dram_bytes"] / r["time_ns"]
    return f"{g:.3g} ({100 * g / hbm:.2g} %)"


def read_ncu_csv(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, {}
    for r in rows:
        if len(r) > 5 and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            name = re.sub(r"\([^()]*\)$", "", d["Kernel Name"].strip())
            name = name.replace("void ", "").replace("sr::<unnamed>::", "")
            key = (int(d["ID"]), name)
            data.setdefault(key, {})[d["Metric Name"]] = d["Metric Value"].replace(",", "")
    return [(k[1], v) for k, v in sorted(data.items())]


def mangle_match(demangled, mangled):
    """'divloop_spec<125, false>' vs '_ZN..12divloop_specILi125ELb0EE..'"""
    m = re.search(r"(\w+)<([^<>]*)>\s*$", demangled.strip())
    if not m:
        return False
    name, args = m.group(1), [a.strip() for a in m.group(2).split(",")]
    enc = ""
    for a in args:
        v = a.replace("(bool)", "").replace("(int)", "").strip()
        v = {"true": "1", "false": "0"}.get(v, v)
        enc += r"L[bi]%sE" % re.escape(v)   # ncu may print bools as 0/1
    return re.search(r"\d" + name + r"I" + enc + r"E", mangled) is not None


def num(x):
    try:
        return float(x)
    except (TypeError, ValueError):
        return None


def row_of(kname, m):
    ratio = num(m.get("smsp__thread_inst_executed_per_inst_executed.ratio"))
    return dict(kernel=kname, simt_efficiency=ratio / 32 if ratio else None,
                thread_inst=num(m.get("smsp__thread_inst_executed.sum")),
                inst=num(m.get("smsp__inst_executed.sum")),
                issue_active_pct=num(m.get("smsp__issue_active.avg.pct_of_peak_sustained_active")),
                warps_active_pct=num(m.get("smsp__warps_active.avg.pct_of_peak_sustained_active")),
                time_ns=num(m.get("gpu__time_duration.sum")),
                sm_hz=num(m.get("sm__cycles_elapsed.avg.per_second")),
                dram_bytes=(num(m.get("dram__bytes_read.sum")) or 0) +
                (num(m.get("dram__bytes_write.sum")) or 0),
                l2_bytes=num(m.get("lts__t_bytes.sum")),
                ffma_thread_inst=num(m.get("sm__sass_thread_inst_executed_op_ffma_pred_on.sum")),
                ffma2_thread_inst=num(m.get("sm__sass_thread_inst_executed_op_ffma2_pred_on.sum")),
                regs=num(m.get("launch__registers_per_thread")),
                grid=num(m.get("launch__grid_size")), block=num(m.get("launch__block_size")))


def main():
    tag = sys.argv[1]
    os.makedirs(PROF, exist_ok=True)
    js = {}
    for fname, labels in ((f"simt_{tag}.csv", LABELS_ALL),
                          (f"simt_mcstatic_{tag}.csv", LABELS_MCSTATIC),
                          (f"simt_mcstatic8_{tag}.csv", LABELS_MCSTATIC8),
                          (f"simt_mcstaticu4_{tag}.csv", LABELS_MCSTATICU4),
                          (f"simt_dlbatch_{tag}.csv", LABELS_DLBATCH),
                          (f"simt_rsstatic_{tag}.csv", LABELS_RSSTATIC),
                          (f"simt_dlpool_{tag}.csv", LABELS_DLPOOL),
                          (f"simt_dlpool4_{tag}.csv", LABELS_DLPOOL4),
                          (f"simt_ptpool_{tag}.csv", LABELS_PTPOOL)):
        path = os.path.join(OUT, fname)
        if not os.path.exists(path):
            continue
        for lab, (kname, m) in zip(labels, read_ncu_csv(path)):
            js[lab] = row_of(kname, m)
    js["_source"] = (f"ncu --metrics ... --clock-control none; tools/one_launch.py; round tag {tag};"
                     " libsr built from this commit")
    sys.path.insert(0, os.path.join(ROOT, "tools"))
    import sass_regions
    hpath = os.path.join(OUT, f"sass_hashes_{tag}.json")
    if os.path.exists(hpath):   # hashed on the GPU box, from the build it measured
        hashes = json.load(open(hpath))
    else:
        print("warning: no box-side SASS hashes; hashing the local build", file=sys.stderr)
        hashes = sass_regions.kernel_hashes("divloop_|commoncall_|mcml_|pt_|rs_")
    for lab, r in js.items():
        if isinstance(r, dict):
            mangled = [k for k in hashes if mangle_match(r["kernel"], k)]
            r["sass_sha"] = hashes[mangled[0]] if len(mangled) == 1 else None
    json.dump(js, open(os.path.join(PROF, "simt_efficiency.json"), "w"), indent=1)
    md = [f"# ncu per-kernel summary ({tag})", "",
          "One launch of each kernel (tools/one_launch.py), `ncu --clock-control none`. "
          "SIMT efficiency = `smsp__thread_inst_executed_per_inst_executed.ratio / 32` "
          "(P:234-236). `*_static` rows: the simulator-validation launches (16384 lanes x 8 "
          "photons, static assignment).", "",
          "| kernel | SIMT eff | thread-inst | warp-inst | issue active % | warps active % | "
          "time us | DRAM bytes | DRAM GB/s (% of HBM peak) | L2 bytes | regs | grid x block |",
          "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    hbm = peaks.get("hbm_gbs", 6537.0)
    for lab, r in js.items():
        if lab.startswith("_"):
            continue
        f = lambda v, fmt: (fmt % v) if v is not None else "-"
        md.append(f"| {lab} | {f(r['simt_efficiency'], '%.3f')} | {f(r['thread_inst'], '%.4g')} | "
                  f"{f(r['inst'], '%.4g')} | {f(r['issue_active_pct'], '%.1f')} | "
                  f"{f(r['warps_active_pct'], '%.1f')} | {f(r['time_ns'] and r['time_ns'] / 1e3, '%.1f')} | "
                  f"{f(r['dram_bytes'], '%.3g')} | {gbs(r, hbm)} | "
                  f"{f(r['l2_bytes'], '%.3g')} | {f(r['regs'], '%.0f')} | "
                  f"{f(r['grid'], '%.0f')}x{f(r['block'], '%.0f')} |")
    open(os.path.join(PROF, f"simt_{tag}.md"), "w").write("\n".join(md) + "\n")

    # algorithmic work per unit (PDOM thread-instructions = the work every lane must do)
    wpu = json.load(open(os.path.join(PROF, "work_per_unit.json"))) if os.path.exists(
        os.path.join(PROF, "work_per_unit.json")) else {}
    bj = os.path.join(OUT, f"bench_{tag}.json")
    if os.path.exists(bj) and "mcml_pdom" in js:
        b = json.load(open(bj))
        spp = b["steps_per_photon"]
        photons = b["config"]["photons_per_gpu"]
        wpu["mcml_thread_inst_per_step"] = js["mcml_pdom"]["thread_inst"] / (photons * spp)
        wpu["mcml_steps_per_photon"] = spp
        wpu["basis"] = ("PDOM kernel smsp__thread_inst_executed.sum (active lanes only = the work "
                        "every lane must do) / (photons x steps per photon); ncu " + tag)
    tpath = os.path.join(OUT, f"traffic_{tag}.csv")
    if os.path.exists(tpath):
        t = read_ncu_csv(tpath)
        if t:
            m = t[0][1]
            wpu["mcml_spec_dram_bytes_per_launch"] = (num(m.get("dram__bytes_read.sum")) or 0) + \
                (num(m.get("dram__bytes_write.sum")) or 0)
    json.dump(wpu, open(os.path.join(PROF, "work_per_unit.json"), "w"), indent=1)

    lpath = os.path.join(OUT, f"launches_{tag}.csv")
    if os.path.exists(lpath):
        L = read_ncu_csv(lpath)
        tot = sum(num(m.get("gpu__time_duration.sum")) or 0 for _, m in L)
        lines = [f"# launch list of `bench.py --steps 2 --warmup 1` under ncu ({tag})", "",
                 "ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, "
                 "serialised: compare shares, not absolutes).", "",
                 "| # | kernel | time us | share |", "|---|---|---|---|"]
        for i, (k, m) in enumerate(L):
            t = num(m.get("gpu__time_duration.sum")) or 0
            lines.append(f"| {i} | {k[:70]} | {t / 1e3:.1f} | {t / tot:.3f} |")
        open(os.path.join(PROF, f"launches_{tag}.md"), "w").write("\n".join(lines) + "\n")
    print(json.dumps(wpu, indent=1))


if __name__ == "__main__":
    main()
