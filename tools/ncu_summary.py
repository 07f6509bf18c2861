"""Summarise ncu outputs from gpurun_out/ into tracked files under profiles/.

    python tools/ncu_summary.py <round-tag> <config> [...]

For each config: launches_<cfg>.csv (one-pass metrics of every libgd launch) ->
profiles/<tag>_<cfg>_launches.md (per-kernel count, mean time, share of device time,
DRAM and PCIe bytes per launch) and updates profiles/traffic.json (per-kernel DRAM bytes
per launch, steady state = the last third of the launches).  Every prof_<k>_<cfg>.ncu-rep
(--set full) -> profiles/<tag>_<cfg>_<k>_full.md with the key raw metrics.
"""
import collections
import csv
import glob
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GO = os.environ.get("NCU_DIR", os.path.join(ROOT, "gpurun_out"))
PROF = os.path.join(ROOT, "profiles")


def short(name):
    name = name.split("(")[0].replace("void ", "")
    return name


def launches(cfg):
    p = os.path.join(GO, f"launches_{cfg}.csv")
    rows = list(csv.reader(open(p)))
    hdr = None
    per = collections.defaultdict(lambda: collections.defaultdict(dict))
    order = []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        key = (int(d["ID"]), short(d["Kernel Name"]))
        if key not in per:
            order.append(key)
        unit = d["Metric Unit"]
        try:
            v = float(d["Metric Value"].replace(",", "") or 0)
        except ValueError:
            v = 0.0
        scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3,
                 "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "sector": 1.0}.get(unit, 1.0)
        per[key][d["Metric Name"]] = v * scale
    return order, per


def summarize_launches(tag, cfg):
    order, per = launches(cfg)
    by = collections.defaultdict(list)
    for key in order:
        by[key[1]].append(per[key])
    tot = sum(m.get("gpu__time_duration.sum", 0) for k in order for m in [per[k]])
    lines = [f"# ncu launch list — {cfg} ({tag})", "",
             "One-pass metrics of every libgd kernel launch of `tools/profile.sh " + cfg + "` "
             "(bench.py, 6 timed steps after pre-warm; ncu serialises launches and runs them cold, so compare "
             "SHARES, not absolute times, with bench.py's live event timings).", "",
             "| kernel | launches | mean us | share of device time | DRAM read MB/launch | DRAM write MB/launch | PCIe read MB/launch |",
             "|---|---|---|---|---|---|---|"]
    traffic = {}
    for k, ms in sorted(by.items(), key=lambda kv: -sum(m.get("gpu__time_duration.sum", 0) for m in kv[1])):
        steady = ms[len(ms) * 2 // 3:] or ms
        t = [m.get("gpu__time_duration.sum", 0) for m in ms]
        rd = sum(m.get("dram__bytes_read.sum", 0) for m in steady) / len(steady)
        wr = sum(m.get("dram__bytes_write.sum", 0) for m in steady) / len(steady)
        pc = sum(m.get("pcie__read_bytes.sum", 0) for m in steady) / len(steady)
        lines.append(f"| {k} | {len(ms)} | {sum(t)/len(t):.1f} | {100*sum(t)/max(tot,1e-9):.1f}% | "
                     f"{rd/1e6:.2f} | {wr/1e6:.2f} | {pc/1e6:.2f} |")
        traffic[k] = round(rd + wr)
    out = os.path.join(PROF, f"{tag}_{cfg}_launches.md")
    open(out, "w").write("\n".join(lines) + "\n")
    tp = os.path.join(PROF, "traffic.json")
    allt = json.load(open(tp)) if os.path.exists(tp) else {}
    allt[cfg] = {"_note": f"dram__bytes_read.sum + dram__bytes_write.sum per launch (bytes), steady-state "
                          f"launches of {tag}_{cfg}_launches.md", **traffic}
    json.dump(allt, open(tp, "w"), indent=1)
    print(out)


WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__occupancy_limit_registers", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed.sum"]


def summarize_full(tag, cfg):
    for rep in sorted(glob.glob(os.path.join(GO, f"prof_*_{cfg}.ncu-rep"))):
        k = os.path.basename(rep)[len("prof_"):-len(f"_{cfg}.ncu-rep")]
        txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(txt)))
        if len(rows) < 3:
            continue
        h, u = rows[0], rows[1]
        lines = [f"# ncu --set full — {k} on {cfg} ({tag})", "", "| metric | value | unit |", "|---|---|---|"]
        for r in rows[2:]:
            for i, name in enumerate(h):
                if name in WANT or name.startswith("smsp__pcsamp_warps_issue_stalled") and False:
                    lines.append(f"| {name} | {r[i]} | {u[i]} |")
            lines.append("| | | |")
        # top stall reasons
        stall = [(h[i], r[i]) for r in rows[2:3] for i in range(len(h))
                 if h[i].startswith("smsp__average_warp_latency_issue_stalled") and h[i].endswith(".ratio")]
        if stall:
            lines += ["", "Top stall reasons (warp latency per issue, ratio):", ""]
            for n, v in sorted(stall, key=lambda x: -float(x[1] or 0))[:6]:
                lines.append(f"- {n}: {v}")
        out = os.path.join(PROF, f"{tag}_{cfg}_{k}_full.md")
        open(out, "w").write("\n".join(lines) + "\n")
        print(out)


if __name__ == "__main__":
    os.makedirs(PROF, exist_ok=True)
    tag = sys.argv[1]
    for cfg in sys.argv[2:]:
        if os.path.exists(os.path.join(GO, f"launches_{cfg}.csv")):
            summarize_launches(tag, cfg)
        summarize_full(tag, cfg)
