"""Markdown table of the committed bench lines (profiles/<tag>_<config>_bench.json) for
DESIGN.md §8 / README.md, so quoted numbers are the committed JSON's, not retyped.

    python tools/bench_table.py [tag]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r02"
rows = ["| config | batches/s | e2e | dominant bound | hit gather live / alone | parity in the run | CPU oracle (all cores / 1 thread) |",
        "|---|---|---|---|---|---|---|"]
for c in ("papers100m", "friendster", "mag240m", "products", "tiny"):
    p = os.path.join(ROOT, "profiles", f"{tag}_{c}_bench.json")
    if not os.path.exists(p):
        continue
    d = json.load(open(p))
    r = d["roofline"]
    if r["bound"] == "host_link":
        bound = f"host link {r['achieved']} / {r['peak']} GB/s = {r['frac']:.1%}"
    else:
        bound = f"{r['bound']} (no misses): sampling latency"
    g = d["roofline_gather"]
    gi = g.get("isolated") or {}
    par = d["parity"]
    first, ss = par["first"], par["steady_state"]
    pstr = (f"first {first['batches']} in full + replay of {ss['batches']} batches "
            f"({'bit-exact' if par['bit_exact'] else 'MISMATCH'}, final state {'equal' if ss['final_state_equal'] else 'differs'})")
    cb = d.get("cpu_baseline") or {}
    st = cb.get("single_thread_full_oracle") or {}
    rows.append(f"| {c} | {d['value']:.0f} | {d['e2e']['value']:.0f} | {bound} | {g['frac']:.1%} / "
                f"{gi.get('frac', 0):.1%} | {pstr} | {cb.get('value', '-')} ({cb.get('cores', '-')} cores) / "
                f"{st.get('value', '-')} |")
print("\n".join(rows))
