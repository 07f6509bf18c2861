"""The same configs on the pool's boxes (the host side varies box to box): one row per config,
one column per box, from profiles/r02_boxes/box<X>_<config>_bench.json and the final lines
profiles/r02_<config>_bench.json (box C, final code).

    python tools/boxes_table.py
"""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = os.path.join(ROOT, "profiles")
BOXES = [("A", os.path.join(P, "r02_boxes", "boxA_{}_bench.json"), "code before the double-buffered hash, sample-ahead 3"),
         ("B", os.path.join(P, "r02_boxes", "boxB_{}_bench.json"), "code before the double-buffered hash, sample-ahead 3"),
         ("C", os.path.join(P, "r02_boxes", "boxC_{}_bench.json"), "double-buffered hash, sample-ahead 3"),
         ("D", os.path.join(P, "r02_boxes", "boxD_{}_bench.json"), "sample-ahead 0 with a miss path"),
         ("E", os.path.join(P, "r02_boxes", "boxE_{}_bench.json"), "4 positions per thread in k_relabel_pad"),
         ("final", os.path.join(P, "r02_{}_bench.json"), "final code (e2e region with its own warm-up steps): the "
                                                          "committed lines, all from one box")]


def cell(path):
    if not os.path.exists(path):
        return "-"
    d = json.loads(open(path).readline())
    r = d["roofline"]
    s = f"{d['value']:.0f}"
    if r["bound"] == "host_link":
        hg = (r.get("per_path_GBps") or {}).get("host_gather_phase1")
        s += f" (link {r['frac']:.0%}, host gather {hg:.0f} GB/s)" if hg else f" (link {r['frac']:.0%})"
    return s


print("| config | " + " | ".join(f"box {b}" for b, _, _ in BOXES) + " |")
print("|---|" + "---|" * len(BOXES))
for c in ("papers100m", "friendster", "mag240m", "products", "tiny"):
    print(f"| {c} | " + " | ".join(cell(t.format(c)) for _, t, _ in BOXES) + " |")
print()
print("; ".join(f"box {b}: {why}" for b, _, why in BOXES) + ".  batches/s of the default `bench.py --config <config>` line.")
