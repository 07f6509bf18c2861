"""Kernel / copy timeline of a few pipelined steps (the overlap evidence nsys would give; nsys
is not in this image).  bench.py --timeline <out.md> runs extra steps under torch.profiler
(CUPTI activity tracing: every kernel of the process, libgd's included, and every memcpy with
its stream and device timestamps) and calls summarise() on the chrome trace.

The summary answers one question of the paper's design ("asynchronous extraction", P:207
overlapping I/O with computation): while the misses of batch b stream in (zero-copy kernel,
copy-engine H2D chunks, staged scatter), is the GPU already sampling batch b + 1?
"""
from __future__ import annotations

import collections
import json

SAMPLING = ("k_seed_intake", "k_sample_hop", "k_relabel_hop", "k_sample_pad", "k_relabel_pad", "k_col_resolve",
            "k_hash_clear")
BOOKKEEPING = ("k_lookup", "k_pop_assign", "k_release", "k_compact")
CATS = [
    ("sampling (a1-a4)", lambda n, k: k == "kernel" and n.startswith(SAMPLING)),
    ("bookkeeping (a5, a6, a9)", lambda n, k: k == "kernel" and n.startswith(BOOKKEEPING)),
    ("hit gather (a8)", lambda n, k: k == "kernel" and n.startswith(("k_gather_rows", "k_gather_tma", "k_gather_hits"))),
    ("miss zero-copy kernel (a7)", lambda n, k: k == "kernel" and n.startswith(("k_miss_copy<4, 0>", "k_miss_copy<4, false>",
                                                                             "k_miss_copy_w4<false>", "k_miss_copy_w4<0>"))),
    ("miss copy-engine H2D (a7)", lambda n, k: k == "gpu_memcpy" and "HtoD" in n),
    ("miss staged scatter (a7)", lambda n, k: k == "kernel" and n.startswith(("k_miss_copy<4, 1>", "k_miss_copy<4, true>",
                                                                           "k_miss_copy_w4<true>", "k_miss_copy_w4<1>"))),
]


def _short(name: str) -> str:
    n = name.replace("void ", "").replace("gd::", "")
    return n.split("(")[0]


def _union(iv):
    out = []
    for a, b in sorted(iv):
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def _length(iv):
    return sum(b - a for a, b in iv)


def _intersect(x, y):
    i = j = 0
    out = []
    while i < len(x) and j < len(y):
        a, b = max(x[i][0], y[j][0]), min(x[i][1], y[j][1])
        if a < b:
            out.append([a, b])
        if x[i][1] < y[j][1]:
            i += 1
        else:
            j += 1
    return out


def summarise(trace_path: str, out_md: str, steps: int, title: str) -> dict:
    ev = json.load(open(trace_path))
    ev = ev["traceEvents"] if isinstance(ev, dict) else ev
    acts = []
    for e in ev:
        cat = e.get("cat", "")
        if cat not in ("kernel", "gpu_memcpy") or "dur" not in e:
            continue
        name = _short(e.get("name", ""))
        if cat == "kernel" and not name.startswith(("k_", "umma::")):
            continue        # torch's own copies / fills of the bench loop
        acts.append((float(e["ts"]), float(e["dur"]), name, cat, e.get("args", {}).get("stream", -1)))
    if not acts:
        open(out_md, "w").write(f"# {title}\n\nno GPU activity captured\n")
        return {}
    t0 = min(a[0] for a in acts)
    t1 = max(a[0] + a[1] for a in acts)
    win = t1 - t0
    cats = {}
    for cname, pred in CATS:
        cats[cname] = _union([[a[0], a[0] + a[1]] for a in acts if pred(a[2], a[3])])
    samp = cats["sampling (a1-a4)"]
    rows = []
    for cname, _ in CATS:
        iv = cats[cname]
        busy = _length(iv)
        ov = _length(_intersect(iv, samp)) if cname != "sampling (a1-a4)" else None
        rows.append((cname, busy, busy / win if win else 0, ov, (ov / busy) if (ov is not None and busy) else None))
    miss = _union([x for c in ("miss zero-copy kernel (a7)", "miss copy-engine H2D (a7)", "miss staged scatter (a7)")
                   for x in cats[c]])
    miss_busy = _length(miss)
    miss_ov = _length(_intersect(miss, samp))
    per_stream = collections.defaultdict(lambda: collections.Counter())
    for ts, dur, name, cat, st in acts:
        per_stream[st][name.split("<")[0] if cat == "kernel" else ("memcpy " + name)] += dur
    lines = [f"# {title}", "",
             f"{steps} pipelined steps under torch.profiler (CUPTI activity trace of every kernel and copy in the",
             "process; the profiler's own overhead stretches the steps, so read overlaps and shares, not rates).",
             f"Window {win / 1e3:.2f} ms = {win / 1e3 / steps:.3f} ms per step.", "",
             "| activity | busy ms | share of window | overlapped with sampling ms | share of it overlapped |",
             "|---|---|---|---|---|"]
    for c, busy, sh, ov, osh in rows:
        lines.append(f"| {c} | {busy / 1e3:.3f} | {sh:.1%} | {'-' if ov is None else f'{ov / 1e3:.3f}'} | "
                     f"{'-' if osh is None else f'{osh:.1%}'} |")
    lines += ["", f"All miss-path activity (union): {miss_busy / 1e3:.3f} ms busy, {miss_ov / 1e3:.3f} ms of it "
              f"({(miss_ov / miss_busy if miss_busy else 0):.1%}) concurrent with sampling kernels.", "",
              "## Busy time per stream (ms)", "", "| stream | top activities |", "|---|---|"]
    for st, cnt in sorted(per_stream.items(), key=lambda kv: -sum(kv[1].values())):
        top = ", ".join(f"{k} {v / 1e3:.2f}" for k, v in cnt.most_common(5))
        lines.append(f"| {st} | {top} |")
    # ASCII Gantt of the middle two steps, 20 columns per step-width slice
    mid0 = t0 + win * 0.4
    mid1 = mid0 + 2 * win / steps
    cols = 100
    lines += ["", f"## Gantt, two steps from {((mid0 - t0) / 1e3):.2f} ms ({(mid1 - mid0) / cols:.1f} us per column)", "",
              "```"]
    for cname, _ in CATS:
        row = [" "] * cols
        for a, b in cats[cname]:
            if b < mid0 or a > mid1:
                continue
            for c in range(max(0, int((a - mid0) / (mid1 - mid0) * cols)), min(cols, int((b - mid0) / (mid1 - mid0) * cols) + 1)):
                row[c] = "#"
        lines.append(f"{cname[:28]:28s} |{''.join(row)}|")
    lines += ["```", ""]
    open(out_md, "w").write("\n".join(lines) + "\n")
    return {"window_ms": round(win / 1e3, 3), "miss_busy_ms": round(miss_busy / 1e3, 3),
            "miss_overlapped_with_sampling_ms": round(miss_ov / 1e3, 3),
            "miss_overlap_share": round(miss_ov / miss_busy, 4) if miss_busy else None}
