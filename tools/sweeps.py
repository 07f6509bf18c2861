"""f3: the paper's sweeps on the built path, one bench.py process per
point, every point with its first batches checked against the oracle and the oracle replay of
its whole schedule (steady-state parity); raw JSON lines to profiles/<tag>_sweeps/, the table
to profiles/<tag>_sweeps_<config>.md.

    python tools/sweeps.py <tag> [config] [steps]

* buffer size (Fig. 12; reading R13): buffer_frac in {0.04, 0.10, 0.20, 0.40} of N
* feature dimension (Fig. 8): 32, 64, 128, 256, 512 fp32.  512 would be a 227 GB
  host table, above this pool's 196 GB of host RAM: that point runs on a bounded physical
  table of 40M rows (node v -> row v mod 40M, reading R15; the same bytes cross the link per miss)
* mini-batch size (Fig. 10): 500, 1000, 2000, 4000
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r02"
cfg = sys.argv[2] if len(sys.argv) > 2 else "papers100m"
steps = sys.argv[3] if len(sys.argv) > 3 else "100"
points = [("buffer_frac", v, ["--buffer-frac", str(v)]) for v in (0.04, 0.10, 0.20, 0.40)]
points += [("feat_dim", v, ["--feat-dim", str(v)]) for v in (32, 64, 256)]
points += [("feat_dim", 512, ["--feat-dim", "512", "--table-rows", "40000000"])]
points += [("batch_size", v, ["--batch-size", str(v)]) for v in (500, 2000, 4000)]
rows = []
raw = os.path.join(ROOT, "profiles", f"{tag}_sweeps")
os.makedirs(raw, exist_ok=True)
for name, v, extra in points:
    out = os.path.join(raw, f"{cfg}_{name}_{v}.json")
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", cfg, "--steps", steps, "--warmup", "8",
           "--no-cpu-baseline", "--no-e2e", "--parity-batches", "2", "--out", out] + extra
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1500)
    try:
        d = json.load(open(out))
    except Exception:  # noqa: BLE001
        print(name, v, "failed", r.stderr[-2000:])
        continue
    pb = d["per_batch"]
    par = d["parity"]
    rows.append((name, v, d["value"], d["roofline"]["bound"], d["roofline"]["achieved"], d["roofline"]["frac"],
                 pb["hit_rate"], pb["n_nodes"], pb["misses"], par["first"]["batches"],
                 par["steady_state"]["batches"] if par["steady_state"] else 0, par["bit_exact"],
                 d["config"]["host_table_rows"]))
    print(rows[-1], flush=True)
lines = [f"# f3 sweeps on the built path — {cfg} ({tag})", "",
         f"One bench.py process per point ({steps} timed steps after pre-warm, 1 B200).  The paper's",
         "figures report end-to-end epoch time with training (P:183-212); here the same knobs are",
         "swept on the sample+extract path.  `parity`: first batches checked in full + the oracle",
         "replay of the whole schedule (per-batch sizes, hits/misses, final buffer state).  Raw JSON",
         f"lines: `profiles/{tag}_sweeps/`.", "",
         "| knob | value | batches/s | bound | achieved GB/s | frac | hit rate | nodes/batch | misses/batch | "
         "first-batch parity | replayed batches | bit-exact | host table rows |",
         "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
for r in rows:
    lines.append("| " + " | ".join(str(round(x, 4)) if isinstance(x, float) else str(x) for x in r) + " |")
open(os.path.join(ROOT, "profiles", f"{tag}_sweeps_{cfg}.md"), "w").write("\n".join(lines) + "\n")
