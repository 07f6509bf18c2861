"""f3: the paper's sweeps on the built path, one bench.py process per
point, results to profiles/<tag>_sweeps.md.

    python tools/sweeps.py <tag> [config]

* buffer size (Fig. 12): buffer_frac in {0.04, 0.10, 0.20, 0.40} of N
* feature dimension (Fig. 8): 32, 64, 128, 256 fp32 (512 -> a 227 GB host table,
  above this pool's 196 GB of host RAM)
* mini-batch size (Fig. 10): 500, 1000, 2000, 4000
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
cfg = sys.argv[2] if len(sys.argv) > 2 else "papers100m"
points = [("buffer_frac", v, ["--buffer-frac", str(v)]) for v in (0.04, 0.10, 0.20, 0.40)]
points += [("feat_dim", v, ["--feat-dim", str(v)]) for v in (32, 64, 256)]
points += [("batch_size", v, ["--batch-size", str(v)]) for v in (500, 2000, 4000)]
rows = []
os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
for name, v, extra in points:
    out = os.path.join(ROOT, "gpurun_out", f"sweep_{cfg}_{name}_{v}.json")
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", cfg, "--steps", "100", "--warmup", "8",
           "--no-cpu-baseline", "--no-e2e", "--parity-batches", "0", "--out", out] + extra
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1200)
    try:
        d = json.load(open(out))
    except Exception:  # noqa: BLE001
        print(name, v, "failed", r.stderr[-2000:])
        continue
    pb = d["per_batch"]
    rows.append((name, v, d["value"], d["roofline"]["bound"], d["roofline"]["achieved"], d["roofline"]["frac"],
                 pb["hit_rate"], pb["n_nodes"], pb["misses"]))
    print(rows[-1], flush=True)
lines = [f"# f3 sweeps on the built path — {cfg} ({tag})", "",
         "One bench.py process per point (100 timed steps after pre-warm, 1 B200).  The paper's",
         "figures report end-to-end epoch time with training (P:183-212); here the same knobs are",
         "swept on the sample+extract path.", "",
         "| knob | value | batches/s | bound | achieved GB/s | frac | hit rate | nodes/batch | misses/batch |",
         "|---|---|---|---|---|---|---|---|---|"]
for r in rows:
    lines.append("| " + " | ".join(str(round(x, 4)) if isinstance(x, float) else str(x) for x in r) + " |")
open(os.path.join(ROOT, "profiles", f"{tag}_sweeps_{cfg}.md"), "w").write("\n".join(lines) + "\n")
