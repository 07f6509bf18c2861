"""bench.py end to end on the GPU (small workloads): the JSON contract, first-batch parity and
the steady-state oracle replay (whole schedule: per-batch sizes and hits/misses, the last
batches' n_id / alias, the final buffer state), at 1 rank and at 2 ranks under torchrun on
the one GPU of the box (GD_BENCH_SAME_DEVICE=1, gloo: each rank its own segment, buffer and
replay; the multi-GPU host logic of SURVEY 8(e))."""
import json
import os
import socket
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(cmd, env=None, timeout=900):
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    p = subprocess.run(cmd, cwd=ROOT, env=dict(os.environ, **(env or {})), capture_output=True, text=True,
                       timeout=timeout)
    assert p.returncode == 0, p.stderr[-4000:]
    lines = [json.loads(x) for x in p.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1, p.stdout[-2000:]
    return lines[0], p.stderr


def _check_replay(rep, steps):
    assert rep["bit_exact"], rep
    assert rep["sizes_equal"] and rep["hits_misses_equal"] and rep["tail_equal"] and rep["final_state_equal"], rep
    assert rep["batches"] >= 2 * steps and rep["misses"] > 0


# tiny with the buffer below the touched set (S = Q * M_b = 9216 of 10k nodes): eviction every batch
ARGS = ["--config", "tiny", "--buffer-frac", "0.3", "--steps", "24", "--warmup", "3", "--cpu-seconds", "2"]


def test_bench_single_rank_parity_and_replay():
    rec, err = _run([sys.executable, "bench.py", *ARGS])
    assert rec["n_gpus"] == 1 and rec["value"] > 0 and rec["e2e"]["value"] > 0
    assert rec["parity"]["bit_exact"], rec["parity"]
    first = rec["parity"]["first"]
    assert first["bit_exact"] and first["batches"] >= 8
    _check_replay(rec["parity"]["steady_state"], 24)
    assert rec["rows_check"]["ok"] and rec["rows_check"]["n_id_vs_oracle"]
    cb = rec["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == len(os.sched_getaffinity(0)) and cb["value"] > 0
    assert cb["single_thread_full_oracle"]["cores"] == 1
    assert rec["miss_policy"] is not None and rec["miss_policy"]["misses_est"] > 0
    assert rec["roofline"]["peak"] > 0 and rec["gpu_launches"] > 0


def test_bench_two_ranks_same_gpu_per_rank_parity():
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_free_port()), "bench.py", "--gpus", "2", *ARGS]
    rec, err = _run(cmd, env={"GD_BENCH_SAME_DEVICE": "1"})
    assert rec["n_gpus"] == 2 and rec["value"] > 0
    par = rec["parity"]
    assert par["bit_exact"], par
    assert len(par["first"]) == 2 and len(par["steady_state"]) == 2       # one entry per rank
    for f in par["first"]:
        assert f["bit_exact"] and f["batches"] >= 4
    for r in par["steady_state"]:
        _check_replay(r, 24)
    assert rec["rows_check"]["ok"]
    peaks = rec["host_link_peaks_GBps"]
    assert peaks["alone"] > 0 and peaks["concurrent"] > 0
    assert "rank0" in rec["roofline_miss"]
    leg = rec["peer_leg"]                        # f2 leg: both ranks' buffers attached as peers
    assert leg is not None and leg["value"] > 0 and leg["probed_misses"] > 0 and leg["served_rows"] >= 0
