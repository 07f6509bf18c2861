"""Multi-GPU host logic on CPU: world-size-2 gloo process groups (no GPU needed).

Covers the data-parallel sharding of §8(e) ("segments", P:142 shared host data):
contiguous, disjoint, complete batch segments; per-rank schedules with epoch wrap; the
/dev/shm host table created by rank 0 and mapped by every rank; max/sum over ranks.
"""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, shm_dir, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_jiangj024_b200 import multigpu as M
        out = {}
        out["seg"] = list(M.segment(1209, rank, world))
        out["sched"] = M.batch_schedule(10, rank, world, 12)
        t = M.HostTable(1000, 64, "test", rank, world, shm_dir=shm_dir)
        if rank == 0:
            t.array[:] = (np.arange(1000 * 64) % 251).astype(np.uint8).reshape(1000, 64)
        M.barrier()
        out["table_sum"] = int(t.array.astype(np.int64).sum())
        out["table_row7"] = t.array[7].tolist()
        out["max"] = M.max_over_ranks(float(rank * 10 + 1))
        out["sum"] = M.sum_over_ranks(float(rank + 1))
        # f4 data parallelism: each rank's oracle gradients on its own batch, summed
        # by the same all-reduce helper the GPU path uses, scaled by 1/world = the mean
        from paper_conf_icpp_jiangj024_b200 import train as T
        from oracle import sage as S
        sys.path.insert(0, os.path.join(ROOT, "tests"))
        from test_oracle_sage import small_problem
        mine = small_problem(B=5 + rank, seed=3 + rank)
        loss, cache = S.forward(mine[0], mine[1], mine[2], mine[3])
        flat = torch.from_numpy(T.flatten_params(S.backward(mine[0], cache, mine[3])))
        scale = T.allreduce_flat(flat)
        out["ddp_scale"] = scale
        out["ddp_mean"] = (flat * scale).numpy()
        M.barrier()
        t.close(unlink=True)
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


@pytest.fixture(scope="module")
def results():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    with tempfile.TemporaryDirectory() as d:
        port = _free_port()
        procs = [ctx.Process(target=_worker, args=(r, world, port, d, q)) for r in range(world)]
        for p in procs:
            p.start()
        res = dict(q.get(timeout=120) for _ in range(world))
        for p in procs:
            p.join(timeout=60)
            assert p.exitcode == 0
        assert not os.listdir(d)        # rank 0 unlinked the shared table
    return res


def test_segments_disjoint_and_complete(results):
    a, b = results[0]["seg"], results[1]["seg"]
    assert a == list(range(0, 604)) and b == list(range(604, 1209))
    assert sorted(a + b) == list(range(1209))


def test_schedule_wraps_with_epochs(results):
    s0, s1 = results[0]["sched"], results[1]["sched"]
    assert s0[:5] == [(b, 0) for b in range(5)] and s0[5:10] == [(b, 1) for b in range(5)]
    assert s1[:5] == [(b, 0) for b in range(5, 10)]
    # the Philox batch key epoch * num_batches + b is distinct across ranks and epochs
    keys = [ep * 10 + b for b, ep in s0 + s1]
    assert len(set(keys)) == len(keys)


def test_shared_host_table_visible_to_all_ranks(results):
    expect = (np.arange(1000 * 64) % 251).astype(np.int64)
    assert results[0]["table_sum"] == results[1]["table_sum"] == int(expect.sum())
    assert results[1]["table_row7"] == expect.reshape(1000, 64)[7].tolist()


def test_ddp_gradient_mean(results):
    """The all-reduced flat gradient equals the mean of the per-rank oracle gradients."""
    from oracle import sage as S
    from paper_conf_icpp_jiangj024_b200 import train as T
    import sys
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    from test_oracle_sage import small_problem
    per = []
    for rank in range(2):
        p, f, bl, lab = small_problem(B=5 + rank, seed=3 + rank)
        _, cache = S.forward(p, f, bl, lab)
        per.append(T.flatten_params(S.backward(p, cache, lab)))
    want = (per[0] + per[1]) / 2
    for rank in range(2):
        assert results[rank]["ddp_scale"] == 0.5
        assert np.allclose(results[rank]["ddp_mean"], want, rtol=1e-12, atol=1e-15)


def test_max_and_sum_over_ranks(results):
    assert results[0]["max"] == results[1]["max"] == 11.0
    assert results[0]["sum"] == results[1]["sum"] == 3.0


def test_single_process_fallbacks():
    from paper_conf_icpp_jiangj024_b200 import multigpu as M
    assert M.max_over_ranks(3.5) == 3.5 and M.sum_over_ranks(2.0) == 2.0
    assert list(M.segment(7, 0, 1)) == list(range(7))
    assert M.batch_schedule(3, 0, 1, 7) == [(0, 0), (1, 0), (2, 0), (0, 1), (1, 1), (2, 1), (0, 2)]
    assert M.batch_schedule(1, 1, 4, 3) == []       # more ranks than batches: an empty segment


def test_numa_helpers():
    """NUMA placement (bench.py, world > 1): node-list parsing, an interleave policy call that
    never raises (False on single-node hosts), and the per-rank socket binding, which is a
    no-op (reported, not raised) where the GPU's PCIe locality is unknown or the host has one
    node."""
    from synth import host as H
    assert H.parse_cpulist("0-1,3\n") == [0, 1, 3]
    assert H.parse_cpulist("0") == [0]
    nodes = H.numa_nodes()
    assert all(isinstance(n, int) for n in nodes)
    ok = H.set_interleave(True)
    assert ok == (len(nodes) >= 2) or not ok
    H.set_interleave(False)
    before = os.sched_getaffinity(0)
    rep = H.bind_to_gpu_socket(0)
    assert rep["cpus"] >= 1 and (rep["bound"] or os.sched_getaffinity(0) == before)
    os.sched_setaffinity(0, before)


def test_shared_array_refuses_a_short_shm(monkeypatch, tmp_path):
    """Rank 0 checks the shared-memory filesystem's free space before creating the table and
    fails with a clear message (instead of a SIGBUS mid-fill)."""
    from synth import host as H
    monkeypatch.setattr(H, "shm_free_bytes", lambda path: 1000)
    with pytest.raises(RuntimeError, match="GiB free"):
        H.HostTable(100, 64, "short", rank=0, world=2, shm_dir=str(tmp_path))
    assert not os.listdir(tmp_path)
    monkeypatch.setattr(H, "shm_free_bytes", lambda path: 1 << 40)
    t = H.HostTable(100, 64, "ok", rank=0, world=2, shm_dir=str(tmp_path))
    t.array[:] = 7
    assert int(t.array.sum()) == 7 * 6400
    t.close()
    assert not os.listdir(tmp_path)


def test_reference_arm_under_torchrun_world2():
    """bench.py --impl reference launched like the driver's N>1 runs (torchrun, 2 ranks,
    127.0.0.1): rank 0 alone runs the oracle and prints one JSON line, the other rank exits 0
    without work (CPU here: gloo).  Rank 0's single-rank workload must not enter collectives."""
    import json
    import subprocess
    import sys
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="", OMP_NUM_THREADS="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "tiny", "--gpus", "2",
           "--steps", "3", "--warmup", "1"]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [json.loads(x) for x in p.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1, p.stdout
    rec = lines[0]
    assert rec["impl"] == "reference" and rec["n_gpus"] == 2 and rec["value"] > 0
    assert rec["e2e"]["h2d_bytes_per_step"] == 0 and rec["cpu_baseline"]["kind"] == "oracle"
    # reference-arm hygiene: the oracle only, never the product library
    assert rec["native_libs_loaded"] == ["oracle/libgd_oracle.so"], rec["native_libs_loaded"]
    assert rec["cpu_baseline"]["cores"] == len(os.sched_getaffinity(0))
    assert rec["config"]["workload"] == "tiny" and rec["config"]["release_lag"] == 4
