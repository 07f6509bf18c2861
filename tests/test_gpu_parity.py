"""GPU parity: the sm_100a path (through the C ABI) against the CPU oracle, bit-exact.

Sampling (n_id, rowptr, col, eid, sizes) and extraction (out bytes, alias, hits/misses,
and the whole buffer state: map, reverse, standby order) must be identical element by
element.  Sizes span several tiles with ragged tails; edge cases cover empty inputs,
degree-0 rows, fanout -1 / 0 / > 32, duplicate and out-of-range ids, exhausted capacity.
"""
import json
import os

import numpy as np
import pytest
import torch

import synth
from oracle import oracle as O

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def gd():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_icpp_jiangj024_b200 as gd
    return gd


def make_graph(N, E, seed=1):
    indptr, indices = synth.chung_lu_csr(N, E, seed=seed)
    return indptr, indices


def compare_sample(res_gpu, res_o, K):
    h = res_gpu.to_host()
    assert np.array_equal(h["sizes"], res_o.sizes), (h["sizes"], res_o.sizes)
    assert np.array_equal(h["n_id"], res_o.n_id)
    for k in range(K):
        assert np.array_equal(h["rowptr"][k], res_o.rowptr[k]), f"rowptr hop {k+1}"
        assert np.array_equal(h["col"][k], res_o.col[k]), f"col hop {k+1}"
        if h["eid"][k] is not None:
            assert np.array_equal(h["eid"][k], res_o.eid[k]), f"eid hop {k+1}"


@pytest.fixture(scope="module")
def tiny(gd):
    cfg = synth.CONFIGS["tiny"]
    indptr, indices = make_graph(cfg.num_nodes, cfg.num_edges)
    g = gd.Graph(indptr, indices, device=0)
    order = synth.epoch_order(synth.train_nodes(cfg.num_nodes, cfg.train_frac))
    return cfg, g, indptr.numpy(), indices.numpy(), order


@pytest.mark.parametrize("fanouts", [(5, 5), (15, 10, 5), (25, 15), (10, 10, 10), (-1, 3), (0, 4), (40, 2),
                                     (100,), (33, 1), (1, 1, 1, 1, 1, 1, 1, 1), (32, 17, 16, 2)])
@pytest.mark.parametrize("padded", [True, False])
def test_sample_parity_tiny(tiny, gd, fanouts, padded):
    cfg, g, indptr, indices, order = tiny
    g.sampler(padded)
    for b in range(6):
        seeds = synth.batch_seeds(order, cfg.batch_size, b)
        res = g.sample(seeds.cuda(), fanouts, synth.RNG_SEED, b, with_eid=True)
        torch.cuda.synchronize()
        ref = O.sample(indptr, indices, seeds.numpy(), list(fanouts), synth.RNG_SEED, b)
        compare_sample(res, ref, len(fanouts))
    g.sampler(True)
    assert g.check() == 0


def test_sample_parity_host_seeds_and_no_eid(tiny, gd):
    cfg, g, indptr, indices, order = tiny
    seeds = synth.batch_seeds(order, cfg.batch_size, 3).pin_memory()
    res = g.sample(seeds, (5, 5), 77, 3)          # pinned host seeds (read through the mapping), no eid
    torch.cuda.synchronize()
    ref = O.sample(indptr, indices, seeds.numpy(), [5, 5], 77, 3)
    compare_sample(res, ref, 2)
    pageable = seeds.clone()                      # pageable host seeds: staged copy
    assert not pageable.is_pinned()
    res2 = g.sample(pageable, (5, 5), 77, 3)
    torch.cuda.synchronize()
    compare_sample(res2, ref, 2)


@pytest.mark.parametrize("padded", [True, False])
def test_sample_parity_multi_tile(gd, padded):
    """~200k nodes, (15,10,5) from 1024 seeds: hundreds of tiles per hop, ragged tails."""
    N, E = 200_000, 3_000_000
    indptr, indices = make_graph(N, E, seed=9)
    g = gd.Graph(indptr, indices)
    g.sampler(padded)
    order = synth.epoch_order(synth.train_nodes(N, 0.05))
    ip, ix = indptr.numpy(), indices.numpy()
    for b, B in [(0, 1024), (1, 1000), (2, 1), (3, 777)]:
        seeds = order[b * 1024: b * 1024 + B]
        res = g.sample(seeds.cuda(), (15, 10, 5), 3, b, with_eid=True)
        torch.cuda.synchronize()
        compare_sample(res, O.sample(ip, ix, seeds.numpy(), [15, 10, 5], 3, b), 3)


@pytest.mark.parametrize("padded", [True, False])
def test_sample_edge_cases(gd, padded):
    # isolated nodes, self loops, multi-edges; empty seed list
    rows = [[1, 2], [1, 0, 4], [0, 0, 4], [], [5], [2], [], [3, 3, 3, 3]]
    indptr = torch.tensor(np.cumsum([0] + [len(r) for r in rows]), dtype=torch.int64)
    indices = torch.tensor([u for r in rows for u in r], dtype=torch.int32)
    g = gd.Graph(indptr, indices)
    g.sampler(padded)
    for seeds, fan in [([3], [2, 2]), ([6, 3], [5]), ([0, 7, 5], [1, 2, 3]), ([7], [-1, -1, -1]), ([], [2, 2])]:
        s = torch.tensor(seeds, dtype=torch.int32)
        res = g.sample(s.cuda() if len(seeds) else s.cuda(), fan, 1, 0, with_eid=True)
        torch.cuda.synchronize()
        compare_sample(res, O.sample(indptr.numpy(), indices.numpy(), s.numpy(), fan, 1, 0), len(fan))
    assert g.check() == 0


def test_sample_duplicate_and_bad_seed_flagged(gd):
    indptr, indices = make_graph(1000, 5000)
    g = gd.Graph(indptr, indices)
    g.sample(torch.tensor([1, 2, 1], dtype=torch.int32).cuda(), [3], 1, 0)
    with pytest.raises(gd.GdError) as e:
        g.check()
    assert e.value.status == 5
    g2 = gd.Graph(indptr, indices)
    g2.sample(torch.tensor([5, 1000], dtype=torch.int32).cuda(), [3], 1, 0)
    with pytest.raises(gd.GdError):
        g2.check()


def test_graph_create_rejects_bad_csr(gd):
    with pytest.raises(gd.GdError):
        gd.Graph(torch.tensor([0, 2, 1], dtype=torch.int64), torch.tensor([0, 1], dtype=torch.int32))
    with pytest.raises(gd.GdError):
        gd.Graph(torch.tensor([0, 1, 2], dtype=torch.int64), torch.tensor([0, 7], dtype=torch.int32))


# ----------------------------------------------------------------------- extraction


def table_np(N, R, seed=4):
    return synth.feature_rows(0, N, R, seed).numpy()


def compare_state(buf, ob):
    a, b = buf.snapshot(), ob.state()
    for k in ("slot", "rc", "valid", "reverse", "standby"):
        assert np.array_equal(a[k], b[k]), k


def run_schedule(gd, g, ip, ix, feat, S, Q, seeds_list, fanouts, preload=False, check_state_every=1, config=None,
                 num_nodes=None, stage_mode=None):
    P, R = feat.shape
    N = num_nodes or P
    nb, _ = O.sample_bounds(max(len(s) for s in seeds_list), fanouts, N, int(ip[-1]))
    n_max = nb[-1]
    buf = gd.FeatureBuffer(torch.from_numpy(feat), S, Q, n_max, preload=preload, num_nodes=N)
    if stage_mode is not None:
        buf.stage_mode(stage_mode)
    if config is not None:
        buf.config(*config)
    ob = O.Buffer(feat, S, preload=preload, num_nodes=N)
    pending = []
    for b, seeds in enumerate(seeds_list):
        res = g.sample(torch.as_tensor(seeds).cuda(), fanouts, 3, b)
        alias = torch.empty(n_max, dtype=torch.int32, device="cuda")
        stats = torch.zeros(4, dtype=torch.int64, device="cuda")
        out, _, done = buf.extract(res.n_id, res.num_nodes_dev, res.max_nodes, alias=alias, stats=stats)
        done.synchronize()
        n_id = res.to_host()["n_id"]
        o_out, o_alias, o_stats = ob.extract(n_id)
        n = len(n_id)
        assert tuple(stats.cpu().tolist()[:2]) == o_stats
        assert np.array_equal(alias[:n].cpu().numpy(), o_alias)
        assert np.array_equal(out[:n].cpu().numpy(), o_out)
        assert np.array_equal(o_out, feat[n_id % P])              # closed form
        pending.append((res, n_id))
        if len(pending) == Q:
            r0, n0 = pending.pop(0)
            buf.release(r0.n_id, r0.num_nodes_dev, r0.max_nodes)
            ob.release(n0)
        if check_state_every and b % check_state_every == 0:
            compare_state(buf, ob)
    compare_state(buf, ob)
    assert buf.check() == 0
    return buf, ob


def test_extract_parity_tiny_preload(tiny, gd):
    cfg, g, ip, ix, order = tiny
    feat = table_np(cfg.num_nodes, cfg.row_bytes)
    seeds = [synth.batch_seeds(order, cfg.batch_size, b).numpy() for b in range(12)]
    run_schedule(gd, g, ip, ix, feat, cfg.num_nodes, 4, seeds, list(cfg.fanouts), preload=True)


@pytest.mark.parametrize("Q", [1, 2, 4])
def test_extract_parity_tiny_evict(tiny, gd, Q):
    """tiny-evict: S = Q * M_b, the minimum legal capacity: heavy eviction."""
    cfg, g, ip, ix, order = tiny
    feat = table_np(cfg.num_nodes, cfg.row_bytes)
    nb, _ = O.sample_bounds(cfg.batch_size, list(cfg.fanouts), cfg.num_nodes, cfg.num_edges)
    S = Q * nb[-1]
    seeds = [synth.batch_seeds(order, cfg.batch_size, b).numpy() for b in range(30)]
    run_schedule(gd, g, ip, ix, feat, S, Q, seeds, list(cfg.fanouts))


@pytest.mark.parametrize("own_stream,row_bytes,chunk_kb", [(False, None, None), (True, None, None), (True, 1024, "16"),
                                                        (False, 1536, "24")])
def test_release_on_its_own_stream_matches_oracle(tiny, gd, own_stream, row_bytes, chunk_kb, monkeypatch):
    """bench.py's schedule: release(j - Q) on a second stream, ordered after extract(j)'s
    bookkeeping and before extract(j + 1)'s by events, overlapping sample(j + 1); no host
    sync until the end.  Outputs and the final buffer state equal the sequential oracle's.
    The small-chunk cases give the staged copy-engine path many chunks per batch, so the
    host-callback argument ring (1024 slots) wraps during the run."""
    if chunk_kb is not None:
        monkeypatch.setenv("GD_STAGE_CHUNK_KB", chunk_kb)
    cfg, g, ip, ix, order = tiny
    feat = table_np(cfg.num_nodes, row_bytes or cfg.row_bytes)
    fan = list(cfg.fanouts)
    Q = 4
    nb, _ = O.sample_bounds(cfg.batch_size, fan, cfg.num_nodes, cfg.num_edges)
    n_max = nb[-1]
    buf = gd.FeatureBuffer(torch.from_numpy(feat), Q * n_max, Q, n_max)
    main = torch.cuda.current_stream()
    rel = torch.cuda.Stream() if own_stream else main
    ev_bk, ev_rel = torch.cuda.Event(), torch.cuda.Event()
    nbat = 24
    seeds = [synth.batch_seeds(order, cfg.batch_size, b).cuda() for b in range(nbat)]
    res, outs, aliases, stats, pending, rel_live = [], [], [], [], [], False
    for b in range(nbat):
        r = g.sample(seeds[b], fan, 3, b, stream=main)
        if rel_live:
            main.wait_event(ev_rel)
        a = torch.empty(n_max, dtype=torch.int32, device="cuda")
        st = torch.zeros(4, dtype=torch.int64, device="cuda")
        out, _, done = buf.extract(r.n_id, r.num_nodes_dev, r.max_nodes, alias=a, stats=st, stream=main)
        res.append(r), outs.append(out), aliases.append(a), stats.append(st)
        pending.append(r)
        if len(pending) == Q:
            r0 = pending.pop(0)
            ev_bk.record(main)
            rel.wait_event(ev_bk)
            buf.release(r0.n_id, r0.num_nodes_dev, r0.max_nodes, stream=rel)
            ev_rel.record(rel)
            rel_live = True
    torch.cuda.synchronize()
    ob = O.Buffer(feat, Q * n_max)
    opend = []
    for b in range(nbat):
        n_id = res[b].to_host()["n_id"]
        o_out, o_alias, o_stats = ob.extract(n_id)
        n = len(n_id)
        assert tuple(stats[b].cpu().tolist()[:2]) == o_stats, b
        assert np.array_equal(aliases[b][:n].cpu().numpy(), o_alias), b
        assert np.array_equal(outs[b][:n].cpu().numpy(), o_out), b
        opend.append(n_id)
        if len(opend) == Q:
            ob.release(opend.pop(0))
    compare_state(buf, ob)
    assert buf.check() == 0


def test_share_tuner_runs_and_stays_exact(gd, monkeypatch):
    """GD_SHARE_TUNER=1: the hill-climbing share tuner measures windows and moves the zero-copy
    share (in [0, 0.4]) while the outputs and the buffer state stay the oracle's."""
    monkeypatch.setenv("GD_SHARE_TUNER", "1")
    N, E, B, fan, Q, nbat = 200_000, 2_000_000, 1000, [10, 5], 4, 60
    indptr, indices = make_graph(N, E, seed=23)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, 512)
    order = synth.epoch_order(synth.train_nodes(N, 0.5))
    nb, _ = O.sample_bounds(B, fan, N, E)
    n_max = nb[-1]
    buf = gd.FeatureBuffer(torch.from_numpy(feat), Q * n_max, Q, n_max)
    buf.config(4, -1.0)
    ob = O.Buffer(feat, Q * n_max)
    pend, opend = [], []
    for b in range(nbat):
        r = g.sample(order[(b % 100) * B:((b % 100) + 1) * B].cuda(), fan, 3, b)
        st = torch.zeros(4, dtype=torch.int64, device="cuda")
        out, _, done = buf.extract(r.n_id, r.num_nodes_dev, r.max_nodes, stats=st)
        done.synchronize()                      # completed batches let the tuner measure windows
        n_id = r.to_host()["n_id"]
        o_out, _, o_st = ob.extract(n_id)
        assert tuple(st.cpu().tolist()[:2]) == o_st and np.array_equal(out[:len(n_id)].cpu().numpy(), o_out), b
        pend.append(r), opend.append(n_id)
        if len(pend) == Q:
            r0 = pend.pop(0)
            buf.release(r0.n_id, r0.num_nodes_dev, r0.max_nodes)
            ob.release(opend.pop(0))
    pol = buf.policy_read()
    assert pol["tuner_on"] and pol["tuner_windows"] >= 2 and 0.0 <= pol["zero_copy_share"] <= 0.4, pol
    compare_state(buf, ob)
    assert buf.check() == 0


def test_adaptive_split_stages_without_host_sync(gd):
    """a caller that never synchronises (the host may run many batches ahead of the
    device) still gets a miss-count estimate for the copy-engine staging size (each batch's
    count is published with its epoch into mapped host memory), so the staged share starts
    after warm-up instead of every miss going zero-copy; all 40 batches stay bit-exact."""
    N, E, B, fan, Q, nbat = 200_000, 2_000_000, 1000, [10, 5], 4, 40
    indptr, indices = make_graph(N, E, seed=21)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, 512)
    order = synth.epoch_order(synth.train_nodes(N, 0.5))
    nb, _ = O.sample_bounds(B, fan, N, E)
    n_max = nb[-1]
    buf = gd.FeatureBuffer(torch.from_numpy(feat), Q * n_max, Q, n_max)
    buf.config(4, -1.0)
    seeds = [order[b * B:(b + 1) * B].cuda() for b in range(nbat)]
    stats = torch.zeros((nbat, 4), dtype=torch.int64, device="cuda")
    res, outs, aliases, pending = [], [], [], []
    for b in range(nbat):
        r = g.sample(seeds[b], fan, 3, b)
        a = torch.empty(n_max, dtype=torch.int32, device="cuda")
        out, _, _ = buf.extract(r.n_id, r.num_nodes_dev, r.max_nodes, alias=a, stats=stats[b])
        res.append(r), outs.append(out), aliases.append(a)
        pending.append(r)
        if len(pending) == Q:
            r0 = pending.pop(0)
            buf.release(r0.n_id, r0.num_nodes_dev, r0.max_nodes)
    torch.cuda.synchronize()
    st = stats.cpu()
    assert int(st[:, 1].sum()) > 0
    assert int(st[10:, 3].sum()) > 0, st[:, 2:].tolist()        # the staged share ran
    pol = buf.policy_read()
    assert pol["misses_est"] > 0 and 0.05 <= pol["zero_copy_share"] <= 0.15 and not pol["tuner_on"], pol
    ob = O.Buffer(feat, Q * n_max)
    opend = []
    for b in range(nbat):
        n_id = res[b].to_host()["n_id"]
        o_out, o_alias, o_stats = ob.extract(n_id)
        n = len(n_id)
        assert tuple(st[b].tolist()[:2]) == o_stats, b
        assert int(st[b][2] + st[b][3]) == o_stats[1], b               # the split covers every miss
        assert np.array_equal(aliases[b][:n].cpu().numpy(), o_alias), b
        assert np.array_equal(outs[b][:n].cpu().numpy(), o_out), b
        opend.append(n_id)
        if len(opend) == Q:
            ob.release(opend.pop(0))
    compare_state(buf, ob)
    assert buf.check() == 0


# phase 2 of the staged share: SM pull of the pinned slot, or copy engine with the
# default 8 MB chunk ring, with 64 KB chunks (many chunks per batch, ring reuse), or
# with one chunk per batch (GD_STAGE_CHUNK_KB=0)
STAGE_MODES = {"pull": (False, None), "ce": (True, None), "ce-64k": (True, "64"), "ce-whole": (True, "0")}


@pytest.mark.parametrize("mode", list(STAGE_MODES))
@pytest.mark.parametrize("config", [(0, -1.0), (4, 0.0), (4, 1.0), (3, 0.3), (8, -1.0), (1, 0.9)])
def test_extract_parity_miss_paths(gd, config, mode, monkeypatch):
    """The miss stream split between zero-copy and the staged (host gather + copy engine
    or SM pull) path: every split gives the same bytes, alias and state."""
    N, E = 60_000, 600_000
    indptr, indices = make_graph(N, E, seed=8)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, 512)
    order = synth.epoch_order(synth.train_nodes(N, 0.3))
    seeds = [order[b * 500:(b + 1) * 500].numpy() for b in range(16)]
    nb, _ = O.sample_bounds(500, [10, 5], N, E)
    copy_engine, chunk_kb = STAGE_MODES[mode]
    if chunk_kb is not None:
        monkeypatch.setenv("GD_STAGE_CHUNK_KB", chunk_kb)
    run_schedule(gd, g, indptr.numpy(), indices.numpy(), feat, 3 * nb[-1], 3, seeds, [10, 5],
                 check_state_every=4, config=config, stage_mode=copy_engine)


@pytest.mark.parametrize("preload", [False, True])
def test_extract_parity_bounded_table(gd, preload):
    """mag240m-style bounded host table (node v -> row v mod P), zero-copy + staged paths."""
    N, E, P = 30_000, 240_000, 7_001
    indptr, indices = make_graph(N, E, seed=13)
    g = gd.Graph(indptr, indices)
    feat = table_np(P, 1536)
    order = synth.epoch_order(synth.train_nodes(N, 0.3))
    seeds = [order[b * 200:(b + 1) * 200].numpy() for b in range(10)]
    nb, _ = O.sample_bounds(200, [25, 15], N, E)
    S = N if preload else 2 * nb[-1]
    run_schedule(gd, g, indptr.numpy(), indices.numpy(), feat, S, 2, seeds, [25, 15], preload=preload,
                 check_state_every=3, num_nodes=N)


@pytest.mark.parametrize("mode", list(STAGE_MODES))
@pytest.mark.parametrize("R", [400, 12, 1536])
def test_extract_parity_row_sizes(gd, R, mode, monkeypatch):
    """Row widths: 16-byte vector path (400 = products, 1536 = mag240m fp16) and the 4-byte path."""
    N, E = 20_000, 150_000
    indptr, indices = make_graph(N, E, seed=5)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, R if R % 8 == 0 else 16)[:, :R].copy()
    order = synth.epoch_order(synth.train_nodes(N, 0.2))
    seeds = [order[b * 300:(b + 1) * 300].numpy() for b in range(10)]
    nb, _ = O.sample_bounds(300, [10, 5], N, E)
    copy_engine, chunk_kb = STAGE_MODES[mode]
    if chunk_kb is not None:
        monkeypatch.setenv("GD_STAGE_CHUNK_KB", chunk_kb)
    run_schedule(gd, g, indptr.numpy(), indices.numpy(), feat, 2 * nb[-1] + 17, 2, seeds, [10, 5], check_state_every=3,
                 config=(4, 0.3), stage_mode=copy_engine)


@pytest.mark.parametrize("variant", ["tma", "static", "low-priority", "u8-2bps", "zc-after-gather"])
@pytest.mark.parametrize("R", [400, 512, 1536, 2048, 12])
def test_hit_gather_variants(gd, R, variant, monkeypatch):
    """a8 variants (selected at buffer init): the TMA gather4 kernel (GD_GATHER_TMA=1), the
    warp-per-row kernel with a static row partition (GD_GATHER_DYNAMIC=0), the gather
    stream at default priority, 8 rows in flight per warp on 2 blocks per SM (GD_GATHER_U=8,
    GD_GATHER_BPS=2), and the zero-copy kernel ordered after the hit gather
    (GD_ZC_AFTER_GATHER=1): the same bytes, alias and state as the oracle (R = 12: the
    4-byte kernel, whichever variant is asked for)."""
    envs = {"tma": [("GD_GATHER_TMA", "1")], "static": [("GD_GATHER_DYNAMIC", "0")],
            "low-priority": [("GD_GATHER_PRIORITY", "0")],
            "u8-2bps": [("GD_GATHER_U", "8"), ("GD_GATHER_BPS", "2")],
            "zc-after-gather": [("GD_ZC_AFTER_GATHER", "1")]}[variant]
    for k, v in envs:
        monkeypatch.setenv(k, v)
    N, E = 20_000, 150_000
    indptr, indices = make_graph(N, E, seed=17)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, R if R % 8 == 0 else 16)[:, :R].copy()
    order = synth.epoch_order(synth.train_nodes(N, 0.2))
    seeds = [order[b * 300:(b + 1) * 300].numpy() for b in range(8)]
    nb, _ = O.sample_bounds(300, [10, 5], N, E)
    run_schedule(gd, g, indptr.numpy(), indices.numpy(), feat, 2 * nb[-1] + 5, 2, seeds, [10, 5], check_state_every=4,
                 config=(4, 0.3))


def test_extract_ring_compaction(gd):
    """Many batches with a small capacity and lag: the standby ring compacts repeatedly."""
    N, E = 3000, 30000
    indptr, indices = make_graph(N, E, seed=6)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, 32)
    order = synth.epoch_order(synth.train_nodes(N, 0.5))
    seeds = [order[(b * 40) % 1400:(b * 40) % 1400 + 40].numpy() for b in range(80)]
    nb, _ = O.sample_bounds(40, [4, 4], N, E)
    run_schedule(gd, g, indptr.numpy(), indices.numpy(), feat, 3 * nb[-1], 3, seeds, [4, 4], check_state_every=7)


def test_figure6_on_gpu(gd):
    gdict = json.load(open(os.path.join(HERE, "golden", "fig6.json")))
    N, S = gdict["num_nodes"], gdict["num_slots"]
    feat = table_np(N, 16)
    buf = gd.FeatureBuffer(torch.from_numpy(feat), S, 1, 5)     # S=6 >= min(N, 1 x 5)
    buf.set_state(gdict["map_slot"], gdict["map_rc"], gdict["map_valid"], gdict["reverse"], gdict["standby"])
    ids = torch.tensor(gdict["batch"], dtype=torch.int32, device="cuda")
    n = torch.tensor([len(gdict["batch"])], dtype=torch.int64, device="cuda")
    alias = torch.empty(5, dtype=torch.int32, device="cuda")
    stats = torch.zeros(4, dtype=torch.int64, device="cuda")
    out, _, done = buf.extract(ids, n, 5, alias=alias, stats=stats)
    done.synchronize()
    assert alias[:5].cpu().tolist() == gdict["expect_alias"]
    assert stats.cpu().tolist()[:2] == [gdict["expect_hits"], gdict["expect_misses"]]
    st = buf.snapshot()
    assert st["reverse"].tolist() == gdict["expect_reverse"]
    assert st["standby"].tolist() == gdict["expect_standby_after_extract"]
    for v in gdict["expect_invalidated"]:
        assert st["valid"][v] == 0 and st["slot"][v] == -1
    assert np.array_equal(out[:5].cpu().numpy(), feat[gdict["batch"]])
    rel = torch.tensor(gdict["release"], dtype=torch.int32, device="cuda")
    buf.release(rel, torch.tensor([1], dtype=torch.int64, device="cuda"), 5)
    assert buf.snapshot()["standby"].tolist() == gdict["expect_standby_after_release"]


def test_extract_capacity_and_errors(gd):
    feat = table_np(100, 16)
    with pytest.raises(gd.GdError) as e:
        gd.FeatureBuffer(torch.from_numpy(feat), 10, 2, 8)          # 10 < min(100, 2*8)
    assert e.value.status == 4
    buf = gd.FeatureBuffer(torch.from_numpy(feat), 16, 2, 8)
    ids = torch.arange(8, dtype=torch.int32, device="cuda")
    n = torch.tensor([8], dtype=torch.int64, device="cuda")
    buf.extract(ids, n, 8)
    buf.extract(ids + 8, n, 8)
    with pytest.raises(gd.GdError) as e:
        buf.extract(ids + 16, n, 8)                                   # third unreleased batch
    assert e.value.status == 4
    with pytest.raises(gd.GdError):
        buf.extract(ids, n, 9)                                        # n_max > max_nodes_per_batch
    buf.release(ids, n, 8)
    buf.release(ids, n, 8)                                            # refcount underflow
    with pytest.raises(gd.GdError) as e:
        buf.check()
    assert e.value.status == 5


def test_extract_empty_batch(gd):
    feat = table_np(50, 16)
    buf = gd.FeatureBuffer(torch.from_numpy(feat), 20, 2, 8)
    ids = torch.empty(8, dtype=torch.int32, device="cuda")
    n = torch.zeros(1, dtype=torch.int64, device="cuda")
    stats = torch.full((4,), -1, dtype=torch.int64, device="cuda")
    _, _, done = buf.extract(ids, n, 8, stats=stats)
    done.synchronize()
    assert stats.cpu().tolist() == [0, 0, 0, 0]
    buf.release(ids, n, 8)
    assert buf.check() == 0
    assert buf.snapshot()["standby"].tolist() == list(range(20))


# ----------------------------------------------------------------------- f1 pipeline


@pytest.mark.parametrize("samplers,reorder", [(1, False), (3, False), (3, True), (4, True)])
def test_pipeline_parity_in_extraction_order(gd, samplers, reorder):
    """SET pipeline with S concurrent sampler streams (own workspaces) and out-of-order
    extraction: the oracle replayed in the recorded extraction order gives the same
    alias, hit/miss counts and rows, and the same final buffer state."""
    from paper_conf_icpp_jiangj024_b200.pipeline import SETPipeline
    N, E, B, fan, Q = 40_000, 400_000, 300, [10, 5], 3
    indptr, indices = make_graph(N, E, seed=12)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, 64)
    nb, _ = O.sample_bounds(B, fan, N, E)
    S = Q * nb[-1]
    buf = gd.FeatureBuffer(torch.from_numpy(feat), S, Q, nb[-1])
    order = synth.epoch_order(synth.train_nodes(N, 0.3))
    seeds = [order[b * B:(b + 1) * B].cuda() for b in range(24)]
    bids = list(range(100, 124))
    rows = {}

    def consumer(k, out, alias, done):
        done.synchronize()
        rows[k] = (out.cpu().numpy().copy(), alias.cpu().numpy().copy())

    pipe = SETPipeline(g, buf, fan, B, 7, samplers=samplers, release_lag=Q, reorder=reorder)
    ext_order, stats = pipe.run(seeds, bids, consumer=consumer)
    torch.cuda.synchronize()
    assert sorted(ext_order) == list(range(24))
    ob = O.Buffer(feat, S)
    pend = []
    ip, ix = indptr.numpy(), indices.numpy()
    for k in ext_order:
        ref = O.sample(ip, ix, seeds[k].cpu().numpy(), fan, 7, bids[k])
        o_out, o_alias, o_st = ob.extract(ref.n_id)
        n = len(ref.n_id)
        out, alias = rows[k]
        assert tuple(stats[k].cpu().tolist()[:2]) == o_st
        assert np.array_equal(alias[:n], o_alias) and np.array_equal(out[:n], o_out)
        pend.append(ref.n_id)
        if len(pend) == Q:
            ob.release(pend.pop(0))
    while pend:
        ob.release(pend.pop(0))
    compare_state(buf, ob)
    assert buf.check() == 0 and g.check() == 0


def test_run_twice_bitwise_identical_and_gpu_count_independent(gd):
    """P8: the whole path run twice gives identical bytes; a batch's sample depends only on
    (rng_seed, global batch id), so two workspaces / streams / orders agree (any GPU count)."""
    N, E = 50_000, 500_000
    indptr, indices = make_graph(N, E, seed=21)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, 512)
    order = synth.epoch_order(synth.train_nodes(N, 0.2))
    seeds = [order[b * 400:(b + 1) * 400].cuda() for b in range(8)]

    def run():
        buf = gd.FeatureBuffer(torch.from_numpy(feat), N, 3, g.bounds(400, [15, 10, 5])[0][-1])   # S >= min(N, Q M_b)
        outs, pend = [], []
        for b, sd in enumerate(seeds):
            o = g.sample(sd, [15, 10, 5], 3, b)
            f, _, done = buf.extract(o.n_id, o.num_nodes_dev, o.max_nodes)
            done.synchronize()
            h = o.to_host()
            outs.append((h["n_id"], [c for c in h["col"]], f[:len(h["n_id"])].cpu().numpy()))
            pend.append(o)
            if len(pend) == 3:
                r = pend.pop(0)
                buf.release(r.n_id, r.num_nodes_dev, r.max_nodes)
        return outs

    a, b = run(), run()
    for x, y in zip(a, b):
        assert np.array_equal(x[0], y[0]) and all(np.array_equal(p, q) for p, q in zip(x[1], y[1]))
        assert np.array_equal(x[2], y[2])
    # the same batch sampled through another workspace and stream, in reverse order
    ws = g.workspace()
    st = torch.cuda.Stream()
    for bid in reversed(range(8)):
        o = g.sample(seeds[bid], [15, 10, 5], 3, bid, stream=st, workspace=ws)
        st.synchronize()
        assert np.array_equal(o.to_host()["n_id"], a[bid][0])


# ------------------------------------------------------------- f2: peer feature buffers


def _peer_setup(gd, N=60_000, E=600_000, B=500, fan=(10, 5)):
    indptr, indices = make_graph(N, E, seed=8)
    g = gd.Graph(indptr, indices)
    feat = table_np(N, 512)
    order = synth.epoch_order(synth.train_nodes(N, 0.3))
    nb, _ = O.sample_bounds(B, list(fan), N, E)
    return g, feat, order, nb[-1], list(fan), B


@pytest.mark.parametrize("mode", ["ce", "pull"])
def test_peer_buffer_parity_and_reuse(gd, mode):
    """f2: buffer B with buffer A attached as a peer.  A miss of B whose row A holds is
    copied from A's slot (served > 0); out, alias, hits/misses and B's whole state equal the
    oracle, which knows nothing about peers (Alg. 1 is unchanged)."""
    g, feat, order, n_max, fan, B = _peer_setup(gd)
    S = 3 * n_max
    bufA = gd.FeatureBuffer(torch.from_numpy(feat), S, 3, n_max)
    bufB = gd.FeatureBuffer(torch.from_numpy(feat), S, 3, n_max)
    for buf in (bufA, bufB):
        buf.stage_mode(mode == "ce")
        buf.config(4, 0.3)
    # A loads batches 0..5 and keeps them (released, still valid: delayed invalidation)
    pendA = []
    for b in range(6):
        res = g.sample(order[b * B:(b + 1) * B].cuda(), fan, 3, b)
        _, _, done = bufA.extract(res.n_id, res.num_nodes_dev, res.max_nodes)
        done.synchronize()
        pendA.append(res)
        if len(pendA) == 3:
            r = pendA.pop(0)
            bufA.release(r.n_id, r.num_nodes_dev, r.max_nodes)
    for r in pendA:
        bufA.release(r.n_id, r.num_nodes_dev, r.max_nodes)
    torch.cuda.synchronize()
    bufB.peer_attach([bufA])
    ob = O.Buffer(feat, S)
    pend = []
    for b in range(2, 12):       # overlaps A's batches 2..5 exactly, then new batches
        res = g.sample(order[b * B:(b + 1) * B].cuda(), fan, 3, b)
        alias = torch.empty(n_max, dtype=torch.int32, device="cuda")
        stats = torch.zeros(4, dtype=torch.int64, device="cuda")
        out, _, done = bufB.extract(res.n_id, res.num_nodes_dev, res.max_nodes, alias=alias, stats=stats)
        done.synchronize()
        n_id = res.to_host()["n_id"]
        o_out, o_alias, o_stats = ob.extract(n_id)
        n = len(n_id)
        assert tuple(stats.cpu().tolist()[:2]) == o_stats
        assert np.array_equal(alias[:n].cpu().numpy(), o_alias)
        assert np.array_equal(out[:n].cpu().numpy(), o_out)
        pend.append((res, n_id))
        if len(pend) == 3:
            r0, n0 = pend.pop(0)
            bufB.release(r0.n_id, r0.num_nodes_dev, r0.max_nodes)
            ob.release(n0)
    compare_state(bufB, ob)
    served, probed = bufB.peer_stats()
    assert probed > 0 and served > 0, (served, probed)
    assert bufA.peer_stats() == (0, 0)
    assert bufA.check() == 0 and bufB.check() == 0
    bufB.peer_attach([])


def test_peer_buffers_concurrent_eviction(gd):
    """Two buffers attached to each other run concurrently on their own streams with the
    minimum capacity (heavy eviction: peer slots are refilled while being read).  The seqlock
    tags must reject every stale copy: both outputs stay bit-exact with the oracle."""
    g, feat, order, n_max, fan, B = _peer_setup(gd, B=300)
    Q = 2
    S = Q * n_max
    bufs = [gd.FeatureBuffer(torch.from_numpy(feat), S, Q, n_max) for _ in range(2)]
    for buf in bufs:
        buf.config(4, 0.5)
    bufs[0].peer_attach([bufs[1]])
    bufs[1].peer_attach([bufs[0]])
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    wss = [g.workspace(), g.workspace()]          # concurrent samplers need their own workspace
    oracles = [O.Buffer(feat, S), O.Buffer(feat, S)]
    nbat = 24
    # rank r takes batches r, r+2, ... with a shift so the two share many nodes in flight
    sched = [[(2 * j + r) % 40 for j in range(nbat)] for r in range(2)]
    results = [[], []]
    pend = [[], []]
    for j in range(nbat):
        for r in range(2):
            b = sched[r][j]
            with torch.cuda.stream(streams[r]):
                res = g.sample(order[b * B:(b + 1) * B].cuda(non_blocking=True), fan, 3, b, stream=streams[r],
                               workspace=wss[r])
                out = torch.empty((n_max, 512), dtype=torch.uint8, device="cuda")
                alias = torch.empty(n_max, dtype=torch.int32, device="cuda")
                _, _, done = bufs[r].extract(res.n_id, res.num_nodes_dev, res.max_nodes, out=out, alias=alias,
                                             stream=streams[r])
                streams[r].wait_event(done)
                results[r].append((res, out, alias))
                pend[r].append(res)
                if len(pend[r]) == Q:
                    r0 = pend[r].pop(0)
                    bufs[r].release(r0.n_id, r0.num_nodes_dev, r0.max_nodes, stream=streams[r])
    torch.cuda.synchronize()
    for r in range(2):
        opend = []
        for j, (res, out, alias) in enumerate(results[r]):
            n_id = res.to_host()["n_id"]
            o_out, o_alias, _ = oracles[r].extract(n_id)
            n = len(n_id)
            assert np.array_equal(out[:n].cpu().numpy(), o_out), (r, j)
            assert np.array_equal(alias[:n].cpu().numpy(), o_alias), (r, j)
            opend.append(n_id)
            if len(opend) == Q:
                oracles[r].release(opend.pop(0))
        compare_state(bufs[r], oracles[r])
    s0, _ = bufs[0].peer_stats()
    s1, _ = bufs[1].peer_stats()
    assert s0 + s1 > 0
    for buf in bufs:
        buf.peer_attach([])
        assert buf.check() == 0
