"""Pins for oracle C3-C5 (Floyd sampling, cumulative frontier, first-occurrence relabel).

Floyd is pinned by exhaustive enumeration (every f-subset of [0, d) is produced by exactly
f! of the d!/(d-f)! draw sequences), sampling by invariants + a chi-square uniformity test,
and multi-hop sampling by the textbook BFS special case (fanout >= max degree), brute-force
K-hop balls on hand-built graphs (isolated node, self-loop, multi-edge, star, path) and the
structural invariants of SURVEY §8(c) P4.  CPU only.
"""
import itertools
import math
from collections import Counter, deque

import numpy as np
import pytest
import torch

from oracle import oracle as O
import synth


@pytest.mark.parametrize("d,f", [(5, 3), (6, 2), (7, 4), (8, 8), (9, 1), (10, 5), (4, 0)])
def test_floyd_enumeration_uniform(d, f):
    counts = Counter()
    for draws in itertools.product(*[range(d - f + t + 1) for t in range(f)]):
        pos = O.floyd(d, f, list(draws))
        assert pos == sorted(set(pos)) and len(pos) == f and all(0 <= p < d for p in pos)
        counts[tuple(pos)] += 1
    assert len(counts) == math.comb(d, f)
    assert set(counts.values()) == {math.factorial(f)}


def test_floyd_exclusive_bound_would_be_biased():
    """Sanity of the reading C9: with the inclusive bound, d=2, f=1 can pick position 1."""
    assert O.floyd(2, 1, [1]) == [1]
    assert O.floyd(2, 1, [0]) == [0]


def test_sample_positions_special_cases():
    for d in range(0, 12):
        for f in [-1, 0, 1, 3, 5, 11, 40]:
            pos = O.sample_positions(v=17, d=d, f=f, h=1, b=3, seed=99)
            if f < 0 or d <= f:
                assert pos == list(range(d))              # the CSR row verbatim (C11)
            else:
                assert len(pos) == f and pos == sorted(set(pos)) and all(0 <= p < d for p in pos)


def test_sample_positions_is_floyd_of_the_drawn_words():
    seed = 3
    for (v, d, f, h, b) in [(5, 100, 15, 0, 0), (123, 7, 5, 2, 9), (2**31 - 1, 1000, 25, 1, 77)]:
        draws = [O.randint(O.draw_word(t, v, h, b, seed), d - f + t) for t in range(f)]
        assert O.sample_positions(v, d, f, h, b, seed) == O.floyd(d, f, draws)


def test_sample_positions_chi_square():
    """Star-graph hub with d=6, f=2 over 30000 independent keys: uniform over 15 subsets."""
    from scipy.stats import chisquare
    counts = Counter()
    for v in range(30000):
        counts[tuple(O.sample_positions(v, 6, 2, 0, 1, 3))] += 1
    obs = [counts[c] for c in itertools.combinations(range(6), 2)]
    assert sum(obs) == 30000
    assert chisquare(obs).pvalue > 1e-4
    # each position marginally selected with probability f/d = 1/3
    per_pos = Counter(p for c, k in counts.items() for p in c for _ in range(k))
    for p in range(6):
        assert abs(per_pos[p] / 30000 - 1 / 3) < 0.02


# ----------------------------------------------------------------------------- multi-hop


def csr_from_lists(rows):
    indptr = np.zeros(len(rows) + 1, dtype=np.int64)
    for i, r in enumerate(rows):
        indptr[i + 1] = indptr[i] + len(r)
    indices = np.array([u for r in rows for u in r], dtype=np.int32)
    return indptr, indices


HAND_GRAPHS = {
    # node 3 isolated, node 1 has a self-loop, node 2 a multi-edge
    "mixed": [[1, 2], [1, 0, 4], [0, 0, 4], [], [5], [2]],
    "star": [[1, 2, 3, 4, 5, 6, 7, 8]] + [[0] for _ in range(8)],
    "path": [[1], [2], [3], [4], [5], [6], [7], [8], [9], [10], [11], []],
    "cycle_multi": [[1, 1, 1], [2, 2], [0], [0, 1, 2]],
}


def bfs_order(indptr, indices, seeds, K):
    """Textbook level-synchronous BFS visit order (first discovery), K levels."""
    seen = {int(s): i for i, s in enumerate(seeds)}
    order = [int(s) for s in seeds]
    q = deque((int(s), 0) for s in seeds)
    while q:
        v, lvl = q.popleft()
        if lvl == K:
            continue
        for u in indices[indptr[v]:indptr[v + 1]]:
            u = int(u)
            if u not in seen:
                seen[u] = len(order)
                order.append(u)
                q.append((u, lvl + 1))
    return order


def check_invariants(indptr, indices, seeds, fanouts, res):
    K = len(fanouts)
    n_id, sizes = res.n_id, res.sizes
    assert len(set(n_id.tolist())) == len(n_id)                 # relabel is a bijection
    assert np.array_equal(n_id[: len(seeds)], seeds)            # seeds first
    for h in range(1, K + 1):
        n_prev, n_h, e_h = int(sizes[h - 1]), int(sizes[h]), int(sizes[K + h])
        f = fanouts[h - 1]
        rp, col, eid = res.rowptr[h - 1], res.col[h - 1], res.eid[h - 1]
        assert len(rp) == n_prev + 1 and rp[0] == 0 and rp[-1] == e_h
        for i in range(n_prev):
            v = int(n_id[i])
            d = int(indptr[v + 1] - indptr[v])
            cnt = int(rp[i + 1] - rp[i])
            assert cnt == (d if f < 0 else min(f, d))            # count = min(fanout, degree)
            e = eid[rp[i]:rp[i + 1]]
            assert np.all(e >= indptr[v]) and np.all(e < indptr[v + 1])
            assert np.all(np.diff(e) > 0)                        # distinct, ascending positions
        assert np.all(col >= 0) and np.all(col < n_h)
        assert np.array_equal(n_id[col], indices[eid])           # every sampled edge exists
        # new local ids appear in increasing first-occurrence order
        nxt = n_prev
        for c in col.tolist():
            if c >= nxt:
                assert c == nxt
                nxt += 1
        assert nxt == n_h


@pytest.mark.parametrize("name", sorted(HAND_GRAPHS))
def test_hand_graphs_bfs_and_ball(name):
    indptr, indices = csr_from_lists(HAND_GRAPHS[name])
    N = len(indptr) - 1
    maxdeg = int(np.max(np.diff(indptr)))
    for seeds in ([0], [3, 0], list(range(min(N, 3)))):
        seeds = np.array(seeds, dtype=np.int32)
        for K in (1, 2, 3):
            for fan in ([-1] * K, [maxdeg] * K, [maxdeg + 5] * K):
                res = O.sample(indptr, indices, seeds, fan, rng_seed=3, batch_id=0)
                check_invariants(indptr, indices, seeds, fan, res)
                assert res.n_id.tolist() == bfs_order(indptr, indices, seeds, K)
            # small fanouts: result inside the K-hop ball
            ball = set(bfs_order(indptr, indices, seeds, K))
            for b in range(20):
                res = O.sample(indptr, indices, seeds, [1] * K, rng_seed=5, batch_id=b)
                check_invariants(indptr, indices, seeds, [1] * K, res)
                assert set(res.n_id.tolist()) <= ball


@pytest.fixture(scope="module")
def tiny():
    cfg = synth.CONFIGS["tiny"]
    indptr, indices = synth.chung_lu_csr(cfg.num_nodes, cfg.num_edges)
    train = synth.train_nodes(cfg.num_nodes, cfg.train_frac)
    order = synth.epoch_order(train)
    return cfg, indptr.numpy(), indices.numpy(), order


def test_tiny_graph_shape(tiny):
    cfg, indptr, indices, order = tiny
    deg = np.diff(indptr)
    assert indptr[0] == 0 and indptr[-1] == cfg.num_edges and np.all(deg >= 0)
    assert indices.min() >= 0 and indices.max() < cfg.num_nodes
    assert deg.max() > 5 * deg.mean()                      # power law: heavy hubs


def test_tiny_sampling_invariants_and_determinism(tiny):
    cfg, indptr, indices, order = tiny
    for b in range(8):
        seeds = synth.batch_seeds(order, cfg.batch_size, b).numpy()
        res = O.sample(indptr, indices, seeds, list(cfg.fanouts), synth.RNG_SEED, b)
        check_invariants(indptr, indices, seeds, list(cfg.fanouts), res)
        again = O.sample(indptr, indices, seeds, list(cfg.fanouts), synth.RNG_SEED, b)
        assert np.array_equal(res.n_id, again.n_id)
        other = O.sample(indptr, indices, seeds, list(cfg.fanouts), synth.RNG_SEED, b + 1000)
        assert not np.array_equal(res.n_id, other.n_id)     # the batch id keys the draws


def test_three_hop_products_fanouts_on_tiny(tiny):
    cfg, indptr, indices, order = tiny
    seeds = synth.batch_seeds(order, 200, 0).numpy()
    for fan in ([15, 10, 5], [25, 15], [10, 10, 10], [0, 3], [40, 1]):
        res = O.sample(indptr, indices, seeds, fan, 11, 4)
        check_invariants(indptr, indices, seeds, fan, res)


def test_duplicate_or_bad_seed_rejected(tiny):
    cfg, indptr, indices, order = tiny
    with pytest.raises(ValueError):
        O.sample(indptr, indices, np.array([1, 2, 1], dtype=np.int32), [2], 1, 0)
    with pytest.raises(ValueError):
        O.sample(indptr, indices, np.array([cfg.num_nodes], dtype=np.int32), [2], 1, 0)


def test_generator_cpu_is_deterministic():
    a = synth.chung_lu_csr(5000, 40000)
    b = synth.chung_lu_csr(5000, 40000)
    assert torch.equal(a[0], b[0]) and torch.equal(a[1], b[1])


def _py_positions(v, d, f, hop0, b, seed):
    """R2-R3 written out in Python: Floyd over draws floor(u (j+1) / 2^64), u the Philox draw
    word keyed (t, v, hop index, batch id) (the word itself is pinned to curand in
    test_oracle_rng), positions ascending; f < 0 or d <= f: the whole row."""
    if f < 0 or d <= f:
        return list(range(d))
    S = []
    for t in range(f):
        j = d - f + t
        r = (O.draw_word(t, v, hop0, b, seed) * (j + 1)) >> 64
        S.append(j if r in S else r)
    return sorted(S)


def test_sample_rows_are_keyed_by_node_hop_and_batch(tiny):
    """Pins the wiring inside oracle_sample: every row of every hop of a
    multi-hop sample is exactly indptr[v] + positions(v, deg v, f_h, h - 1, batch_id).  A
    swapped or 1-based hop index, a wrong batch id or a frontier-index key fails here, which
    the invariant and BFS pins cannot see."""
    cfg, indptr, indices, order = tiny
    seed = 7
    for b, fan in ((0, [5, 5]), (3, [15, 10, 5]), (123456, [2, 3, 4, 1])):
        seeds = synth.batch_seeds(order, 48, b % 10).numpy()
        res = O.sample(indptr, indices, seeds, fan, seed, b)
        checked = 0
        for h in range(1, len(fan) + 1):
            rp, eid = res.rowptr[h - 1], res.eid[h - 1]
            for i in range(int(res.sizes[h - 1])):
                v = int(res.n_id[i])
                d = int(indptr[v + 1] - indptr[v])
                want = [int(indptr[v]) + p for p in _py_positions(v, d, fan[h - 1], h - 1, b, seed)]
                assert eid[rp[i]:rp[i + 1]].tolist() == want, (b, h, i, v)
                checked += d > fan[h - 1] >= 0
        assert checked > 50      # plenty of rows where the draws decide


def test_star_hub_uniform_through_oracle_sample():
    """SURVEY P3 through the whole sampler: a star hub with 6 leaves sampled with fanout 2 in
    6000 mini-batches (batch id = the only thing that varies) picks each of the 15 leaf pairs
    uniformly (chi-square), and the relabel puts them in ascending position order."""
    from scipy.stats import chisquare
    indptr, indices = csr_from_lists([[1, 2, 3, 4, 5, 6]] + [[0]] * 6)
    seeds = np.array([0], dtype=np.int32)
    counts = Counter()
    for b in range(6000):
        res = O.sample(indptr, indices, seeds, [2], 3, b)
        pair = tuple(res.n_id[1:].tolist())
        assert len(pair) == 2 and pair[0] < pair[1] and res.col[0].tolist() == [1, 2]
        counts[pair] += 1
    obs = [counts[c] for c in itertools.combinations(range(1, 7), 2)]
    assert sum(obs) == 6000
    assert chisquare(obs).pvalue > 1e-4
