"""Pins for oracle C6/C7 (Algorithm 1 extraction, release, LRU standby list).

* the paper's worked example, Figure 6 -> tests/golden/fig6.json;
* release-lag Q = 1: Alg. 1 + release equals an independently written batch-LRU model
  (SURVEY §8(c) P7), including the smallest case where per-access LRU differs;
* closed forms: preload -> no misses; capacity >= distinct nodes -> misses are exactly
  the compulsory first touches; out[i] == feat[ids[i]] bytewise regardless of state;
* the P:107 state table and refcount / standby invariants after every step.
CPU only.
"""
import json
import os
import random

import numpy as np
import pytest

from oracle import oracle as O

HERE = os.path.dirname(os.path.abspath(__file__))


def table(N, R=16, seed=0):
    rng = np.random.default_rng(seed)
    t = rng.integers(0, 256, size=(N, R), dtype=np.uint8)
    t[:, :4] = np.arange(N, dtype=np.int32).view(np.uint8).reshape(N, 4)
    return t


def test_figure6_worked_example():
    g = json.load(open(os.path.join(HERE, "golden", "fig6.json")))
    feat = table(g["num_nodes"])
    B = O.Buffer(feat, g["num_slots"])
    B.set_state(g["map_slot"], g["map_rc"], g["map_valid"], g["reverse"], g["standby"])
    out, alias, (hits, misses) = B.extract(np.array(g["batch"], dtype=np.int32))
    assert alias.tolist() == g["expect_alias"]
    assert (hits, misses) == (g["expect_hits"], g["expect_misses"])
    st = B.state()
    assert st["reverse"].tolist() == g["expect_reverse"]
    for v in g["expect_invalidated"]:
        assert st["valid"][v] == 0 and st["slot"][v] == -1
    assert st["standby"].tolist() == g["expect_standby_after_extract"]
    assert np.array_equal(out, feat[g["batch"]])
    B.release(np.array(g["release"], dtype=np.int32))
    assert B.state()["standby"].tolist() == g["expect_standby_after_release"]


def test_smallest_case_differs_from_per_access_lru():
    feat = table(3)
    B = O.Buffer(feat, 2)
    _, a1, s1 = B.extract(np.array([0, 1], dtype=np.int32))
    assert a1.tolist() == [0, 1] and s1 == (0, 2)
    B.release(np.array([0, 1], dtype=np.int32))
    _, a2, s2 = B.extract(np.array([2, 0], dtype=np.int32))
    assert a2.tolist() == [1, 0] and s2 == (1, 1)      # per-access LRU would give 0 hits


class BatchLRU:
    """Independent model for release lag 1: a recency list of slots,
    free slots first in ascending order.  Per batch: drop the batch's hits from the list;
    its misses take the oldest entries in order (evicting their nodes); then append all
    of the batch's slots at the MRU end in node-list order."""

    def __init__(self, S):
        self.rec = list(range(S))
        self.node_of = {}
        self.slot_of = {}

    def batch(self, ids):
        alias = [self.slot_of.get(v, -1) for v in ids]
        hits = sum(a >= 0 for a in alias)
        hit_slots = {a for a in alias if a >= 0}
        self.rec = [s for s in self.rec if s not in hit_slots]
        for i, v in enumerate(ids):
            if alias[i] < 0:
                s = self.rec.pop(0)
                if s in self.node_of:
                    del self.slot_of[self.node_of[s]]
                self.node_of[s] = v
                self.slot_of[v] = s
                alias[i] = s
        self.rec += alias
        return alias, hits, len(ids) - hits


@pytest.mark.parametrize("trial", range(60))
def test_release_lag_one_equals_batch_lru(trial):
    rng = random.Random(trial)
    N = rng.randint(3, 30)
    M = rng.randint(1, min(N, 8))
    S = rng.randint(M, N + 3)
    feat = table(N, seed=trial)
    B = O.Buffer(feat, S)
    model = BatchLRU(S)
    for _ in range(25):
        ids = rng.sample(range(N), rng.randint(0, M))
        out, alias, (h, m) = B.extract(np.array(ids, dtype=np.int32))
        ea, eh, em = model.batch(ids)
        assert alias.tolist() == ea and (h, m) == (eh, em)
        assert np.array_equal(out, feat[ids])
        B.release(np.array(ids, dtype=np.int32))


def check_state(B, unreleased):
    st = B.state()
    slot, rc, valid, rev = st["slot"], st["rc"], st["valid"], st["reverse"]
    assert not np.any((slot == -1) & (valid == 1))                 # P:107 impossible state
    for v in np.nonzero(valid)[0]:
        assert rev[slot[v]] == v                                   # map <-> reverse bijection
    expect_rc = np.zeros(B.N, dtype=np.int64)
    for ids in unreleased:
        expect_rc[ids] += 1
    assert np.array_equal(rc, expect_rc)                           # rc = #unreleased batches
    standby = st["standby"].tolist()
    assert len(set(standby)) == len(standby)
    busy = {int(slot[v]) for v in np.nonzero(rc > 0)[0]}
    assert set(standby) == set(range(B.S)) - busy                  # standby = rc-0 slots


@pytest.mark.parametrize("Q", [1, 2, 4])
def test_random_schedule_invariants(Q):
    rng = np.random.default_rng(Q)
    N, M = 200, 20
    S = Q * M
    feat = table(N, R=24, seed=Q)
    B = O.Buffer(feat, S)
    pending = []
    for step in range(120):
        w = rng.zipf(1.6, size=400) % N                          # skewed re-use
        ids = np.array(list(dict.fromkeys(w.tolist()))[: rng.integers(1, M + 1)], dtype=np.int32)
        out, alias, _ = B.extract(ids)
        assert np.array_equal(out, feat[ids])                      # closed form, any state
        pending.append(ids)
        if len(pending) == Q:
            B.release(pending.pop(0))
        check_state(B, pending)


def test_compulsory_misses_when_capacity_covers_everything():
    rng = np.random.default_rng(5)
    N = 300
    B = O.Buffer(table(N), N)
    seen = set()
    for _ in range(50):
        ids = rng.choice(N, size=int(rng.integers(1, 40)), replace=False).astype(np.int32)
        _, _, (h, m) = B.extract(ids)
        new = len(set(ids.tolist()) - seen)
        assert m == new and h == len(ids) - new
        seen |= set(ids.tolist())
        if rng.random() < 0.7:
            B.release(ids)


def test_preload_no_misses():
    N = 100
    feat = table(N)
    B = O.Buffer(feat, N, preload=True)
    ids = np.array([5, 99, 0, 42], dtype=np.int32)
    out, alias, st = B.extract(ids)
    assert st == (4, 0) and alias.tolist() == ids.tolist() and np.array_equal(out, feat[ids])


def test_capacity_violation_and_underflow():
    B = O.Buffer(table(10), 2)
    B.extract(np.array([0, 1], dtype=np.int32))
    with pytest.raises(RuntimeError):
        B.extract(np.array([2], dtype=np.int32))            # standby dry: capacity rule
    B2 = O.Buffer(table(10), 4)
    with pytest.raises(RuntimeError):
        B2.release(np.array([3], dtype=np.int32))


def test_bounded_table_rows_mod_p():
    """mag240m's bounded host table: node v's row is table[v mod P] (R15)."""
    rng = np.random.default_rng(9)
    N, P = 500, 37
    feat = table(P, R=32, seed=9)
    B = O.Buffer(feat, 64, num_nodes=N)
    pend = []
    for _ in range(40):
        ids = rng.choice(N, size=20, replace=False).astype(np.int32)
        out, alias, _ = B.extract(ids)
        assert np.array_equal(out, feat[ids % P])
        pend.append(ids)
        if len(pend) == 3:
            B.release(pend.pop(0))
    with pytest.raises(ValueError):
        O.Buffer(feat, 600, preload=True, num_nodes=N + 1000)   # preload needs capacity >= N


@pytest.mark.parametrize("Q,P", [(1, 200), (3, 200), (4, 61)])
def test_bookkeeping_only_buffer_equals_full_buffer(Q, P):
    """keep_rows=False (the full-size replays' oracle: no S x R slot contents) takes exactly the
    same Alg. 1 decisions: alias, hits/misses and the whole state match the full buffer every
    step; its extract refuses `out`.  gather_rows is the closed form feat[ids mod P]."""
    rng = np.random.default_rng(Q * 7 + P)
    N, M = 200, 25
    feat = table(P, R=20, seed=Q)
    A = O.Buffer(feat, Q * M, num_nodes=N)
    B = O.Buffer(feat, Q * M, num_nodes=N, keep_rows=False)
    pending = []
    for step in range(80):
        w = rng.zipf(1.5, size=300) % N
        ids = np.array(list(dict.fromkeys(w.tolist()))[: rng.integers(1, M + 1)], dtype=np.int32)
        out, a1, s1 = A.extract(ids)
        none, a2, s2 = B.extract(ids)
        assert none is None and s1 == s2 and np.array_equal(a1, a2)
        assert np.array_equal(O.gather_rows(feat, ids), out)
        pending.append(ids)
        if len(pending) == Q:
            r = pending.pop(0)
            A.release(r)
            B.release(r)
        sa, sb = A.state(), B.state()
        for k in sa:
            assert np.array_equal(sa[k], sb[k]), k
    with pytest.raises(RuntimeError):
        B.extract(np.array([0], dtype=np.int32), want_out=True)
