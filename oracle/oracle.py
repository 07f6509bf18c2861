"""ctypes binding of the CPU oracle (oracle/gd_oracle.cpp).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference leg.  The product package never
imports this module.  Arrays are numpy; nothing here touches torch or CUDA.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gd_oracle.cpp")
_LIB = os.path.join(_HERE, "libgd_oracle.so")

_i64p = ctypes.POINTER(ctypes.c_int64)
_i32p = ctypes.POINTER(ctypes.c_int32)
_u8p = ctypes.POINTER(ctypes.c_uint8)
_u32p = ctypes.POINTER(ctypes.c_uint32)
_u64p = ctypes.POINTER(ctypes.c_uint64)


def build(force: bool = False) -> str:
    """Compile the oracle with plain g++ (no CUDA headers)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        L.oracle_philox4x32_10.argtypes = [_u32p, _u32p, _u32p]
        L.oracle_philox4x32_10.restype = None
        L.oracle_philox4x32_10_many.argtypes = [ctypes.c_int64, _u32p, _u32p]
        L.oracle_philox4x32_10_many.restype = None
        L.oracle_randint.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.oracle_randint.restype = ctypes.c_uint64
        L.oracle_draw_word.argtypes = [ctypes.c_uint32] * 4 + [ctypes.c_uint64]
        L.oracle_draw_word.restype = ctypes.c_uint64
        L.oracle_floyd.argtypes = [ctypes.c_int64, ctypes.c_int32, _u64p, _i64p]
        L.oracle_floyd.restype = None
        L.oracle_sample_positions.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32,
                                              ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64, _i64p]
        L.oracle_sample_positions.restype = ctypes.c_int64
        L.oracle_sample.argtypes = [_i64p, _i32p, ctypes.c_int64, _i32p, ctypes.c_int64, _i32p,
                                    ctypes.c_int32, ctypes.c_uint64, ctypes.c_uint32, _i32p,
                                    ctypes.POINTER(_i64p), ctypes.POINTER(_i32p),
                                    ctypes.POINTER(_i64p), _i64p]
        L.oracle_sample.restype = ctypes.c_int
        L.oracle_buffer_create.argtypes = [_u8p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                                           ctypes.c_int64]
        L.oracle_buffer_create.restype = ctypes.c_void_p
        L.oracle_buffer_create2.argtypes = [_u8p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                                            ctypes.c_int64, ctypes.c_int]
        L.oracle_buffer_create2.restype = ctypes.c_void_p
        L.oracle_gather_rows.argtypes = [_u8p, ctypes.c_int64, ctypes.c_int64, _i32p, ctypes.c_int64, _u8p]
        L.oracle_gather_rows.restype = None
        L.oracle_buffer_destroy.argtypes = [ctypes.c_void_p]
        L.oracle_buffer_destroy.restype = None
        L.oracle_extract.argtypes = [ctypes.c_void_p, _i32p, ctypes.c_int64, _u8p, _i32p, _i64p]
        L.oracle_extract.restype = ctypes.c_int
        L.oracle_release.argtypes = [ctypes.c_void_p, _i32p, ctypes.c_int64]
        L.oracle_release.restype = ctypes.c_int
        L.oracle_buffer_state.argtypes = [ctypes.c_void_p, _i32p, _i32p, _u8p, _i32p, _i32p]
        L.oracle_buffer_state.restype = ctypes.c_int64
        L.oracle_buffer_set_state.argtypes = [ctypes.c_void_p, _i32p, _i32p, _u8p, _i32p, _i32p, ctypes.c_int64]
        L.oracle_buffer_set_state.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a, t):
    return a.ctypes.data_as(t) if a is not None else None


def philox4x32_10(ctr, key):
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    o = np.zeros(4, dtype=np.uint32)
    lib().oracle_philox4x32_10(_p(c, _u32p), _p(k, _u32p), _p(o, _u32p))
    return [int(x) for x in o]


def philox4x32_10_many(ctr_key: np.ndarray) -> np.ndarray:
    ck = np.ascontiguousarray(ctr_key, dtype=np.uint32).reshape(-1, 6)
    o = np.zeros((len(ck), 4), dtype=np.uint32)
    lib().oracle_philox4x32_10_many(len(ck), _p(ck, _u32p), _p(o, _u32p))
    return o


def randint(u: int, j: int) -> int:
    return int(lib().oracle_randint(u, j))


def draw_word(t: int, v: int, h: int, b: int, seed: int) -> int:
    return int(lib().oracle_draw_word(t, v, h, b, seed))


def floyd(d: int, f: int, draws) -> list[int]:
    r = np.asarray(draws, dtype=np.uint64)
    pos = np.zeros(max(f, 1), dtype=np.int64)
    lib().oracle_floyd(d, f, _p(r, _u64p), _p(pos, _i64p))
    return [int(x) for x in pos[:f]]


def sample_positions(v: int, d: int, f: int, h: int, b: int, seed: int) -> list[int]:
    pos = np.zeros(max(d, 1), dtype=np.int64)
    n = lib().oracle_sample_positions(v, d, f, h, b, seed, _p(pos, _i64p))
    return [int(x) for x in pos[:n]]


def sample_bounds(num_seeds: int, fanouts, num_nodes: int, num_edges: int):
    """Worst-case sizes: n_h <= min(N, n_{h-1}(1+f_h)), e_h <= min(E, n_{h-1} f_h) (f<0: E)."""
    n = [num_seeds]
    e = []
    for f in fanouts:
        eh = num_edges if f < 0 else min(num_edges, n[-1] * f)
        e.append(eh)
        n.append(min(num_nodes, n[-1] + eh))
    return n, e


def gather_rows(feat_u8: np.ndarray, ids: np.ndarray, out: np.ndarray | None = None) -> np.ndarray:
    """CPU-variant data path: out[i] = feat_u8[ids[i] mod P] (releases the GIL)."""
    ids = np.ascontiguousarray(ids, dtype=np.int32)
    P, R = feat_u8.shape
    if out is None:
        out = np.empty((len(ids), R), dtype=np.uint8)
    assert out.flags.c_contiguous and out.shape[0] >= len(ids) and out.shape[1] == R
    lib().oracle_gather_rows(_p(feat_u8, _u8p), P, R, _p(ids, _i32p), len(ids), _p(out, _u8p))
    return out


class SampleResult:
    def __init__(self, n_id, rowptr, col, eid, sizes):
        self.n_id, self.rowptr, self.col, self.eid, self.sizes = n_id, rowptr, col, eid, sizes


def sample(indptr: np.ndarray, indices: np.ndarray, seeds: np.ndarray, fanouts, rng_seed: int,
           batch_id: int) -> SampleResult:
    """C3-C5 multi-hop sampling + relabel of one mini-batch (see gd_oracle.cpp)."""
    indptr = np.ascontiguousarray(indptr, dtype=np.int64)
    indices = np.ascontiguousarray(indices, dtype=np.int32)
    seeds = np.ascontiguousarray(seeds, dtype=np.int32)
    fan = np.ascontiguousarray(fanouts, dtype=np.int32)
    K = len(fan)
    N = indptr.shape[0] - 1
    nb, eb = sample_bounds(len(seeds), list(fan), N, int(indptr[-1]))
    n_id = np.zeros(max(nb[-1], 1), dtype=np.int32)
    rp = [np.zeros(nb[h] + 1, dtype=np.int64) for h in range(K)]
    cl = [np.zeros(max(eb[h], 1), dtype=np.int32) for h in range(K)]
    ed = [np.zeros(max(eb[h], 1), dtype=np.int64) for h in range(K)]
    sizes = np.zeros(2 * K + 1, dtype=np.int64)
    RP = (_i64p * K)(*[_p(a, _i64p) for a in rp])
    CL = (_i32p * K)(*[_p(a, _i32p) for a in cl])
    ED = (_i64p * K)(*[_p(a, _i64p) for a in ed])
    rc = lib().oracle_sample(_p(indptr, _i64p), _p(indices, _i32p), N, _p(seeds, _i32p), len(seeds),
                             _p(fan, _i32p), K, rng_seed, batch_id, _p(n_id, _i32p), RP, CL, ED,
                             _p(sizes, _i64p))
    if rc != 0:
        raise ValueError("oracle_sample: precondition violated (duplicate or out-of-range seed)")
    nK = int(sizes[K])
    rowptr = [rp[h][: int(sizes[h]) + 1] for h in range(K)]
    col = [cl[h][: int(sizes[K + 1 + h])] for h in range(K)]
    eid = [ed[h][: int(sizes[K + 1 + h])] for h in range(K)]
    return SampleResult(n_id[:nK].copy(), rowptr, col, eid, sizes)


class Buffer:
    """Algorithm 1 feature buffer over a host table feat[N, R] (uint8 view)."""

    def __init__(self, feat_u8: np.ndarray, capacity_slots: int, preload: bool = False, num_nodes: int | None = None,
                 keep_rows: bool = True):
        """feat_u8 [P, R]: node v's row is feat_u8[v mod P]; num_nodes defaults to P.
        keep_rows=False: bookkeeping only (no S x R slot contents; extract(want_out=True) fails)."""
        assert feat_u8.dtype == np.uint8 and feat_u8.ndim == 2 and feat_u8.flags.c_contiguous
        self.feat = feat_u8
        self.P, self.R = feat_u8.shape
        self.N = int(num_nodes) if num_nodes is not None else self.P
        self.S = int(capacity_slots)
        self.keep_rows = bool(keep_rows)
        self.h = lib().oracle_buffer_create2(_p(feat_u8, _u8p), self.N, self.R, self.S, int(preload), self.P,
                                             int(self.keep_rows))
        if not self.h:
            raise ValueError("oracle_buffer_create: preload requires capacity >= N, and 1 <= P <= N")

    def __del__(self):
        if getattr(self, "h", None):
            lib().oracle_buffer_destroy(self.h)
            self.h = None

    def extract(self, ids: np.ndarray, want_out: bool | None = None):
        if want_out is None:
            want_out = self.keep_rows
        ids = np.ascontiguousarray(ids, dtype=np.int32)
        n = len(ids)
        out = np.zeros((n, self.R), dtype=np.uint8) if want_out else None
        alias = np.zeros(max(n, 1), dtype=np.int32)
        stats = np.zeros(2, dtype=np.int64)
        rc = lib().oracle_extract(self.h, _p(ids, _i32p), n, _p(out, _u8p), _p(alias, _i32p), _p(stats, _i64p))
        if rc == -2:
            raise RuntimeError("oracle_extract: a bookkeeping-only buffer (keep_rows=False) has no rows for `out`")
        if rc != 0:
            raise RuntimeError("oracle_extract: standby list ran dry (capacity rule violated)")
        return out, alias[:n], (int(stats[0]), int(stats[1]))

    def release(self, ids: np.ndarray):
        ids = np.ascontiguousarray(ids, dtype=np.int32)
        if lib().oracle_release(self.h, _p(ids, _i32p), len(ids)) != 0:
            raise RuntimeError("oracle_release: reference count underflow")

    def state(self):
        ms = np.zeros(self.N, dtype=np.int32)
        mr = np.zeros(self.N, dtype=np.int32)
        mv = np.zeros(self.N, dtype=np.uint8)
        rv = np.zeros(self.S, dtype=np.int32)
        sb = np.zeros(max(self.S, 1), dtype=np.int32)
        k = lib().oracle_buffer_state(self.h, _p(ms, _i32p), _p(mr, _i32p), _p(mv, _u8p), _p(rv, _i32p), _p(sb, _i32p))
        return {"slot": ms, "rc": mr, "valid": mv, "reverse": rv, "standby": sb[:k].copy()}

    def set_state(self, slot, rc, valid, reverse, standby):
        slot = np.ascontiguousarray(slot, dtype=np.int32)
        rc = np.ascontiguousarray(rc, dtype=np.int32)
        valid = np.ascontiguousarray(valid, dtype=np.uint8)
        reverse = np.ascontiguousarray(reverse, dtype=np.int32)
        standby = np.ascontiguousarray(standby, dtype=np.int32)
        lib().oracle_buffer_set_state(self.h, _p(slot, _i32p), _p(rc, _i32p), _p(valid, _u8p),
                                      _p(reverse, _i32p), _p(standby, _i32p), len(standby))
