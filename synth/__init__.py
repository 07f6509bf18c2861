"""Seeded synthetic inputs shaped like the paper's workloads (Table 1).

This module is the ONE place both sides (the CUDA path and the oracle, via tests/bench)
take their inputs from.  It holds none of the method's arithmetic: no Philox, no Floyd,
no relabel, no buffer logic.  Its only randomness is SplitMix64 (Steele et al., OOPSLA'14)
over integer counters, written with torch int64 ops so CPU and GPU produce identical bits.

Recipe:
  * graph: Chung-Lu power law.  Node v has rank r = rank[v] under a SplitMix64-keyed
    permutation; weight w_r = (r + r0)^-alpha (alpha 0.8, r0 100), quantised to int64
    wfix_r = max(1, floor(2^20 * w_r / w_0)).  indptr[v+1] = floor(cum_v * E / W) with
    cum the prefix sum of wfix over node order (float64 product, exact-rounded on every
    device), indptr[N] = E.  Edge k's neighbour is drawn by inverse CDF over the same
    weights (in rank order) with x_k = SplitMix64(seed, k) mod W.  Multi-edges and
    self-loops occur, rows are unsorted — as in real CSRs.
  * features: row-major [N x R bytes] in ascending node id; word c of row v is
    lo32(SplitMix64(fseed, v*W + c)), the first 8 bytes are v (int64 tag).  Random bits
    include NaN payloads, -0.0, denormals and inf; a few rows are forced to them.
  * seeds: train set = first T nodes of a SplitMix64 permutation (train_seed), epoch
    order another permutation; global batch b = order[b*B:(b+1)*B] (distinct ids).
"""
from __future__ import annotations

import dataclasses
import hashlib

import numpy as np
import torch

_GOLDEN = -7046029254386353131        # 0x9E3779B97F4A7C15 as int64
_M1 = -4658895280553007687            # 0xBF58476D1CE4E5B9
_M2 = -7723592293110705685            # 0x94D049BB133111EB


def _lsr(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 (torch >> is arithmetic)."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    z = x + _GOLDEN
    z = (z ^ _lsr(z, 30)) * _M1
    z = (z ^ _lsr(z, 27)) * _M2
    return z ^ _lsr(z, 31)


def _mix_seed(seed: int, salt: int) -> int:
    v = splitmix64(torch.tensor([seed * 1000003 + salt], dtype=torch.int64))
    return int(v.item())


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    num_nodes: int
    num_edges: int
    feat_dim: int
    elem_bytes: int
    batch_size: int
    fanouts: tuple
    buffer_frac: float          # capacity S as a fraction of N (1.0 + preload = all resident)
    preload: bool
    train_frac: float
    table_rows: int | None = None   # physical host-table rows P (node v -> row v mod P); None = N

    @property
    def row_bytes(self) -> int:
        return self.feat_dim * self.elem_bytes

    @property
    def host_rows(self) -> int:
        return self.table_rows or self.num_nodes


# BASELINE.json configs; shapes from SURVEY.md §8.0
CONFIGS = {
    "tiny": Config("tiny", 10_000, 100_000, 128, 4, 64, (5, 5), 1.0, True, 0.10),
    "products": Config("products", 2_400_000, 62_000_000, 100, 4, 1024, (15, 10, 5), 1.0, True, 0.08),
    "papers100m": Config("papers100m", 111_000_000, 1_600_000_000, 128, 4, 1000, (15, 10, 5), 0.10, False, 0.0109),
    "friendster": Config("friendster", 65_000_000, 1_800_000_000, 256, 4, 1000, (10, 10, 10), -1.0, False, 0.01),
    # 375 GB logical table > the 196 GB of host RAM of this pool's boxes: a bounded physical
    # table of 64M rows (98 GB), node v -> row v mod 64M (R15)
    "mag240m": Config("mag240m", 244_000_000, 1_700_000_000, 768, 2, 1000, (25, 15), 0.10, False, 0.0046,
                      table_rows=64_000_000),
}

GRAPH_SEED, TRAIN_SEED, RNG_SEED, FEATURE_SEED = 1, 2, 3, 4


def node_rank_order(num_nodes: int, seed: int, device="cpu") -> torch.Tensor:
    """order[r] = node with rank r (a SplitMix64-keyed permutation; keys are distinct)."""
    key = splitmix64(torch.arange(num_nodes, dtype=torch.int64, device=device) ^ _mix_seed(seed, 11))
    return torch.argsort(key)


def rank_weights(num_nodes: int, alpha: float = 0.8, r0: float = 100.0) -> np.ndarray:
    r = np.arange(num_nodes, dtype=np.float64)
    w = np.power((r + r0) / r0, -alpha)        # w_r / w_0
    return np.maximum(1, np.floor(w * (1 << 20))).astype(np.int64)


def chung_lu_csr(num_nodes: int, num_edges: int, seed: int = GRAPH_SEED, alpha: float = 0.8,
                 r0: float = 100.0, device="cpu", chunk: int = 1 << 26):
    """Returns (indptr int64[N+1], indices int32[E]) as torch tensors on `device`."""
    N, E = int(num_nodes), int(num_edges)
    order = node_rank_order(N, seed, device)                          # rank -> node
    wfix_rank = torch.from_numpy(rank_weights(N, alpha, r0)).to(device)
    rank = torch.empty_like(order)
    rank[order] = torch.arange(N, dtype=torch.int64, device=device)   # node -> rank
    cum_node = torch.cumsum(wfix_rank[rank], 0)                       # over node order
    W = int(cum_node[-1].item())
    scale = float(E) / float(W)
    indptr = torch.zeros(N + 1, dtype=torch.int64, device=device)
    indptr[1:] = torch.clamp(torch.floor(cum_node.to(torch.float64) * scale).to(torch.int64), max=E)
    indptr[N] = E
    del cum_node, rank
    cum_rank = torch.cumsum(wfix_rank, 0)                             # over rank order
    del wfix_rank
    indices = torch.empty(E, dtype=torch.int32, device=device)
    salt = _mix_seed(seed, 12)
    for s in range(0, E, chunk):
        k = torch.arange(s, min(E, s + chunk), dtype=torch.int64, device=device)
        x = _lsr(splitmix64(k ^ salt), 1) % W
        r = torch.searchsorted(cum_rank, x, right=True)
        indices[s:s + len(k)] = order[r].to(torch.int32)
        del k, x, r
    return indptr, indices


def feature_rows(v0: int, v1: int, row_bytes: int, seed: int = FEATURE_SEED, device="cpu") -> torch.Tensor:
    """Rows v0..v1-1 of the feature table as uint8 [v1-v0, row_bytes]."""
    assert row_bytes % 8 == 0
    W = row_bytes // 4
    v = torch.arange(v0, v1, dtype=torch.int64, device=device)
    c = torch.arange(W, dtype=torch.int64, device=device)
    key = (v[:, None] * W + c[None, :]) ^ _mix_seed(seed, 13)
    words = (splitmix64(key) & 0xFFFFFFFF).to(torch.int32)   # two's complement lo32
    words[:, 0] = (v & 0xFFFFFFFF).to(torch.int32)           # int64 tag = v (little endian)
    words[:, 1] = _lsr(v, 32).to(torch.int32)
    special = torch.tensor([0x7FC00001, -0x80000000, 0x00000001, 0x7F800000, -0x800000, 0x7FA00000],
                           dtype=torch.int32, device=device)
    sel = (v % 997) == 3                                      # a handful of rows: NaN payloads,
    if bool(sel.any()) and W > 2:                             # -0.0, denormal, +/-inf, sNaN
        rep = special.repeat((W - 2 + len(special) - 1) // len(special))[: W - 2]
        words[sel, 2:] = rep
    return words.view(torch.uint8).reshape(v1 - v0, row_bytes)


def feature_table(num_nodes: int, row_bytes: int, seed: int = FEATURE_SEED, out: torch.Tensor | None = None,
                  gen_device="cpu", chunk_rows: int = 1 << 20) -> torch.Tensor:
    """Fill (or allocate on CPU) the full [N, row_bytes] uint8 table."""
    if out is None:
        out = torch.empty((num_nodes, row_bytes), dtype=torch.uint8)
    for s in range(0, num_nodes, chunk_rows):
        e = min(num_nodes, s + chunk_rows)
        out[s:e].copy_(feature_rows(s, e, row_bytes, seed, gen_device), non_blocking=False)
    return out


def train_nodes(num_nodes: int, frac: float, seed: int = TRAIN_SEED, device="cpu") -> torch.Tensor:
    T = max(1, int(round(num_nodes * frac)))
    key = splitmix64(torch.arange(num_nodes, dtype=torch.int64, device=device) ^ _mix_seed(seed, 21))
    return torch.argsort(key)[:T].to(torch.int32)


def epoch_order(train: torch.Tensor, epoch: int = 0, seed: int = TRAIN_SEED) -> torch.Tensor:
    key = splitmix64(torch.arange(len(train), dtype=torch.int64, device=train.device) ^ _mix_seed(seed, 100 + epoch))
    return train[torch.argsort(key)]


def batch_seeds(order: torch.Tensor, batch_size: int, b: int) -> torch.Tensor:
    n = len(order)
    nb = max(1, n // batch_size)
    b = b % nb
    return order[b * batch_size:(b + 1) * batch_size]


def graph_hash(indptr: torch.Tensor, indices: torch.Tensor) -> str:
    h = hashlib.sha256()
    h.update(indptr.cpu().numpy().tobytes())
    ind = indices.cpu().numpy()
    step = 1 << 26
    for s in range(0, len(ind), step):
        h.update(ind[s:s + step].tobytes())
    return h.hexdigest()[:16]


def segment(num_batches: int, rank: int, world: int) -> range:
    """Contiguous batch segment of GPU `rank` (the paper's 'segments')."""
    lo = num_batches * rank // world
    hi = num_batches * (rank + 1) // world
    return range(lo, hi)


# ---------------------------------------------------------------- f4: train stage inputs
# (3-layer GraphSAGE, hidden 256.)  Values are multiples of
# 2^-23 in [-1, 1) (exact in fp32 and fp64), drawn with SplitMix64 like everything above.
LABEL_SEED = 5
WEIGHT_SEED = 6


def _unit(key: torch.Tensor) -> torch.Tensor:
    """SplitMix64(key) -> float64 in [-1, 1), a multiple of 2^-23."""
    u = _lsr(splitmix64(key), 40).to(torch.float64)          # 24 random bits
    return u / float(1 << 23) - 1.0


def numeric_feature_rows(v0: int, v1: int, dim: int, seed: int = FEATURE_SEED, device="cpu") -> torch.Tensor:
    """fp32 rows v0..v1-1 [v1-v0, dim] in [-1, 1) (the train stage needs finite features;
    the extraction path copies bytes and does not care)."""
    v = torch.arange(v0, v1, dtype=torch.int64, device=device)
    c = torch.arange(dim, dtype=torch.int64, device=device)
    return _unit((v[:, None] * dim + c[None, :]) ^ _mix_seed(seed, 31)).to(torch.float32)


def numeric_feature_table(num_nodes: int, dim: int, seed: int = FEATURE_SEED, out: torch.Tensor | None = None,
                          gen_device="cpu", chunk_rows: int = 1 << 20) -> torch.Tensor:
    """The [N, dim*4] uint8 host table holding numeric_feature_rows (fp32 little endian)."""
    if out is None:
        out = torch.empty((num_nodes, dim * 4), dtype=torch.uint8)
    for s in range(0, num_nodes, chunk_rows):
        e = min(num_nodes, s + chunk_rows)
        out[s:e].copy_(numeric_feature_rows(s, e, dim, seed, gen_device).view(torch.uint8), non_blocking=False)
    return out


def labels(nodes: torch.Tensor, num_classes: int, seed: int = LABEL_SEED) -> torch.Tensor:
    """Synthetic class label of each node (the paper trains Friendster on random labels)."""
    key = nodes.to(torch.int64) ^ _mix_seed(seed, 41)
    return (_lsr(splitmix64(key), 33) % num_classes).to(torch.int32)


def sage_init(dims, seed: int = WEIGHT_SEED):
    """Initial parameters of an L-layer SAGE model with layer widths dims[0..L]: per layer
    W [2*d_in, d_out] (rows 0..d_in-1 multiply the node's own features, rows d_in.. the
    neighbour mean) uniform in +-1/sqrt(2 d_in), and b [d_out] uniform in +-0.1; float32
    numpy arrays."""
    out = []
    for l in range(len(dims) - 1):
        di, do = dims[l], dims[l + 1]
        k = torch.arange(2 * di * do, dtype=torch.int64) ^ _mix_seed(seed, 50 + l)
        W = (_unit(k) / np.sqrt(2 * di)).to(torch.float32).reshape(2 * di, do).numpy()
        kb = torch.arange(do, dtype=torch.int64) ^ _mix_seed(seed, 80 + l)
        b = (_unit(kb) * 0.1).to(torch.float32).numpy()
        out.append((W, b))
    return out
