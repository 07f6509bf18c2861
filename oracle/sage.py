"""CPU oracle of the f4 train stage: one GraphSAGE training step on the sampled blocks.

TEST INFRASTRUCTURE ONLY (like oracle.py): imported by tests/ and bench.py's cpu legs,
never by the product package.  Plain numpy float64, one step of the definition at a time.

What it computes ("GraphSAGE ... three layers ... hidden
dimension 256", P:140 gradients averaged across subprocesses by PyTorch DDP):
  * blocks: hop h of gd_sample gives dst = n_id[0:n_{h-1}], src = n_id[0:n_h], CSR
    (rowptr_h, col_h) with col in local src ids; dst i is src row i (the frontier is
    cumulative, so dst nodes are a prefix of the src nodes).
  * layer j (j = 0..L-1) runs on hop h = L - j (outermost block first, as PyG consumes
    NeighborSampler blocks), widths d_in -> d_out (the SAGEConv mean rule of Hamilton et
    al. with root weight; the paper uses PyG's implementation):
        a_i   = [ x_i , mean_{e in row i} x_{col[e]} ]        (mean of an empty row = 0)
        z_i   = a_i W + b,  W: [2 d_in, d_out]
        x'_i  = relu(z_i) for j < L-1; the last layer's z are the logits
  * loss = mean over the n_0 seeds of softmax cross entropy (logits_i, label_i).
  * backward: the chain rule of the above, written out below; SGD: p -= lr * g.
Pinned in tests/test_oracle_sage.py by central finite differences (every parameter
tensor), the closed form loss = ln C at zero weights and biases, and a hand-computed
one-node two-neighbour layer.
"""
from __future__ import annotations

import numpy as np


def layer_hops(L: int):
    """Hop of the block layer j consumes (outermost first)."""
    return [L - j for j in range(L)]


def aggregate(x: np.ndarray, rowptr: np.ndarray, col: np.ndarray, n_dst: int) -> np.ndarray:
    """a = [x_dst | mean of neighbours] for the n_dst rows of one block (float64)."""
    d = x.shape[1]
    a = np.zeros((n_dst, 2 * d), dtype=np.float64)
    a[:, :d] = x[:n_dst]
    for i in range(n_dst):
        lo, hi = int(rowptr[i]), int(rowptr[i + 1])
        if hi > lo:
            a[i, d:] = x[col[lo:hi]].mean(axis=0)
    return a


def forward(params, feats: np.ndarray, blocks, labels: np.ndarray):
    """params: [(W, b)] per layer; feats [n_L, d_0]; blocks[h-1] = (rowptr_h, col_h) for hop
    h = 1..L; labels [n_0].  Returns (loss, cache)."""
    L = len(params)
    x = np.asarray(feats, dtype=np.float64)
    cache = []
    for j, h in enumerate(layer_hops(L)):
        rowptr, col = blocks[h - 1]
        n_dst = len(rowptr) - 1
        W, b = (np.asarray(p, dtype=np.float64) for p in params[j])
        a = aggregate(x, rowptr, col, n_dst)
        z = a @ W + b
        cache.append((x, a, z, rowptr, col))
        x = np.maximum(z, 0.0) if j < L - 1 else z
    logits = x
    m = logits.max(axis=1, keepdims=True)
    lse = m[:, 0] + np.log(np.exp(logits - m).sum(axis=1))
    n0 = logits.shape[0]
    loss = float(np.mean(lse - logits[np.arange(n0), labels]))
    return loss, (cache, logits)


def backward(params, cache_all, labels: np.ndarray, return_dz: bool = False):
    """Gradients [(dW, db)] of the mean loss (and, if asked, d loss / d z of every layer)."""
    cache, logits = cache_all
    L = len(params)
    n0 = logits.shape[0]
    p = np.exp(logits - logits.max(axis=1, keepdims=True))
    p /= p.sum(axis=1, keepdims=True)
    dz = p.copy()
    dz[np.arange(n0), labels] -= 1.0
    dz /= n0                                           # d loss / d logits
    grads = [None] * L
    dzs = [None] * L
    for j in range(L - 1, -1, -1):
        x, a, z, rowptr, col = cache[j]
        W = np.asarray(params[j][0], dtype=np.float64)
        if j < L - 1:
            dz = dz * (z > 0)                          # relu'
        dzs[j] = dz
        grads[j] = (a.T @ dz, dz.sum(axis=0))
        if j == 0:
            break
        da = dz @ W.T                                  # [n_dst, 2 d_in]
        d = x.shape[1]
        dx = np.zeros_like(x)
        n_dst = a.shape[0]
        dx[:n_dst] += da[:, :d]                        # own features
        for i in range(n_dst):                         # mean over the row's neighbours
            lo, hi = int(rowptr[i]), int(rowptr[i + 1])
            if hi > lo:
                np.add.at(dx, col[lo:hi], da[i, d:] / (hi - lo))
        dz = dx                                        # d loss / d (previous layer output)
    return (grads, dzs) if return_dz else grads


def sgd(params, grads, lr: float):
    return [(np.asarray(W, np.float64) - lr * dW, np.asarray(b, np.float64) - lr * db)
            for (W, b), (dW, db) in zip(params, grads)]


def train_step(params, feats, blocks, labels, lr: float | None = None):
    loss, cache = forward(params, feats, blocks, labels)
    grads = backward(params, cache, labels)
    new = sgd(params, grads, lr) if lr is not None else None
    return loss, grads, new
