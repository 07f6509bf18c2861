"""Pins of the f4 train-stage oracle (oracle/sage.py) against things other than itself:
central finite differences of the loss (every parameter entry of a small model), closed
forms at zero parameters, and a hand-computed layer."""
import numpy as np
import pytest

import synth
from oracle import oracle as O
from oracle import sage as S


def small_problem(dims=(6, 5, 4, 3), fan=(3, 2, 2), N=300, E=1500, B=7, seed=3):
    indptr, indices = synth.chung_lu_csr(N, E, seed=seed)
    order = synth.epoch_order(synth.train_nodes(N, 0.2))
    seeds = order[:B].numpy()
    res = O.sample(indptr.numpy(), indices.numpy(), seeds, list(fan), 3, 0)
    blocks = [(res.rowptr[k], res.col[k]) for k in range(len(fan))]
    feats = synth.numeric_feature_rows(0, N, dims[0]).numpy().astype(np.float64)[res.n_id]
    labels = synth.labels(torch_tensor(res.n_id[:B]), dims[-1]).numpy()
    params = [(W.astype(np.float64), b.astype(np.float64)) for W, b in synth.sage_init(list(dims))]
    return params, feats, blocks, labels


def torch_tensor(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a))


def test_gradients_match_central_differences():
    params, feats, blocks, labels = small_problem()
    loss, cache = S.forward(params, feats, blocks, labels)
    grads = S.backward(params, cache, labels)
    eps = 1e-6
    for j, (W, b) in enumerate(params):
        for arr, g in ((W, grads[j][0]), (b, grads[j][1])):
            num = np.zeros_like(arr)
            it = np.nditer(arr, flags=["multi_index"])
            for _ in it:
                idx = it.multi_index
                old = arr[idx]
                arr[idx] = old + eps
                lp, _ = S.forward(params, feats, blocks, labels)
                arr[idx] = old - eps
                lm, _ = S.forward(params, feats, blocks, labels)
                arr[idx] = old
                num[idx] = (lp - lm) / (2 * eps)
            assert np.allclose(g, num, rtol=1e-5, atol=1e-8), (j, np.abs(g - num).max())


def test_zero_parameters_closed_form():
    """All-zero W, b: every logit is 0, loss = ln C; d loss/d b_last = mean(1/C - onehot)."""
    params, feats, blocks, labels = small_problem()
    C = params[-1][1].shape[0]
    zero = [(np.zeros_like(W), np.zeros_like(b)) for W, b in params]
    loss, cache = S.forward(zero, feats, blocks, labels)
    assert abs(loss - np.log(C)) < 1e-12
    grads = S.backward(zero, cache, labels)
    n0 = len(labels)
    expect = np.full(C, 1.0 / C) - np.bincount(labels, minlength=C) / n0
    assert np.allclose(grads[-1][1], expect, atol=1e-15)
    for dW, db in grads[:-1]:                     # relu'(0) = 0 blocks everything below
        assert not dW.any() and not db.any()


def test_hand_computed_layer():
    """One layer, dst node 0 with neighbours 1 and 2 (and 2 again: multi-edge)."""
    x = np.array([[1.0, 2.0], [3.0, -1.0], [5.0, 7.0]])
    rowptr = np.array([0, 3])
    col = np.array([1, 2, 2])
    a = S.aggregate(x, rowptr, col, 1)
    assert np.array_equal(a, [[1.0, 2.0, 13.0 / 3.0, 13.0 / 3.0]])
    W = np.arange(8.0).reshape(4, 2)
    b = np.array([0.5, -0.5])
    loss, (cache, logits) = S.forward([(W, b)], x, [(rowptr, col)], np.array([1]))
    z = np.array([1 * 0 + 2 * 2 + 13 / 3 * 4 + 13 / 3 * 6 + 0.5, 1 * 1 + 2 * 3 + 13 / 3 * 5 + 13 / 3 * 7 - 0.5])
    assert np.allclose(logits[0], z)
    assert abs(loss - (np.log(np.exp(z).sum()) - z[1])) < 1e-12


def test_empty_rows_and_layer_hops():
    assert S.layer_hops(3) == [3, 2, 1]
    x = np.ones((3, 2))
    a = S.aggregate(x, np.array([0, 0, 1]), np.array([2]), 2)
    assert np.array_equal(a, [[1, 1, 0, 0], [1, 1, 1, 1]])


def test_sgd_step_decreases_loss():
    params, feats, blocks, labels = small_problem()
    loss0, grads, new = S.train_step(params, feats, blocks, labels, lr=0.5)
    loss1, _ = S.forward(new, feats, blocks, labels)
    assert loss1 < loss0
