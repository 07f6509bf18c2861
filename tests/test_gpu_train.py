"""f4 GPU parity: gd_sage_step (sm_100a aggregation kernels + tcgen05 bf16 GEMMs) against the
float64 oracle (oracle/sage.py) on blocks and rows produced by the CUDA sample + extract
path (themselves bit-exact with the oracle, tests/test_gpu_parity.py).

Tolerances: the GPU rounds both GEMM operands to bf16 (unit roundoff
u = 2^-9 each) and accumulates in fp32, so an output entry obeys
|z_gpu - z| <= (2u + u^2 + K 2^-24) (|a| |W|) <= 2^-7 (|a| |W|) for K <= 2^15; the
aggregation rounds once to bf16: |a_gpu - a| <= 2^-8 |a| + 1e-6.  A gradient of layer j is
the end of a chain of at most 2L GEMMs (forward through every layer, backward down to j), each
adding <= 2^-7 relative to the magnitudes |A||B| it multiplies, so
||dW_gpu - dW|| <= 2^-4 || |a|^T |dz| || and ||db_gpu - db|| <= 2^-4 || sum_i |dz_i| || (6 x 2^-7
< 2^-4; the magnitudes, not the values, bound the error: sums of gradients cancel).  The bound
is normwise, not entrywise: where a pre-activation lies within rounding of 0 the two sides can
take different relu branches (a decision made in different precisions), which moves single
entries by up to their own size.  The loss is within 2e-2 relative."""
import numpy as np
import pytest
import torch

import synth
from oracle import oracle as O
from oracle import sage as S

pytestmark = pytest.mark.gpu

DIMS = [32, 64, 64, 16]
FAN = [5, 4, 3]


@pytest.fixture(scope="module")
def gd():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_icpp_jiangj024_b200 as gd
    from paper_conf_icpp_jiangj024_b200 import train
    return gd, train


@pytest.fixture(scope="module")
def problem(gd):
    gdm, train = gd
    N, E, B = 20_000, 200_000, 64
    indptr, indices = synth.chung_lu_csr(N, E, seed=17)
    g = gdm.Graph(indptr, indices)
    table = synth.numeric_feature_table(N, DIMS[0])
    order = synth.epoch_order(synth.train_nodes(N, 0.2))
    nm, _ = g.bounds(B, FAN)
    buf = gdm.FeatureBuffer(table, N, 2, nm[-1], preload=True)
    return dict(gd=gdm, train=train, g=g, buf=buf, table=table, order=order, B=B, nm=nm,
                ip=indptr.numpy(), ix=indices.numpy(), N=N)


def run_batch(P, b, model=None, steps=0, lr=0.0):
    gdm, g, buf = P["gd"], P["g"], P["buf"]
    seeds = synth.batch_seeds(P["order"], P["B"], b)
    res = g.sample(seeds.cuda(), FAN, 3, b)
    out, _, done = buf.extract(res.n_id, res.num_nodes_dev, res.max_nodes)
    torch.cuda.current_stream().wait_event(done)
    buf.release(res.n_id, res.num_nodes_dev, res.max_nodes)   # preload: rows stay resident
    labels = synth.labels(seeds, DIMS[-1]).cuda()
    return res, out, labels, seeds


def oracle_blocks(P, seeds, b):
    ref = O.sample(P["ip"], P["ix"], seeds.numpy(), FAN, 3, b)
    blocks = [(ref.rowptr[k], ref.col[k]) for k in range(len(FAN))]
    feats = synth.numeric_feature_rows(0, P["N"], DIMS[0]).numpy().astype(np.float64)[ref.n_id]
    return ref, blocks, feats


def rel(a, b):
    return float(np.linalg.norm(a - b) / max(1e-30, np.linalg.norm(b)))


def cos(a, b):
    a, b = a.ravel(), b.ravel()
    return float(a @ b / max(1e-30, np.linalg.norm(a) * np.linalg.norm(b)))


def test_sage_step_parity(problem):
    P = problem
    params = synth.sage_init(DIMS)
    model = P["train"].SageModel(DIMS, params, P["nm"])
    for b in range(3):
        res, out, labels, seeds = run_batch(P, b)
        loss = model.step(res, out, labels)
        torch.cuda.synchronize()
        ref, blocks, feats = oracle_blocks(P, seeds, b)
        assert np.array_equal(res.to_host()["n_id"], ref.n_id)
        p64 = [(W.astype(np.float64), bb.astype(np.float64)) for W, bb in params]
        lab = synth.labels(seeds, DIMS[-1]).numpy()
        l_ref, cache = S.forward(p64, feats, blocks, lab)
        grads, dzs = S.backward(p64, cache, lab, return_dz=True)
        # layer 0 (outermost block): aggregation and pre-activation, entrywise bounds
        n_dst = len(blocks[len(FAN) - 1][0]) - 1
        a_ref = cache[0][0][1]
        z_ref = cache[0][0][2]
        a = model.get_activation(P["train"].GD_SAGE_A16, 0, P["nm"][len(FAN) - 1])
        assert np.all(np.abs(a[:n_dst] - a_ref) <= 2.0 ** -8 * np.abs(a_ref) + 1e-6)
        # hidden activations are stored as bf16 relu(z + b): one more rounding (2^-9 relative)
        # on top of the GEMM bound; relu is 1-Lipschitz
        hgt = model.get_activation(P["train"].GD_SAGE_H, 0, P["nm"][len(FAN) - 1])
        bound = 2.0 ** -7 * (np.abs(a_ref) @ np.abs(p64[0][0])) + 2.0 ** -8 * np.abs(z_ref) + 1e-5
        h_ref = np.maximum(z_ref, 0.0)
        assert np.all(np.abs(hgt[:n_dst] - h_ref) <= bound), np.abs(hgt[:n_dst] - h_ref).max()
        # end to end: loss and every gradient tensor
        assert abs(float(loss.item()) - l_ref) <= 2e-2 * abs(l_ref), (float(loss.item()), l_ref)
        for j in range(len(DIMS) - 1):
            dW, db = model.get(P["train"].GD_SAGE_DW, j), model.get(P["train"].GD_SAGE_DB, j)
            a_j, dz_j = cache[0][j][1], dzs[j]
            mags = {"dW": np.abs(a_j).T @ np.abs(dz_j), "db": np.abs(dz_j).sum(axis=0)}
            for got, want, name in ((dW, grads[j][0], "dW"), (db, grads[j][1], "db")):
                err = np.linalg.norm(got - want) / max(1e-30, np.linalg.norm(mags[name]))
                assert err <= 2.0 ** -4 and cos(got, want) >= 0.99, (b, j, name, err, cos(got, want))
    model.close()


def test_sgd_update_and_training_reduces_loss(problem):
    P = problem
    params = synth.sage_init(DIMS)
    model = P["train"].SageModel(DIMS, params, P["nm"])
    res, out, labels, seeds = run_batch(P, 5)
    loss0 = float(model.step(res, out, labels).item())
    W0 = model.get(P["train"].GD_SAGE_W, 1)
    g0 = model.get(P["train"].GD_SAGE_DW, 1)
    model.apply_sgd(0.5)
    torch.cuda.synchronize()
    W1 = model.get(P["train"].GD_SAGE_W, 1)
    want = (W0.astype(np.float64) - np.float64(np.float32(0.5)) * g0).astype(np.float32)   # one rounding (fma)
    assert np.max(np.abs(W1 - want) / np.maximum(np.spacing(np.abs(want)), 1e-45)) <= 1.0
    losses = [loss0]
    for _ in range(30):
        losses.append(float(model.step(res, out, labels).item()))
        model.apply_sgd(0.5)
    torch.cuda.synchronize()
    assert losses[-1] < 0.9 * losses[0], losses[::5]                       # full-batch SGD descends
    assert sum(b < a for a, b in zip(losses, losses[1:])) >= 27, losses
    model.close()


def test_sage_matches_oracle_sgd_trajectory(problem):
    """Three SGD steps on three batches: parameters track the oracle's float64 trajectory."""
    P = problem
    params = synth.sage_init(DIMS)
    model = P["train"].SageModel(DIMS, params, P["nm"])
    p64 = [(W.astype(np.float64), bb.astype(np.float64)) for W, bb in params]
    for b in range(3):
        res, out, labels, seeds = run_batch(P, 10 + b)
        model.step(res, out, labels)
        model.apply_sgd(0.1)
        ref, blocks, feats = oracle_blocks(P, seeds, 10 + b)
        _, _, p64 = S.train_step(p64, feats, blocks, synth.labels(seeds, DIMS[-1]).numpy(), lr=0.1)
    torch.cuda.synchronize()
    for j in range(len(DIMS) - 1):
        W = model.get(P["train"].GD_SAGE_W, j)
        assert rel(W, p64[j][0]) <= 1e-2, (j, rel(W, p64[j][0]))
    model.close()
