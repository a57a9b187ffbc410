"""Pins of the fp64 oracle against things other than itself (CPU only).

Each test fixes part of oracle/gcn.py by an independent route:
library routines (scipy.sparse, torch.autograd, torch cross-entropy,
torch.optim.Adam), central finite differences, associativity,
and closed forms (DESIGN.md pins P1–P4).
"""
import math

import numpy as np
import pytest
import scipy.sparse as sp
import torch

import synth
from oracle import gcn


def to_scipy(g):
    return sp.csr_matrix((g.val.astype(np.float64), g.col, g.rowptr), shape=(g.n, g.n))


@pytest.fixture(scope="module")
def dgraph():
    return synth.random_directed(97, 900, seed=3, empty_rows=5)


def test_spmm_matches_scipy(dgraph):
    rng = np.random.default_rng(0)
    X = rng.standard_normal((dgraph.n, 13))
    A = to_scipy(dgraph)
    np.testing.assert_allclose(gcn.spmm(dgraph, X), A @ X, rtol=0, atol=1e-12)
    np.testing.assert_allclose(gcn.spmm_t(dgraph, X), A.T @ X, rtol=0, atol=1e-12)
    rows = np.array([0, 5, 96, 17, 17])
    np.testing.assert_allclose(gcn.spmm_rows(dgraph, X.astype(np.float32), rows),
                               (A @ X.astype(np.float32).astype(np.float64))[rows], atol=1e-12)


def test_spmm_rows_leading_dim(dgraph):
    rng = np.random.default_rng(1)
    big = rng.standard_normal((dgraph.n, 20)).astype(np.float32)
    view = big[:, 3:11]      # ld = 20, f = 8
    A = to_scipy(dgraph)
    rows = np.arange(dgraph.n)
    np.testing.assert_allclose(gcn.spmm_rows(dgraph, view, rows), A @ view.astype(np.float64), atol=1e-12)


def test_empty_rows_give_zero(dgraph):
    X = np.ones((dgraph.n, 4))
    Y = gcn.spmm(dgraph, X)
    empty = np.diff(dgraph.rowptr) == 0
    assert empty.sum() >= 5
    assert np.all(Y[empty] == 0)


def test_associativity_both_orders():
    """(AᵀH)W == Aᵀ(HW) on a non-symmetric graph."""
    g = synth.random_directed(64, 500, seed=9)
    rng = np.random.default_rng(2)
    H = rng.standard_normal((64, 11))
    W = rng.standard_normal((11, 5))
    zs = gcn.layer_forward(g, H, W, "S")
    zd = gcn.layer_forward(g, H, W, "D")
    assert gcn.max_rel_err(zs, zd) < 1e-13


def _torch_model(g, H0, Ws, labels, mask):
    """Independent torch fp64 forward with dense Â; gradients by autograd."""
    A = torch.tensor(to_scipy(g).toarray())
    H = torch.tensor(np.asarray(H0, np.float64), requires_grad=True)
    Wt = [torch.tensor(np.asarray(W, np.float64), requires_grad=True) for W in Ws]
    x = H
    for l, W in enumerate(Wt):
        x = A.T @ x @ W
        if l < len(Wt) - 1:
            x = torch.relu(x)
    m = torch.tensor(mask.astype(bool))
    loss = torch.nn.functional.cross_entropy(x[m], torch.tensor(labels.astype(np.int64))[m])
    loss.backward()
    return float(loss.detach()), [W.grad.numpy() for W in Wt], H.grad.numpy()


@pytest.mark.parametrize("directed", [False, True])
def test_gradients_match_autograd(directed):
    n, f = 60, (9, 7, 5)
    if directed:
        g = synth.random_directed(n, 400, seed=4)
    else:
        g = synth.rmat(n, 150, seed=4)
    H0 = synth.features(n, f[0])
    Ws = synth.weights(f)
    y = synth.labels(n, f[-1])
    m = synth.train_mask(n, 0.7, seed=8)
    res = gcn.epoch(g, H0, Ws, y, m)
    tl, tW, tH = _torch_model(g, H0, Ws, y, m)
    assert abs(res.loss - tl) <= 1e-12 * abs(tl)
    for l in (1, 2):
        assert gcn.max_rel_err(res.Y[l], tW[l - 1]) < 1e-11
    assert gcn.max_rel_err(res.G[0], tH) < 1e-11


def test_finite_differences_three_layers():
    """Central differences on W^l and H^0 entries (pin P3)."""
    n, f = 40, (6, 5, 4, 3)
    g = synth.rmat(n, 120, seed=12)
    H0 = synth.features(n, f[0]).astype(np.float64)
    Ws = [w.astype(np.float64) for w in synth.weights(f)]
    y = synth.labels(n, f[-1])
    m = synth.train_mask(n)
    res = gcn.epoch(g, H0, Ws, y, m)
    rng = np.random.default_rng(5)

    def loss_of(Ws_, H0_):
        return gcn.forward(g, H0_, Ws_, y, m)

    checked = 0
    for l in range(1, len(f)):
        for _ in range(12):
            i, j = rng.integers(0, f[l - 1]), rng.integers(0, f[l])
            h = 1e-6 * max(1.0, abs(Ws[l - 1][i, j]))
            Wp = [w.copy() for w in Ws]
            Wm = [w.copy() for w in Ws]
            Wp[l - 1][i, j] += h
            Wm[l - 1][i, j] -= h
            rp, rm = loss_of(Wp, H0), loss_of(Wm, H0)
            # discard probes that flip a ReLU (kink)
            if any(np.any(np.sign(rp.Z[k]) != np.sign(rm.Z[k])) for k in range(1, len(f) - 1)):
                continue
            fd = (rp.loss - rm.loss) / (2 * h)
            assert abs(fd - res.Y[l][i, j]) <= 1e-6 * max(1e-3, abs(fd))
            checked += 1
    for _ in range(12):
        i, j = rng.integers(0, n), rng.integers(0, f[0])
        h = 1e-6
        Hp, Hm = H0.copy(), H0.copy()
        Hp[i, j] += h
        Hm[i, j] -= h
        rp, rm = loss_of(Ws, Hp), loss_of(Ws, Hm)
        if any(np.any(np.sign(rp.Z[k]) != np.sign(rm.Z[k])) for k in range(1, len(f) - 1)):
            continue
        fd = (rp.loss - rm.loss) / (2 * h)
        assert abs(fd - res.G[0][i, j]) <= 1e-6 * max(1e-3, abs(fd))
        checked += 1
    assert checked >= 30


@pytest.mark.parametrize("C", [7, 41, 47, 172])
def test_zero_last_weights_give_ln_C(C):
    """W^L = 0 → logits 0 → ℓ = ln C exactly, G^L = (1/C − onehot)·m/n_train (pin P4-ii)."""
    n, f = 50, (8, 6, C)
    g = synth.rmat(n, 100, seed=1)
    H0 = synth.features(n, f[0])
    Ws = synth.weights(f)
    Ws[-1] = np.zeros_like(Ws[-1])
    y = synth.labels(n, C)
    m = synth.train_mask(n, 0.5, seed=3)
    res = gcn.epoch(g, H0, Ws, y, m)
    assert abs(res.loss - math.log(C)) < 1e-14
    GL = np.full((n, C), 1.0 / C)
    GL[np.arange(n), y] -= 1.0
    GL *= m[:, None] / m.sum()
    np.testing.assert_allclose(res.G[2], GL, atol=1e-16)


def test_identity_graph_is_mlp():
    """Â = I: the GCN is a plain MLP (pin P4-i), compared with torch.nn.Linear layers."""
    n, f = 30, (5, 4, 3)
    g = synth.identity_graph(n)
    H0 = synth.features(n, f[0])
    Ws = synth.weights(f)
    y = synth.labels(n, f[-1])
    m = synth.train_mask(n)
    res = gcn.forward(g, H0, Ws, y, m)
    lin = [torch.nn.Linear(f[i], f[i + 1], bias=False).double() for i in range(2)]
    with torch.no_grad():
        for i in range(2):
            lin[i].weight.copy_(torch.tensor(Ws[i].astype(np.float64).T))
        out = lin[1](torch.relu(lin[0](torch.tensor(H0.astype(np.float64)))))
    np.testing.assert_allclose(res.Z[2], out.numpy(), atol=1e-13)


def test_complete_graph_is_column_mean():
    """K_n with self loops, symmetric normalization: Â = J/n, rows of ÂᵀH = column mean (P4-iii)."""
    n = 17
    g = synth.complete_graph(n)
    H = synth.features(n, 6).astype(np.float64)
    T = gcn.spmm_t(g, H)
    np.testing.assert_allclose(T, np.tile(H.mean(axis=0), (n, 1)), atol=1e-7)  # fp32 values of 1/n


def test_star_graph_hub_row():
    """Star: the hub row aggregates every vertex (pin P4-v)."""
    n = 200
    g = synth.star_graph(n)
    H = np.ones((n, 3))
    T = gcn.spmm(g, H)
    d = np.diff(g.rowptr).astype(np.float64)
    assert d[0] == n
    # hub: 1/n (self) + sum_{leaves} 1/sqrt(n*2)
    expect = 1.0 / n + (n - 1) / math.sqrt(2.0 * n)
    assert abs(T[0, 0] - expect) < 1e-6
    # leaf: 1/sqrt(2n) (hub) + 1/2 (self)
    assert abs(T[5, 0] - (1.0 / math.sqrt(2.0 * n) + 0.5)) < 1e-6


def test_loss_matches_torch_cross_entropy():
    rng = np.random.default_rng(7)
    Z = rng.standard_normal((40, 11)) * 5
    y = rng.integers(0, 11, size=40)
    m = rng.random(40) < 0.6
    loss, G = gcn.softmax_xent(Z, y, m)
    Zt = torch.tensor(Z, requires_grad=True)
    lt = torch.nn.functional.cross_entropy(Zt[torch.tensor(m)], torch.tensor(y)[torch.tensor(m)])
    lt.backward()
    assert abs(loss - float(lt)) < 1e-13
    np.testing.assert_allclose(G, Zt.grad.numpy(), atol=1e-15)


def test_adam_matches_torch():
    rng = np.random.default_rng(8)
    p0 = rng.standard_normal((6, 5))
    grads = [rng.standard_normal((6, 5)) for _ in range(4)]
    pt = torch.tensor(p0.copy(), requires_grad=True)
    opt = torch.optim.Adam([pt], lr=0.01)
    p, m, v = p0.copy(), np.zeros_like(p0), np.zeros_like(p0)
    for t, gr in enumerate(grads, start=1):
        opt.zero_grad()
        pt.grad = torch.tensor(gr)
        opt.step()
        p, m, v = gcn.adam(p, gr, m, v, t)
    np.testing.assert_allclose(p, pt.detach().numpy(), atol=1e-13)


def test_symmetric_rmat_properties():
    """Generator conventions the oracle relies on: symmetric, one self loop per vertex, nnz."""
    g = synth.rmat(500, 3000, seed=21)
    A = to_scipy(g)
    assert g.nnz == 2 * 3000 + 500
    assert abs(A - A.T).max() == 0
    assert np.all(A.diagonal() > 0)
    assert np.all(np.diff(g.col[g.rowptr[0]:g.rowptr[1]]) > 0)


def test_max_rel_err_catches_perturbations():
    """Negative pins of the parity comparator (reading R26): a one-element 2e-4
    perturbation fails the 1e-4 gate; zeros, empty inputs, shape mismatches and
    non-finite values are handled explicitly."""
    rng = np.random.default_rng(5)
    r = rng.standard_normal((300, 17))
    assert gcn.max_rel_err(r, r) == 0.0
    x = r.copy()
    i, j = 123, 7
    x[i, j] += 2e-4 * np.abs(r).max()
    e = gcn.max_rel_err(x, r)
    assert e == pytest.approx(2e-4, rel=1e-9)
    assert not e < 1e-4
    x = r.copy()
    x[0, 0] += 0.9e-4 * np.abs(r).max()
    assert gcn.max_rel_err(x, r) < 1e-4
    # the error is normwise: a small element wrong by 100 % of itself passes only if tiny
    x = r.copy()
    k = np.unravel_index(np.argmin(np.abs(r)), r.shape)
    x[k] = 2 * r[k]
    assert gcn.max_rel_err(x, r) == pytest.approx(abs(r[k]) / np.abs(r).max())
    # zeros / empty / non-finite / shapes
    z = np.zeros((4, 3))
    assert gcn.max_rel_err(z, z) == 0.0
    assert gcn.max_rel_err(z + 1e-3, z) == pytest.approx(1e-3)
    assert gcn.max_rel_err(np.zeros((0, 5)), np.zeros((0, 5))) == 0.0
    bad = r.copy()
    bad[3, 3] = np.nan
    assert gcn.max_rel_err(bad, r) == float("inf")
    bad[3, 3] = np.inf
    assert not gcn.max_rel_err(bad, r) < 1e-4
    with pytest.raises(ValueError):
        gcn.max_rel_err(r[:, :1], r)          # no broadcasting
    with pytest.raises(ValueError):
        gcn.max_rel_err(r.T, r)


def test_relu_tiebreak_band():
    """tests/parity.py (reading R30): disagreements inside the band are taken
    from the kernel, one outside the band fails, and a tie-broken oracle
    backward equals the plain one when there is nothing to break."""
    from parity import relu_tiebreak
    n, f = 50, (6, 5, 4, 3)
    g = synth.rmat(n, 150, seed=2)
    H0 = synth.features(n, f[0])
    Ws = synth.weights(f)
    y = synth.labels(n, f[-1])
    m = synth.train_mask(n)
    a = gcn.epoch(g, H0, Ws, y, m)
    ref = gcn.forward(g, H0, Ws, y, m)
    Hk = [np.maximum(ref.Z[1], 0), np.maximum(ref.Z[2], 0)]
    assert relu_tiebreak(ref, Hk) == (0, 0.0)
    gcn.backward(g, ref, Ws)
    for l in (1, 2, 3):
        assert np.array_equal(a.Y[l], ref.Y[l])
    # in-band flip: the kernel says positive where the oracle's Z is a tiny negative
    ref = gcn.forward(g, H0, Ws, y, m)
    Z1 = ref.Z[1]
    zmax = np.abs(Z1).max()
    neg = np.argwhere(Z1 < 0)[0]
    Z1[tuple(neg)] = -0.5 * 2.0 ** -16 * zmax
    Hk = [np.maximum(Z1, 0), np.maximum(ref.Z[2], 0)]
    Hk[0][tuple(neg)] = 1e-9
    nd, worst = relu_tiebreak(ref, Hk)
    assert nd == 1 and worst == pytest.approx(0.5 * 2.0 ** -16)
    assert ref.Z[1][tuple(neg)] > 0
    # out-of-band flip is rejected
    ref = gcn.forward(g, H0, Ws, y, m)
    Z1 = ref.Z[1]
    pos = np.argwhere(Z1 > 1e-3 * np.abs(Z1).max())[0]
    Hk = [np.maximum(Z1, 0), np.maximum(ref.Z[2], 0)]
    Hk[0][tuple(pos)] = 0.0
    with pytest.raises(AssertionError):
        relu_tiebreak(ref, Hk)


def _biases(f, seed=21):
    rng = np.random.default_rng(seed)
    return [rng.standard_normal(f[l]) * 0.3 for l in range(1, len(f))]


def test_bias_identity_graph_is_mlp_with_bias():
    """Â = I with biases (reading R8): torch.nn.Linear(bias=True) layers give
    the logits, and autograd gives dW and db (pin P4-i with bias)."""
    n, f = 30, (5, 4, 3)
    g = synth.identity_graph(n)
    H0 = synth.features(n, f[0])
    Ws = synth.weights(f)
    bs = _biases(f)
    y = synth.labels(n, f[-1])
    m = synth.train_mask(n)
    res = gcn.epoch(g, H0, Ws, y, m, bs)
    lin = [torch.nn.Linear(f[i], f[i + 1], bias=True).double() for i in range(2)]
    with torch.no_grad():
        for i in range(2):
            lin[i].weight.copy_(torch.tensor(Ws[i].astype(np.float64).T))
            lin[i].bias.copy_(torch.tensor(bs[i]))
    out = lin[1](torch.relu(lin[0](torch.tensor(H0.astype(np.float64)))))
    mt = torch.tensor(m.astype(bool))
    loss = torch.nn.functional.cross_entropy(out[mt], torch.tensor(y, dtype=torch.long)[mt])
    loss.backward()
    np.testing.assert_allclose(res.Z[2], out.detach().numpy(), atol=1e-13)
    assert abs(res.loss - float(loss)) <= 1e-12 * abs(float(loss))
    for l in (1, 2):
        np.testing.assert_allclose(res.db[l], lin[l - 1].bias.grad.numpy(), atol=1e-13)
        np.testing.assert_allclose(res.Y[l], lin[l - 1].weight.grad.numpy().T, atol=1e-13)


def test_bias_finite_differences_three_layers():
    """Central differences on b^l entries of a 3-layer GCN on an R-MAT graph
    (pin P3 for db^l = 1ᵀ G^l); also checks dW with biases present."""
    n, f = 40, (6, 5, 4, 3)
    g = synth.rmat(n, 120, seed=12)
    H0 = synth.features(n, f[0]).astype(np.float64)
    Ws = [w.astype(np.float64) for w in synth.weights(f)]
    bs = _biases(f)
    y = synth.labels(n, f[-1])
    m = synth.train_mask(n)
    res = gcn.epoch(g, H0, Ws, y, m, bs)
    rng = np.random.default_rng(9)
    checked = 0
    for l in range(1, len(f)):
        for j in range(f[l]):
            h = 1e-6
            bp = [b.copy() for b in bs]
            bm = [b.copy() for b in bs]
            bp[l - 1][j] += h
            bm[l - 1][j] -= h
            rp, rm = gcn.forward(g, H0, Ws, y, m, bp), gcn.forward(g, H0, Ws, y, m, bm)
            if any(np.any(np.sign(rp.Z[k]) != np.sign(rm.Z[k])) for k in range(1, len(f) - 1)):
                continue
            fd = (rp.loss - rm.loss) / (2 * h)
            assert abs(fd - res.db[l][j]) <= 1e-6 * max(1e-3, abs(fd)), (l, j, fd, res.db[l][j])
            checked += 1
        i, j = rng.integers(0, f[l - 1]), rng.integers(0, f[l])
        h = 1e-6 * max(1.0, abs(Ws[l - 1][i, j]))
        Wp = [w.copy() for w in Ws]
        Wm = [w.copy() for w in Ws]
        Wp[l - 1][i, j] += h
        Wm[l - 1][i, j] -= h
        rp, rm = gcn.forward(g, H0, Wp, y, m, bs), gcn.forward(g, H0, Wm, y, m, bs)
        fd = (rp.loss - rm.loss) / (2 * h)
        assert abs(fd - res.Y[l][i, j]) <= 1e-6 * max(1e-3, abs(fd))
    assert checked >= 8
