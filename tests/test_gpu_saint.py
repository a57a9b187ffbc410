"""GraphSAINT-RDM on the GPU (rdm.h rdm_saint_*) against the oracle.

Sampler + induced-subgraph build: bit-exact (indices, counts and the fp32
values, which both sides compute as (float)(1/sqrt((double) d_i d_j))).
Training on the subgraph: the GCN epoch gates of tests/test_gpu_gcn.py
against oracle.gcn.epoch on the oracle's own subgraph, one Adam step per
subgraph (L390), P = 1 and virtual P = 2, 4."""
import numpy as np
import pytest

import synth
from oracle import gcn as og
from oracle import saint as osaint
from parity import BAND_FP32, relu_tiebreak

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rdm():
    import paper_conf_ipps_kurtysps23_b200 as r
    return r


def _sub_np(s):
    return [t.cpu().numpy() for t in s.subgraph()]


@pytest.mark.parametrize("n,E,roots,h", [(2708, 5278, 300, 4), (20000, 200000, 1500, 4),
                                         (500, 4000, 40, 0), (300, 3000, 400, 7)])
def test_sampler_bit_exact(rdm, n, E, roots, h):
    g = synth.rmat(n, E, seed=2)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    s = rdm.Saint(ctx, roots, walk_len=h, seed=17)
    for it in (0, 1, 5):
        n_s, nnz_s = s.sample(it)
        nodes, rp, cs, vs = osaint.sample(g, roots, h, 17, it)
        assert (n_s, nnz_s) == (len(nodes), len(cs))
        gn, grp, gcs, gvs = _sub_np(s)
        assert np.array_equal(gn, nodes)
        assert np.array_equal(grp, rp)
        assert np.array_equal(gcs, cs)
        assert np.array_equal(gvs.view(np.uint32), vs.view(np.uint32))


def test_sampler_whole_graph_capacity(rdm):
    """roots·(h+1) ≥ N: capacity = N; a subgraph may contain every vertex."""
    g = synth.complete_graph(12)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    s = rdm.Saint(ctx, 200, walk_len=2, seed=3)
    n_s, nnz_s = s.sample(0)
    nodes, rp, cs, vs = osaint.sample(g, 200, 2, 3, 0)
    assert n_s == len(nodes) == 12 and nnz_s == 144
    gn, grp, gcs, gvs = _sub_np(s)
    assert np.array_equal(gvs.view(np.uint32), vs.view(np.uint32))


def _saint_run(rdm, g, H0, Ws, y, m, cfg, P, roots, h, seed, iters):
    import torch
    dev = torch.device("cuda:0")
    f = [Ws[0].shape[0]] + [w.shape[1] for w in Ws]
    ctx = rdm.Context(device=0) if P == 1 else rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    s = rdm.Saint(ctx, roots, walk_len=h, seed=seed)
    model = s.gcn(f, cfg)
    Hd = torch.from_numpy(H0).to(dev)
    yd = torch.from_numpy(y).to(dev)
    md = torch.from_numpy(m.astype(np.uint8)).to(dev)
    Wd = [torch.from_numpy(w.copy()).to(dev) for w in Ws]
    dW = [torch.zeros_like(w) for w in Wd]
    mo = [torch.zeros_like(w) for w in Wd]
    ve = [torch.zeros_like(w) for w in Wd]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    out = []
    for it in range(iters):
        s.sample(it)
        model.saint_input(Hd, yd, md)
        W_now = [w.cpu().numpy().copy() for w in Wd]
        model.forward(Wd, loss)
        model.backward(Wd, dW)
        ctx.sync()
        out.append((it, float(loss.item()), [d.cpu().numpy() for d in dW], W_now, model))
        # per-subgraph parity is checked by the caller before the update
        yield out[-1]
        ctx.adam_step(Wd, dW, mo, ve, it + 1)
    model.close()
    s.close()


def _full(rdm, model, which, layer, n, width, P):
    """The full n x width tensor from whichever layout is resident on the P ranks."""
    for layout in (rdm.ROW, rdm.COL):
        try:
            parts = [model.tensor_torch(which, layer, p, layout).cpu().numpy() for p in range(P)]
        except rdm.RdmError:
            continue
        full = np.zeros((n, width))
        for p, t in enumerate(parts):
            lo, hi, _ = rdm.partition(P, layout, n, width, p)
            if P == 1:
                full[:] = t[:, :width]
            elif layout == rdm.ROW:
                full[lo:hi] = t[:, :width]
            else:
                full[:, lo:hi] = t[:, :hi - lo]
        return full
    raise AssertionError(f"tensor {which}/{layer} not resident")


@pytest.mark.parametrize("P,cfg,core", [(1, 3, 0), (1, 10, 0), (2, 3, 0), (4, 10, 0), (4, 2, 0),
                                        (1, 3, 256), (2, 10, 384)])
def test_saint_gcn_matches_oracle(rdm, P, cfg, core, monkeypatch):
    """core > 0 forces a dense hub core of that size on every subgraph
    (RDM_SAINT_CORE_K): the device-built core + residual CSR path."""
    if core:
        monkeypatch.setenv("RDM_SAINT_CORE_K", str(core))
    n, f = 4000, (300, 64, 11)
    g = synth.rmat(n, 40000, seed=6)
    H0 = synth.features(n, f[0])
    Ws = synth.weights(f)
    y = synth.labels(n, f[-1])
    m = synth.train_mask(n, 0.7, seed=2)
    roots, h, seed = 250, 4, 99
    for it, loss, dW, W_now, model in _saint_run(rdm, g, H0, Ws, y, m, cfg, P, roots, h, seed, 3):
        nodes, rp, cs, vs = osaint.sample(g, roots, h, seed, it)
        sub = synth.CSR(len(nodes), rp, cs, vs)
        # forward H^l, then the oracle's backward with ReLU ties broken only in the band (R30)
        Hs = [_full(rdm, model, rdm.T_H, l, len(nodes), f[l], P) for l in range(1, len(Ws))]
        Zk = _full(rdm, model, rdm.T_Z, 0, len(nodes), f[-1], P)
        ref = og.forward(sub, H0[nodes], W_now, y[nodes], m[nodes])
        for l in range(1, len(Ws)):
            assert og.max_rel_err(Hs[l - 1], og.relu(ref.Z[l])) < 1e-4, (it, "H", l)
        assert og.max_rel_err(Zk, ref.Z[len(Ws)]) < 1e-4, (it, "logits")
        relu_tiebreak(ref, Hs, BAND_FP32)
        og.backward(sub, ref, W_now)
        assert abs(loss - ref.loss) <= 1e-5 * abs(ref.loss), (it, loss, ref.loss)
        for l in range(len(Ws)):
            assert og.max_rel_err(dW[l], ref.Y[l + 1]) < 1e-4, (it, l)


def test_saint_requires_sample_and_input(rdm):
    import torch
    g = synth.rmat(500, 3000, seed=1)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    s = rdm.Saint(ctx, 50, walk_len=2, seed=1)
    model = s.gcn([16, 8, 3], 3)
    W = [torch.zeros(16, 8, device="cuda:0"), torch.zeros(8, 3, device="cuda:0")]
    loss = torch.zeros(1, dtype=torch.float64, device="cuda:0")
    with pytest.raises(rdm.RdmError):
        model.forward(W, loss)           # no subgraph yet
    s.sample(0)
    with pytest.raises(rdm.RdmError):
        model.forward(W, loss)           # subgraph without its input
    with pytest.raises(rdm.RdmError):
        model.set_input([torch.zeros(1, 16, device="cuda:0")], [torch.zeros(1, dtype=torch.int32,
                                                                             device="cuda:0")])
    model.close()
    s.close()


def test_saint_core_spmm_matches_oracle(rdm, monkeypatch):
    """Device-built hub core of a subgraph: A_s·X through rdm's SpMM on the
    sampler's graph equals the oracle product on the oracle's subgraph."""
    import torch
    monkeypatch.setenv("RDM_SAINT_CORE_K", "512")
    g = synth.rmat(6000, 90000, seed=8)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    s = rdm.Saint(ctx, 600, walk_len=4, seed=5)
    f = [48, 40, 5]
    model = s.gcn(f, 10)          # D-first forward: SpMM of width 40 and 5
    for it in range(2):
        s.sample(it)
        nodes, rp, cs, vs = osaint.sample(g, 600, 4, 5, it)
        sub = synth.CSR(len(nodes), rp, cs, vs)
        H0 = synth.features(g.n, f[0])
        Ws = synth.weights(f)
        y = synth.labels(g.n, f[-1])
        dev = "cuda:0"
        model.saint_input(torch.from_numpy(H0).to(dev), torch.from_numpy(y).to(dev))
        Wd = [torch.from_numpy(w).to(dev) for w in Ws]
        loss = torch.zeros(1, dtype=torch.float64, device=dev)
        model.forward(Wd, loss)
        ctx.sync()
        Z = model.tensor_torch(rdm.T_Z, 0).cpu().numpy()
        ref = og.forward(sub, H0[nodes], Ws, y[nodes], np.ones(len(nodes), dtype=bool))
        assert og.max_rel_err(Z, ref.Z[len(Ws)]) < 1e-4
    model.close()
    s.close()


@pytest.mark.slow
def test_saint_config4_full_size_sampled(rdm):
    """BASELINE configs[3] at full size in bench.py --saint's launch
    configuration (Reddit-shaped graph, 8,000 roots, walks of 4, 602/256/41,
    P = 1, model-picked config, hub cores on), against the oracle's own
    sampler and induced subgraph: forward rows on 4,096 sampled vertices from the
    GPU's own previous layer, the loss from the GPU's logits, and both weight
    gradients recomputed in fp64 through the whole backward of the subgraph."""
    wl = synth.WORKLOADS["reddit"]
    g = synth.make_graph(wl)
    f = (wl.f[0], 256, wl.f[-1])
    H0 = synth.features(wl.n, f[0])
    Ws = synth.weights(f)
    y = synth.labels(wl.n, f[-1])
    m = synth.train_mask(wl.n)
    roots, h, seed = 8000, 4, 1
    nodes0, rp0, cs0, _ = osaint.sample(g, roots, h, seed, 0)
    _, cfg, _, _ = rdm.select_config(list(f), len(nodes0), len(cs0), 1)
    rng = np.random.default_rng(3)
    for it, loss, dW, W_now, model in _saint_run(rdm, g, H0, Ws, y, m, cfg, 1, roots, h, seed, 2):
        nodes, rp, cs, vs = osaint.sample(g, roots, h, seed, it)
        sub = synth.CSR(len(nodes), rp, cs, vs)
        n = len(nodes)
        rows = np.sort(rng.choice(n, size=min(4096, n), replace=False))
        X0 = H0[nodes]
        H1 = model.tensor_torch(rdm.T_H, 1).cpu().numpy()
        Z = model.tensor_torch(rdm.T_Z, 0).cpu().numpy()
        assert H1.shape == (n, f[1]) and Z.shape == (n, f[2])
        ref1 = np.maximum(og.spmm_rows(sub, X0, rows) @ W_now[0].astype(np.float64), 0)
        assert og.max_rel_err(H1[rows], ref1) < 1e-4, (it, "H1")
        assert og.max_rel_err(Z[rows], og.spmm_rows(sub, H1, rows) @ W_now[1].astype(np.float64)) < 1e-4
        lref, GL = og.softmax_xent(Z, y[nodes], m[nodes])
        assert abs(loss - lref) <= 1e-5 * abs(lref), (it, loss, lref)
        S2 = og.spmm(sub, GL)
        assert og.max_rel_err(dW[1], H1.astype(np.float64).T @ S2) < 1e-4, (it, "Y2")
        G1 = (S2 @ W_now[1].astype(np.float64).T) * (H1 > 0)
        assert og.max_rel_err(dW[0], X0.astype(np.float64).T @ og.spmm(sub, G1)) < 1e-4, (it, "Y1")
