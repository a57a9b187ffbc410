"""GPU parity of the GCN with biases (RDM_GCN_BIAS; reading R8: Z^l =
Â H^{l-1} W^l + 1 (b^l)ᵀ before σ, db^l = 1ᵀ G^l) through the C ABI against the
fp64 oracle (oracle/gcn.py forward(bs=…) / backward → res.db, pinned by
tests/test_oracle_pins.py::test_bias_*).  Gates as the bias-free epoch
(DESIGN.md "Parity gates"): loss 1e-5 relative, logits / H^l / Y^l / db^l /
G^0 1e-4 normwise max-relative (fast variant 2e-2, loss 1e-4)."""
import numpy as np
import pytest

import synth
from oracle import gcn as og
from parity import BAND_FAST, BAND_FP32, relu_tiebreak

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rdm():
    import paper_conf_ipps_kurtysps23_b200 as r
    return r


def _biases(f, seed=3, scale=0.2):
    rng = np.random.default_rng(seed)
    return [(rng.standard_normal(f[l]) * scale).astype(np.float32) for l in range(1, len(f))]


def _problem(n=2708, E=5278, f=(1433, 128, 7), seed=1):
    g = synth.rmat(n, E, seed=seed)
    return g, synth.features(n, f[0]), synth.weights(f), synth.labels(n, f[-1]), synth.train_mask(n, 0.6, seed=7)


def _inputs(rdm, torch, dev, g, H0, y, m, P, f0):
    Hs, ys, ms = [], [], []
    for p in range(P):
        lo, hi, _ = rdm.partition(P, rdm.ROW, g.n, f0, p)
        Hs.append(torch.from_numpy(np.ascontiguousarray(H0[lo:hi])).to(dev))
        ys.append(torch.from_numpy(y[lo:hi]).to(dev))
        ms.append(torch.from_numpy(m[lo:hi]).to(dev))
    return Hs, ys, ms


def _run(rdm, prob, bs, cfg, P=1, transport="nccl", precision="fp32", low_memory=False, panels_ra=0,
         bias=True, epochs=1):
    import torch
    g, H0, Ws, y, m = prob
    dev = torch.device("cuda:0")
    f = [H0.shape[1]] + [w.shape[1] for w in Ws]
    ctx = rdm.Context(device=0) if P == 1 else rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    ctx.set_transport(transport)
    ctx.set_precision(precision)
    if panels_ra:
        ctx.set_graph_panels(panels_ra, g.rowptr, g.col, g.val)
    else:
        ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    model = rdm.GCN(ctx, f, cfg, low_memory=low_memory, panels=bool(panels_ra), bias=bias)
    model.set_input(*_inputs(rdm, torch, dev, g, H0, y, m, P, f[0]))
    Wd = [torch.from_numpy(w.copy()).to(dev) for w in Ws]
    bd = [torch.from_numpy(b.copy()).to(dev) for b in bs] if bias else None
    dW = [torch.zeros_like(w) for w in Wd]
    db = [torch.full_like(b, float("nan")) for b in bd] if bias else None
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    for _ in range(epochs):
        model.forward(Wd, loss, bd)
        model.backward(Wd, dW, db)
    ctx.sync()
    return (float(loss.item()), [d.cpu().numpy() for d in dW],
            [d.cpu().numpy() for d in db] if bias else None, model, ctx)


def _gather(rdm, model, which, layer, n, width, P, ra=0):
    for layout in (rdm.ROW, rdm.COL):
        try:
            parts = [model.tensor_torch(which, layer, p, layout).cpu().numpy() for p in range(P)]
        except rdm.RdmError:
            continue
        full = np.zeros((n, width))
        for p, t in enumerate(parts):
            if P == 1:
                full[:] = t[:, :width]
            elif layout == rdm.ROW:
                lo, hi, _ = rdm.partition(P, rdm.ROW, n, width, p)
                full[lo:hi] = t[:hi - lo, :width]
            elif ra:
                r0, r1, c0, c1, _ = rdm.partition_tile(P, ra, n, width, p)
                full[r0:r1, c0:c1] = t[:r1 - r0, :c1 - c0]
            else:
                lo, hi, _ = rdm.partition(P, rdm.COL, n, width, p)
                full[:, lo:hi] = t[:, :hi - lo]
        return full
    raise AssertionError(f"tensor {which}/{layer} not resident")


def _check(rdm, prob, bs, loss, dW, db, model, P=1, tol=1e-4, ltol=1e-5, ra=0):
    g, H0, Ws, y, m = prob
    L = len(Ws)
    f = [H0.shape[1]] + [w.shape[1] for w in Ws]
    band = BAND_FP32 if tol <= 1e-4 else BAND_FAST
    ref = og.forward(g, H0, Ws, y, m, bs=[b.astype(np.float64) for b in bs])
    Hs = [_gather(rdm, model, rdm.T_H, l, g.n, f[l], P, ra) for l in range(1, L)]
    for l in range(1, L):
        assert og.max_rel_err(Hs[l - 1], og.relu(ref.Z[l])) < tol, ("H", l)
    Z = _gather(rdm, model, rdm.T_Z, 0, g.n, f[L], P, ra)
    assert og.max_rel_err(Z, ref.Z[L]) < tol, "logits"
    relu_tiebreak(ref, Hs, band)
    og.backward(g, ref, Ws)
    assert abs(loss - ref.loss) <= ltol * abs(ref.loss), (loss, ref.loss)
    for l in range(1, L + 1):
        assert og.max_rel_err(dW[l - 1], ref.Y[l]) < tol, ("Y", l)
        assert og.max_rel_err(db[l - 1], ref.db[l]) < tol, ("db", l, og.max_rel_err(db[l - 1], ref.db[l]))
    G0 = _gather(rdm, model, rdm.T_G, 0, g.n, f[0], P, ra)
    assert og.max_rel_err(G0, ref.G[0]) < tol, "G0"


@pytest.fixture(scope="module")
def cora():
    prob = _problem()
    f = [prob[1].shape[1]] + [w.shape[1] for w in prob[2]]
    return prob, _biases(f)


@pytest.mark.parametrize("cfg", list(range(16)))
def test_bias_every_config_p1(rdm, cora, cfg):
    """All 16 Table IV configurations with biases: the bias lands on whichever
    product runs last (GEMM epilogue for order S, SpMM epilogue for order D)."""
    prob, bs = cora
    loss, dW, db, model, _ = _run(rdm, prob, bs, cfg)
    _check(rdm, prob, bs, loss, dW, db, model)


@pytest.mark.parametrize("transport", ["nccl", "p2p"])
@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("cfg", [2, 3, 5, 6, 9, 10, 15])
def test_bias_virtual_group(rdm, cora, P, cfg, transport):
    """Column-slice biases (b^l + the slice's column offset) in SpMM epilogues,
    db^l partials from row slices or column ranges summed across ranks."""
    prob, bs = cora
    loss, dW, db, model, _ = _run(rdm, prob, bs, cfg, P=P, transport=transport)
    _check(rdm, prob, bs, loss, dW, db, model, P=P)


@pytest.mark.parametrize("P,cfg", [(1, 0), (1, 21), (1, 42), (1, 63), (4, 21), (4, 42), (8, 5)])
def test_bias_three_layers(rdm, P, cfg):
    """3-layer products-shaped widths (f = 100, 256, 256, 47), mixed orders."""
    prob = _problem(n=3000, E=30000, f=(100, 256, 256, 47), seed=4)
    bs = _biases([100, 256, 256, 47], seed=8)
    loss, dW, db, model, _ = _run(rdm, prob, bs, cfg, P=P)
    _check(rdm, prob, bs, loss, dW, db, model, P=P)


@pytest.mark.parametrize("P,RA", [(4, 2), (8, 4), (6, 3)])
@pytest.mark.parametrize("cfg", [3, 10, 15])
def test_bias_partial_replication(rdm, cora, P, RA, cfg):
    """R_A < P tiles (RDM_GCN_PANELS): tile-column bias offsets and tile partials of db."""
    prob, bs = cora
    loss, dW, db, model, _ = _run(rdm, prob, bs, cfg, P=P, panels_ra=RA)
    _check(rdm, prob, bs, loss, dW, db, model, P=P, ra=RA)


@pytest.mark.parametrize("P,cfg", [(1, 3), (1, 10), (4, 5)])
def test_bias_fast_variant(rdm, cora, P, cfg):
    prob, bs = cora
    loss, dW, db, model, _ = _run(rdm, prob, bs, cfg, P=P, precision="fast")
    _check(rdm, prob, bs, loss, dW, db, model, P=P, tol=2e-2, ltol=1e-4)


@pytest.mark.parametrize("P,cfg", [(1, 3), (4, 10)])
def test_bias_zero_is_bias_free_model(rdm, cora, P, cfg):
    """b = 0 reproduces the bias-free model bit for bit (the epilogue adds +0.0
    after the accumulation), and db^l is 1ᵀ G^l of that model."""
    prob, bs = cora
    zeros = [np.zeros_like(b) for b in bs]
    la, dWa, dba, ma, _ = _run(rdm, prob, zeros, cfg, P=P)
    lb, dWb, _, mb, _ = _run(rdm, prob, bs, cfg, P=P, bias=False)
    assert la == lb
    for a, b in zip(dWa, dWb):
        assert np.array_equal(a, b)
    g, H0, Ws = prob[0], prob[1], prob[2]
    f = [H0.shape[1]] + [w.shape[1] for w in Ws]
    for l in range(1, len(f)):
        G = _gather(rdm, mb, rdm.T_G, l, g.n, f[l], P)
        assert og.max_rel_err(dba[l - 1], G.sum(axis=0)) < 1e-5, l


@pytest.mark.parametrize("cfg", [3, 10])
def test_bias_low_memory_bitwise(rdm, cora, cfg):
    """RDM_GCN_LOW_MEMORY (shared slabs) gives the same bits with biases, epoch after epoch."""
    prob, bs = cora
    la, dWa, dba, _, _ = _run(rdm, prob, bs, cfg, epochs=2)
    lb, dWb, dbb, _, _ = _run(rdm, prob, bs, cfg, epochs=2, low_memory=True)
    assert la == lb
    for a, b in zip(dWa + dba, dWb + dbb):
        assert np.array_equal(a, b)


def test_bias_required_and_checked(rdm, cora):
    """A bias model refuses a forward without b and a backward without db."""
    import torch
    prob, bs = cora
    g, H0, Ws, y, m = prob
    dev = torch.device("cuda:0")
    f = [H0.shape[1]] + [w.shape[1] for w in Ws]
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    model = rdm.GCN(ctx, f, 3, bias=True)
    model.set_input(*_inputs(rdm, torch, dev, g, H0, y, m, 1, f[0]))
    Wd = [torch.from_numpy(w.copy()).to(dev) for w in Ws]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    with pytest.raises(rdm.RdmError):
        model.forward(Wd, loss)
    bd = [torch.from_numpy(b.copy()).to(dev) for b in bs]
    model.forward(Wd, loss, bd)
    with pytest.raises(rdm.RdmError):
        model.backward(Wd, [torch.zeros_like(w) for w in Wd])
    assert "+b1" in model.describe() and "BSUM" in model.describe()


@pytest.mark.parametrize("P,cfg", [(1, 3), (1, 10), (2, 10), (4, 2)])
def test_bias_saint(rdm, P, cfg):
    """GraphSAINT-RDM with biases: per subgraph, against the oracle on the
    sampled subgraph (oracle/saint.py), through two Adam steps of W only."""
    import torch
    from oracle import saint as osaint
    n, f = 4000, (300, 64, 11)
    g = synth.rmat(n, 40000, seed=6)
    H0, Ws = synth.features(n, f[0]), synth.weights(f)
    y, m = synth.labels(n, f[-1]), synth.train_mask(n, 0.7, seed=2)
    bs = _biases(f, seed=5)
    dev = torch.device("cuda:0")
    ctx = rdm.Context(device=0) if P == 1 else rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    roots, h, seed = 250, 4, 99
    s = rdm.Saint(ctx, roots, walk_len=h, seed=seed)
    model = s.gcn(list(f), cfg, bias=True)
    Hd, yd = torch.from_numpy(H0).to(dev), torch.from_numpy(y).to(dev)
    md = torch.from_numpy(m.astype(np.uint8)).to(dev)
    Wd = [torch.from_numpy(w.copy()).to(dev) for w in Ws]
    bd = [torch.from_numpy(b.copy()).to(dev) for b in bs]
    dW = [torch.zeros_like(w) for w in Wd]
    db = [torch.zeros_like(b) for b in bd]
    mo, ve = [torch.zeros_like(w) for w in Wd], [torch.zeros_like(w) for w in Wd]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    for it in range(3):
        s.sample(it)
        model.saint_input(Hd, yd, md)
        W_now = [w.cpu().numpy().copy() for w in Wd]
        model.forward(Wd, loss, bd)
        model.backward(Wd, dW, db)
        ctx.sync()
        nodes, rp, cs, vs = osaint.sample(g, roots, h, seed, it)
        sub = synth.CSR(len(nodes), rp, cs, vs)
        _check(rdm, (sub, H0[nodes], W_now, y[nodes], m[nodes]), bs, float(loss.item()),
               [d.cpu().numpy() for d in dW], [d.cpu().numpy() for d in db], model, P=P)
        ctx.adam_step(Wd, dW, mo, ve, it + 1)
    model.close()
    s.close()
