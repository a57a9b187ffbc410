"""GPU parity of partial replication R_A < P (PAPER.md
§III-E, Fig. 6; Tables II/III "Comm. (R_A < P)"; §IV-A.4) in a
virtual group of P ranks on one GPU, through the C ABI, against the fp64
oracle.  Gates: redistribution bit-exact; SpMM 1e-4 max relative (fp32) or
2e-2 (fast variant); moved elements equal the model's counts exactly."""
import numpy as np
import pytest

import synth
from oracle import gcn as og

pytestmark = pytest.mark.gpu

GRIDS = [(2, 1), (2, 2), (4, 1), (4, 2), (8, 2), (8, 4), (6, 3)]


@pytest.fixture(scope="module")
def env():
    import torch
    import paper_conf_ipps_kurtysps23_b200 as rdm
    return torch, torch.device("cuda:0"), rdm


def _tiles(torch, dev, rdm, X, P, RA):
    n, f = X.shape
    out = []
    for p in range(P):
        r0, r1, c0, c1, ld = rdm.partition_tile(P, RA, n, f, p)
        t = torch.zeros((max(r1 - r0, 1), ld), dtype=torch.float32, device=dev)
        t[:r1 - r0, :c1 - c0] = torch.from_numpy(np.ascontiguousarray(X[r0:r1, c0:c1], np.float32)).to(dev)
        out.append(t)
    return out


def _rows(torch, dev, rdm, X, P):
    n, f = X.shape
    out = []
    for p in range(P):
        lo, hi, ld = rdm.partition(P, rdm.ROW, n, f, p)
        t = torch.zeros((max(hi - lo, 1), ld), dtype=torch.float32, device=dev)
        t[:hi - lo, :f] = torch.from_numpy(np.ascontiguousarray(X[lo:hi], np.float32)).to(dev)
        out.append(t)
    return out


def _assemble_tiles(rdm, tiles, n, f, P, RA):
    full = np.zeros((n, f))
    for p, t in enumerate(tiles):
        r0, r1, c0, c1, _ = rdm.partition_tile(P, RA, n, f, p)
        full[r0:r1, c0:c1] = t[:r1 - r0, :c1 - c0].cpu().numpy()
    return full


@pytest.mark.parametrize("P,RA", GRIDS)
@pytest.mark.parametrize("n,f", [(1001, 41), (64, 7), (997, 130), (5, 3)])
def test_redistribute_panels_bit_exact(env, P, RA, n, f):
    torch, dev, rdm = env
    rng = np.random.default_rng(n + f)
    X = rng.standard_normal((n, f)).astype(np.float32)
    X[0, 0] = np.float32(np.nan)                     # payloads move untouched
    ctx = rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    rp = np.zeros(n + 1, np.int64)                   # empty graph: only the panel layout matters
    ctx.set_graph_panels(RA, rp, np.zeros(0, np.int32), np.zeros(0, np.float32))
    rows = _rows(torch, dev, rdm, X, P)
    tiles = [torch.full_like(t, -7.0) for t in _tiles(torch, dev, rdm, X, P, RA)]
    for p in range(P):   # padding columns must stay zero; rows of the tile are fully written
        r0, r1, c0, c1, ld = rdm.partition_tile(P, RA, n, f, p)
        tiles[p][:, c1 - c0:] = 0
    ctx.reset_counters()
    ctx.redistribute_panels(rdm.ROW, rows, tiles, n, f)
    ctx.sync()
    got = _assemble_tiles(rdm, tiles, n, f, P, RA)
    assert np.array_equal(got.astype(np.float32).view(np.uint32), X.view(np.uint32))
    # exact payload: inside each panel group, every row block goes to the other R_A − 1 members
    payload = 0
    for p in range(P):
        lo, hi, _ = rdm.partition(P, rdm.ROW, n, f, p)
        i = p // RA
        for j in range(RA):
            q = i * RA + j
            if q != p:
                _, _, c0, c1, _ = rdm.partition_tile(P, RA, n, f, q)
                payload += (hi - lo) * (c1 - c0)
    c = ctx.counters()
    assert c["a2a_elems_payload"] == payload
    assert payload <= (RA - 1) / RA * n * f + RA * f * P   # ≈ (R_A−1)/R_A·N·f (L214)
    back = [torch.zeros_like(t) for t in rows]
    ctx.redistribute_panels(rdm.COL, tiles, back, n, f)
    ctx.sync()
    for p in range(P):
        lo, hi, _ = rdm.partition(P, rdm.ROW, n, f, p)
        assert np.array_equal(back[p][:hi - lo, :f].cpu().numpy().view(np.uint32),
                              X[lo:hi].view(np.uint32))


@pytest.mark.parametrize("P,RA", GRIDS)
@pytest.mark.parametrize("w", [1, 16, 41, 128])
@pytest.mark.parametrize("prec", ["fp32", "fast"])
def test_spmm_panels_matches_oracle(env, P, RA, w, prec):
    torch, dev, rdm = env
    g = synth.rmat(3000, 30000, seed=11)
    ctx = rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    ctx.set_precision(prec)
    ctx.set_graph_panels(RA, g.rowptr, g.col, g.val)
    rng = np.random.default_rng(w)
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    M = rng.standard_normal((g.n, w)).astype(np.float32)
    ins = _tiles(torch, dev, rdm, X, P, RA)
    masks = _tiles(torch, dev, rdm, M, P, RA)
    outs = [torch.zeros_like(t) for t in ins]
    ctx.reset_counters()
    ctx.spmm_panels(ins, outs, w, rdm.EPI_RELU | rdm.EPI_MASK, masks=masks)
    ctx.sync()
    got = _assemble_tiles(rdm, outs, g.n, w, P, RA)
    ref = np.maximum(og.spmm(g, X), 0) * (M > 0)
    assert og.max_rel_err(got, ref) < (1e-4 if prec == "fp32" else 2e-2)
    for p, t in enumerate(outs):   # padding stays zero
        _, _, c0, c1, _ = rdm.partition_tile(P, RA, g.n, w, p)
        assert np.all(t[:, c1 - c0:].cpu().numpy() == 0)
    # broadcast volume: (P/R_A − 1)·N·w elements exactly (L152, L216)
    assert ctx.counters()["bcast_elems"] == (P // RA - 1) * g.n * w


@pytest.mark.parametrize("P,RA", [(4, 2), (8, 2), (8, 4)])
def test_layer_with_partial_replication(env, P, RA):
    """One GCN layer H1 = ReLU(Âᵀ (H0 W)) on the R_A < P grid, composed from
    the boundary calls: GEMM on row slices → row→tile redistribution inside
    the panel groups → panel SpMM (tile broadcast in the column groups);
    equals the oracle's dense layer (eq. 1-2)."""
    torch, dev, rdm = env
    n, f0, f1 = 2708, 96, 41
    g = synth.rmat(n, 5278, seed=1)
    H0 = synth.features(n, f0)
    W = synth.weights((f0, f1))[0]
    ctx = rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    ctx.set_graph_panels(RA, g.rowptr, g.col, g.val)
    rows = _rows(torch, dev, rdm, H0, P)
    Wd = torch.from_numpy(W).to(dev)
    T = []
    for p in range(P):
        lo, hi, ld = rdm.partition(P, rdm.ROW, n, f1, p)
        t = torch.zeros((max(hi - lo, 1), ld), device=dev)
        ctx.gemm(rdm.GEMM_NN, rows[p], Wd, t, hi - lo, f0, f1)
        T.append(t)
    tiles = [torch.zeros_like(t) for t in _tiles(torch, dev, rdm, np.zeros((n, f1), np.float32), P, RA)]
    ctx.redistribute_panels(rdm.ROW, T, tiles, n, f1)
    outs = [torch.zeros_like(t) for t in tiles]
    ctx.spmm_panels(tiles, outs, f1, rdm.EPI_RELU)
    ctx.sync()
    got = _assemble_tiles(rdm, outs, n, f1, P, RA)
    ref = np.maximum(og.spmm_t(g, H0.astype(np.float64) @ W.astype(np.float64)), 0)
    assert og.max_rel_err(got, ref) < 1e-4


@pytest.mark.parametrize("P,RA", [(2, 1), (4, 2), (8, 2), (8, 4), (6, 3)])
@pytest.mark.parametrize("cfg", [2, 3, 5, 10, 15])
def test_gcn_epoch_with_partial_replication(P, RA, cfg):
    """The whole epoch (forward, loss, backward with G^0, Y all-reduce) on the
    R_A < P grid (RDM_GCN_PANELS) agrees with the fp64 oracle at the fp32
    gates; the executor issues the model's widths, the tile broadcasts move
    (P/R_A − 1)·N·(sparse units) elements and the panel-group redistributions
    the exact intra-group payload (Tables II/III R_A rows, reading R35)."""
    import torch
    import paper_conf_ipps_kurtysps23_b200 as rdm
    from test_gpu_gcn import _check, _problem
    prob = _problem()
    g, H0, Ws, y, m = prob
    dev = torch.device("cuda:0")
    f = [H0.shape[1]] + [w.shape[1] for w in Ws]
    ctx = rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    ctx.set_graph_panels(RA, g.rowptr, g.col, g.val)
    model = rdm.GCN(ctx, f, cfg, panels=True)
    Hs, ys, ms = [], [], []
    for p in range(P):
        lo, hi, _ = rdm.partition(P, rdm.ROW, g.n, f[0], p)
        Hs.append(torch.from_numpy(np.ascontiguousarray(H0[lo:hi])).to(dev))
        ys.append(torch.from_numpy(y[lo:hi]).to(dev))
        ms.append(torch.from_numpy(m[lo:hi]).to(dev))
    model.set_input(Hs, ys, ms)
    Wd = [torch.from_numpy(w.copy()).to(dev) for w in Ws]
    dW = [torch.zeros_like(w) for w in Wd]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    ctx.reset_counters()
    model.forward(Wd, loss)
    model.backward(Wd, dW)
    ctx.sync()
    c = ctx.counters()
    info = model.info()
    _check(prob, float(loss.item()), [d.cpu().numpy() for d in dW], model, rdm, P=P, ra=RA)
    assert c["spmm_width_units"] == info["plan_sparse_units"]
    assert c["bcast_elems"] == (P // RA - 1) * g.n * info["plan_sparse_units"]
    assert c["a2a_elems_payload"] == info["a2a_elems"]
