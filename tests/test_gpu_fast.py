"""GPU parity of the RDM_PREC_FAST variant (rdm.h
rdm_set_precision): bf16 SpMM operand with fp32 accumulation, one bf16 piece
in the binary hub tiles, 1xTF32 GEMMs.

Gates:
* north star "2e-2 if a bf16 GEMM variant is enabled" for every layer output,
  gradient and the composed epoch (max relative error per tensor, R26);
* tighter pins on what the variant computes: without hub tiles the SpMM is
  exactly A·bf16(X) accumulated in fp32, or — when every value factors as
  â_ij = s_i·s_j (the GCN normalisation) — s_i·Σ_j bf16(s_j·X_j) (compared
  with fp64 sums of the same rounded inputs, fp32 gate 1e-4); the GEMMs are tf32 products
  (5e-3, a few tf32 unit round-offs 2^-11);
* redistribution stays bit-exact (pure data movement, unchanged).
The bf16 rounding below is test-side (round to nearest even on the fp32 bit
pattern), not library code."""
import numpy as np
import pytest

import synth
from oracle import gcn as og

from test_gpu_gcn import _check, _problem, _run

pytestmark = pytest.mark.gpu

GATE = 2e-2
# loss: the north star's 1e-5 is kept for fp32 (measured <= 1e-9); this
# bf16 variant's loss error is measured at 1.9e-6 - 1.0e-5 over IDs {2,3,5,10,15}
# x P {1,2,4} (profiles/r2_fast_loss.txt: bf16-rounded SpMM inputs move the mean
# cross-entropy by ~1e-5 relative), so its gate is the north star's fp32 output
# gate 1e-4 — 10x the measured error, 200x stricter than the variant's 2e-2
LOSS_GATE = 1e-4


def bf16_rne(x):
    u = np.ascontiguousarray(x, np.float32).view(np.uint32).astype(np.uint64)
    r = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16) << 16
    return r.astype(np.uint32).view(np.float32)


@pytest.fixture(scope="module")
def torch_dev():
    import torch
    return torch, torch.device("cuda:0")


@pytest.fixture(scope="module")
def rdm():
    import paper_conf_ipps_kurtysps23_b200 as r
    return r


def _padded(torch, dev, X):
    n, w = X.shape
    t = torch.zeros((n, (w + 3) // 4 * 4), dtype=torch.float32, device=dev)
    t[:, :w] = torch.from_numpy(np.ascontiguousarray(X, np.float32)).to(dev)
    return t


def test_bf16_rounding_helper():
    x = np.array([1.0, 1.0 + 2**-8, 1.0 + 2**-7 + 2**-8, 3.0e38, -2.5, 0.0], np.float32)
    got = bf16_rne(x)
    assert got[0] == 1.0 and got[1] == 1.0            # tie → even
    assert got[2] == np.float32(1.0 + 2**-6)          # tie → even (up)
    assert got[4] == -2.5 and got[5] == 0.0


def _factor_scale(g):
    """s with val_ij == s_i s_j (fp32 s = 1/sqrt(deg)) on every entry, else None —
    the library's own test (rdm_set_graph) restated on the host."""
    deg = np.diff(g.rowptr).astype(np.float64)
    s = np.where(deg > 0, 1.0 / np.sqrt(np.maximum(deg, 1)), 0.0)
    rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    f = s[rows] * s[g.col]
    if np.all(np.abs(g.val.astype(np.float64) - f) <= np.ldexp(f, -21)):
        return s.astype(np.float32)
    return None


def _spmm_pattern(g, X):
    """Σ_j over the stored entries of row i of X_j (values ignored), fp64."""
    import scipy.sparse as sp
    B = sp.csr_matrix((np.ones(g.nnz), g.col, g.rowptr), shape=(g.n, g.n))
    return B @ X.astype(np.float64)


FAST_GRAPHS = {
    "rmat_cora": lambda: synth.rmat(2708, 5278, seed=1),
    "directed_empty_rows": lambda: synth.random_directed(3000, 40000, seed=5, empty_rows=50),
    "star_heavy": lambda: synth.star_graph(9000),
    "rmat_skewed": lambda: synth.rmat(20000, 400000, seed=3),
    "rmat_unfactored": lambda: _perturbed(synth.rmat(5000, 60000, seed=8)),
}


def _perturbed(g):
    """Same pattern, values off the s_i·s_j factorisation by ~1e-3 (the
    library keeps the valued bf16 kernel)."""
    g.val = (g.val * (1 + 1e-3 * np.random.default_rng(0).standard_normal(g.nnz))).astype(np.float32)
    return g


@pytest.mark.parametrize("gname", list(FAST_GRAPHS))
@pytest.mark.parametrize("w", [1, 3, 5, 16, 41, 128, 130, 256, 301])
def test_fast_spmm_is_bf16_input_fp32_accumulate(torch_dev, rdm, gname, w, monkeypatch):
    torch, dev = torch_dev
    monkeypatch.setenv("RDM_NO_TILES", "1")
    monkeypatch.setenv("RDM_NO_CORE", "1")
    g = FAST_GRAPHS[gname]()
    sym = gname != "directed_empty_rows"
    ctx = rdm.Context(device=0)
    ctx.set_precision("fast")
    assert ctx.precision == "fast"
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=sym)
    rng = np.random.default_rng(w)
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    xd = _padded(torch, dev, X)
    fs = _factor_scale(g) if sym else None
    for transpose in ([0, 1] if not sym else [0]):
        out = torch.zeros_like(xd)
        ctx.spmm(transpose, xd, out, w, rdm.EPI_RELU)
        ctx.sync()
        f = og.spmm_t if transpose else og.spmm
        got = out[:, :w].cpu().numpy()
        if fs is None:   # values used as given: Σ_j a_ij · bf16(X_j)
            exact = np.maximum(f(g, bf16_rne(X)), 0)
        else:            # â_ij = s_i s_j: s_i · Σ_j bf16(fp32(s_j X_j)) (value-free row sums)
            Xs = bf16_rne((fs[:, None] * X).astype(np.float32))
            exact = np.maximum(fs[:, None].astype(np.float64) * _spmm_pattern(g, Xs), 0)
        assert og.max_rel_err(got, exact) < 1e-4               # what the variant computes
        assert og.max_rel_err(got, np.maximum(f(g, X), 0)) < GATE  # vs the plain product
        assert np.all(out[:, w:].cpu().numpy() == 0)


@pytest.mark.parametrize("w", [4, 16, 41, 128, 256])
@pytest.mark.parametrize("min_nnz", [1, 40])
@pytest.mark.parametrize("form", ["i8x2", "bf16"])
def test_fast_spmm_hub_tiles(torch_dev, rdm, w, min_nnz, form, monkeypatch):
    """Fast variant tiles: two int8 digits of a 15-bit per-column fixed point of
    s⊙X on kind::i8 (default) or one bf16 piece on kind::f16
    (RDM_TILE_PIECES_FAST=1), + the bf16 residual CSR, within the 2e-2 gate
    (measured ≈ 1e-3, the residual's bf16 rows)."""
    torch, dev = torch_dev
    monkeypatch.setenv("RDM_TILE_MIN_NNZ", str(min_nnz))
    if form == "bf16":
        monkeypatch.setenv("RDM_TILE_PIECES_FAST", "1")
    g = synth.rmat(6000, 150000, seed=13)
    ctx = rdm.Context(device=0)
    ctx.set_precision("fast")
    ctx.set_graph(g.rowptr, g.col, g.val)
    assert ctx.graph_info()["n_tiles"] > 0
    rng = np.random.default_rng(w)
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    M = rng.standard_normal((g.n, w)).astype(np.float32)
    xd, md = _padded(torch, dev, X), _padded(torch, dev, M)
    out = torch.zeros_like(xd)
    ctx.spmm(0, xd, out, w, rdm.EPI_RELU | rdm.EPI_MASK, mask=md)
    ctx.sync()
    ref = np.maximum(og.spmm(g, X), 0) * (M > 0)
    err = og.max_rel_err(out[:, :w].cpu().numpy(), ref)
    assert err < 1e-2, err
    assert np.all(out[:, w:].cpu().numpy() == 0)


GEMM_SHAPES = [(1000, 7, 128), (2049, 41, 128), (777, 128, 41), (3000, 602, 128),
               (513, 128, 602), (4097, 256, 256), (300, 100, 256), (1, 128, 47), (130, 1433, 128)]


@pytest.mark.parametrize("rows,k,m", GEMM_SHAPES)
def test_fast_gemm_tf32(torch_dev, rdm, rows, k, m):
    torch, dev = torch_dev
    ctx = rdm.Context(device=0)
    ctx.set_precision("fast")
    rng = np.random.default_rng(rows + k + m)
    X = rng.standard_normal((rows, k)).astype(np.float32)
    W = rng.standard_normal((k, m)).astype(np.float32)
    G = rng.standard_normal((rows, m)).astype(np.float32)
    Xd, Gd = _padded(torch, dev, X), _padded(torch, dev, G)
    Wd = torch.from_numpy(W).to(dev)
    C = torch.zeros((rows, (m + 3) // 4 * 4), device=dev)
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m, rdm.EPI_RELU)
    D = torch.zeros((rows, (k + 3) // 4 * 4), device=dev)
    ctx.gemm(rdm.GEMM_NT, Gd, Wd, D, rows, k, m)
    Y = torch.zeros((k, m), device=dev)
    ctx.gemm(rdm.GEMM_TN, Xd, Gd, Y, rows, k, m)
    ctx.sync()
    X64, W64, G64 = X.astype(np.float64), W.astype(np.float64), G.astype(np.float64)
    assert og.max_rel_err(C[:, :m].cpu().numpy(), np.maximum(X64 @ W64, 0)) < 5e-3
    assert og.max_rel_err(D[:, :k].cpu().numpy(), G64 @ W64.T) < 5e-3
    assert og.max_rel_err(Y.cpu().numpy(), X64.T @ G64) < 5e-3
    # and it is a different (cheaper) arithmetic than the default 3xTF32
    ctx.set_precision("fp32")
    C3 = torch.zeros_like(C)
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C3, rows, k, m, rdm.EPI_RELU)
    ctx.sync()
    assert og.max_rel_err(C3[:, :m].cpu().numpy(), np.maximum(X64 @ W64, 0)) < 1e-4


@pytest.fixture(scope="module")
def cora():
    return _problem()


@pytest.mark.parametrize("P", [1, 4])
@pytest.mark.parametrize("cfg", [2, 3, 5, 10, 15])
def test_fast_epoch_within_gate(rdm, cora, P, cfg):
    g, H0, Ws, y, m = cora
    loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, cfg, P=P, precision="fast")
    _check((g, H0, Ws, y, m), loss, dW, model, rdm, P=P, tol=GATE, ltol=LOSS_GATE)


def test_fast_three_layer_products_shaped(rdm):
    prob = _problem(n=6000, E=40000, f=(100, 256, 256, 47), seed=2)
    g, H0, Ws, y, m = prob
    loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, 9, P=2, precision="fast")
    _check(prob, loss, dW, model, rdm, P=2, tol=GATE, ltol=LOSS_GATE)


@pytest.mark.parametrize("cfg", [3, 10])
def test_fast_epoch_hub_tiles(rdm, cfg, monkeypatch):
    monkeypatch.setenv("RDM_TILE_MIN_NNZ", "20")
    prob = _problem(n=8000, E=200000, f=(64, 128, 41), seed=5)
    g, H0, Ws, y, m = prob
    loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, cfg, precision="fast")
    assert ctx.graph_info()["n_tiles"] > 0
    _check(prob, loss, dW, model, rdm, tol=GATE, ltol=LOSS_GATE)


def test_precision_rejects_unknown(rdm):
    ctx = rdm.Context(device=0)
    with pytest.raises(rdm.RdmError):
        ctx._c(rdm._lib.rdm_set_precision(ctx.h, 7))


@pytest.mark.parametrize("P,cfg", [(2, 3), (4, 10), (3, 5), (8, 2)])
def test_fast_bf16_wire_halves_bytes(rdm, cora, P, cfg):
    """RDM_PREC_FAST: the executor's row → column redistributions carry bf16
    (NEXT-3): their bytes on the wire halve against the fp32 variant exactly
    (the per-redistribution wire bytes from rdm_redist_plan), column → row
    moves keep fp32, the payload element count is unchanged, and the epoch
    stays within the 2e-2 gate with the loss within 1e-5."""
    g, H0, Ws, y, m = cora
    _, _, _, ctx32, _ = _run(rdm, g, H0, Ws, y, m, cfg, P=P)
    c32 = ctx32.counters()
    loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, cfg, P=P, precision="fast")
    c16 = ctx.counters()
    assert c16["a2a_elems_payload"] == c32["a2a_elems_payload"]
    assert c16["a2a_width_units"] == c32["a2a_width_units"]
    f = [H0.shape[1]] + [w.shape[1] for w in Ws]
    _, desc = rdm.plan_info(f, cfg, P, g.n)
    want32 = want16 = 0
    for line in desc.splitlines():
        if not line.strip().startswith("A2A"):
            continue
        w = int(line.split("f=")[1].split()[0])
        fr = rdm.ROW if ".row ->" in line else rdm.COL
        b = sum(4 * sum(pl["send_elems"][q] for q in range(P) if q != p)
                for p in range(P) for pl in [rdm.redist_plan(P, p, fr, g.n, w)])
        want32 += b
        want16 += b // 2 if fr == rdm.ROW else b
    assert c32["a2a_bytes_wire"] == want32
    assert c16["a2a_bytes_wire"] == want16 < want32
    _check((g, H0, Ws, y, m), loss, dW, model, rdm, P=P, tol=GATE, ltol=LOSS_GATE)


@pytest.mark.parametrize("cfg", [3, 10, 15])
def test_fast_cast_folded_into_gemm(rdm, cora, cfg, monkeypatch):
    """NEXT-3: at P = 1 the fast variant's GEMM epilogue writes the next SpMM's
    bf16 input itself (× s_i for factored values) instead of a separate cast
    pass — bit-identical results, fewer launches."""
    g, H0, Ws, y, m = cora
    out = {}
    for fold in ("0", "1"):
        monkeypatch.setenv("RDM_FOLD_CAST", fold)
        loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, cfg, P=1, precision="fast")
        out[fold] = (loss, dW, ctx.counters()["kernel_launches"])
        model.close()
        ctx.close()
    assert out["0"][0] == out["1"][0]
    for a, b in zip(out["0"][1], out["1"][1]):
        assert np.array_equal(a, b)
    f = [H0.shape[1]] + [w.shape[1] for w in Ws]
    _, desc = rdm.plan_info(f, cfg, 1, g.n)
    steps = [l.split() for l in desc.splitlines() if l.startswith("  ")]

    def gemm_out(t):   # "GEMM NN X W -> Y.row ..." (not TN)
        return t[t.index("->") + 1].split(".")[0] if t[0] == "GEMM" and t[1] in ("NN", "NT") else None

    def spmm_in(t):    # "SPMM A^T X.col -> ..."
        return t[2].split(".")[0] if t[0] == "SPMM" else None

    folds = sum(1 for a, b in zip(steps, steps[1:]) if gemm_out(a) and gemm_out(a) == spmm_in(b))
    assert out["1"][2] == out["0"][2] - folds, (out, folds)
