"""GPU parity of the communication-free operators and the redistribution,
called through the C ABI, against the fp64 oracle (tolerances: DESIGN.md
"Parity gates": fp32 outputs ≤ 1e-4 normwise max-relative; redistribution
bit-exact)."""
import numpy as np
import pytest

import synth
from oracle import gcn as og
from oracle import redistribution as ordist

pytestmark = pytest.mark.gpu

TOL = 1e-4


@pytest.fixture(scope="module")
def torch_dev():
    import torch
    return torch, torch.device("cuda:0")


@pytest.fixture(scope="module")
def rdm():
    import paper_conf_ipps_kurtysps23_b200 as r
    return r


def _padded(torch, dev, X, ld=None):
    n, w = X.shape
    ld = ld or ((w + 3) // 4 * 4)
    t = torch.zeros((n, ld), dtype=torch.float32, device=dev)
    t[:, :w] = torch.from_numpy(np.ascontiguousarray(X, np.float32)).to(dev)
    return t


GRAPHS = {
    "rmat_cora": lambda: synth.rmat(2708, 5278, seed=1),
    "directed_empty_rows": lambda: synth.random_directed(3000, 40000, seed=5, empty_rows=50),
    "star_heavy": lambda: synth.star_graph(9000),            # one row of degree 9000 > segment
    "rmat_skewed": lambda: synth.rmat(20000, 400000, seed=3),
}


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("w", [1, 3, 4, 5, 16, 41, 76, 128, 130, 301])
def test_spmm_matches_oracle(torch_dev, rdm, gname, w):
    torch, dev = torch_dev
    g = GRAPHS[gname]()
    sym = gname != "directed_empty_rows"
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=sym)
    rng = np.random.default_rng(w)
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    xd = _padded(torch, dev, X)
    for transpose in ([0, 1] if not sym else [0]):
        out = torch.zeros_like(xd)
        ctx.spmm(transpose, xd, out, w)
        ctx.sync()
        ref = og.spmm_t(g, X) if transpose else og.spmm(g, X)
        got = out[:, :w].cpu().numpy()
        assert og.max_rel_err(got, ref) < TOL
        assert np.all(out[:, w:].cpu().numpy() == 0)   # padding stays zero


@pytest.mark.parametrize("w", [16, 41, 128])
def test_spmm_epilogues(torch_dev, rdm, w):
    torch, dev = torch_dev
    g = synth.rmat(5000, 60000, seed=9)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val)
    rng = np.random.default_rng(1)
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    M = rng.standard_normal((g.n, w)).astype(np.float32)
    b = rng.standard_normal(w).astype(np.float32)
    xd, md = _padded(torch, dev, X), _padded(torch, dev, M)
    bd = torch.from_numpy(b).to(dev)
    ref = og.spmm(g, X)
    out = torch.zeros_like(xd)
    ctx.spmm(0, xd, out, w, rdm.EPI_BIAS | rdm.EPI_RELU, bias=bd)
    ctx.sync()
    assert og.max_rel_err(out[:, :w].cpu().numpy(), np.maximum(ref + b, 0)) < TOL
    out.zero_()
    ctx.spmm(0, xd, out, w, rdm.EPI_MASK, mask=md)
    ctx.sync()
    assert og.max_rel_err(out[:, :w].cpu().numpy(), ref * (M > 0)) < TOL


def test_spmm_deterministic(torch_dev, rdm):
    torch, dev = torch_dev
    g = synth.star_graph(20000)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val)
    X = _padded(torch, dev, np.random.default_rng(0).standard_normal((g.n, 32)))
    o1, o2 = torch.zeros_like(X), torch.zeros_like(X)
    ctx.spmm(0, X, o1, 32)
    ctx.spmm(0, X, o2, 32)
    ctx.sync()
    assert torch.equal(o1.view(torch.int32), o2.view(torch.int32))


def test_invalid_csr_rejected(rdm):
    ctx = rdm.Context(device=0)
    rp = np.array([0, 2, 1, 3], dtype=np.int64)
    col = np.array([0, 1, 5], dtype=np.int32)
    val = np.ones(3, dtype=np.float32)
    with pytest.raises(rdm.RdmError) as e:
        ctx.set_graph(rp, col, val)
    assert e.value.status == rdm.ERR_ARG


GEMM_SHAPES = [(1000, 7, 128), (2049, 41, 128), (777, 128, 41), (3000, 602, 128),
               (513, 128, 602), (4097, 256, 256), (300, 100, 256), (1, 128, 47), (130, 1433, 128)]


@pytest.mark.parametrize("rows,k,m", GEMM_SHAPES)
def test_gemm_nn_nt_tn(torch_dev, rdm, rows, k, m):
    torch, dev = torch_dev
    ctx = rdm.Context(device=0)
    rng = np.random.default_rng(rows + k + m)
    X = rng.standard_normal((rows, k)).astype(np.float32)
    W = rng.standard_normal((k, m)).astype(np.float32)
    G = rng.standard_normal((rows, m)).astype(np.float32)
    Xd, Gd = _padded(torch, dev, X), _padded(torch, dev, G)
    Wd = torch.from_numpy(W).to(dev)
    C = torch.zeros((rows, (m + 3) // 4 * 4), device=dev)
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m)
    D = torch.zeros((rows, (k + 3) // 4 * 4), device=dev)
    ctx.gemm(rdm.GEMM_NT, Gd, Wd, D, rows, k, m)
    Y = torch.zeros((k, m), device=dev)
    ctx.gemm(rdm.GEMM_TN, Xd, Gd, Y, rows, k, m)
    ctx.sync()
    X64, W64, G64 = X.astype(np.float64), W.astype(np.float64), G.astype(np.float64)
    assert og.max_rel_err(C[:, :m].cpu().numpy(), X64 @ W64) < TOL
    assert og.max_rel_err(D[:, :k].cpu().numpy(), G64 @ W64.T) < TOL
    assert og.max_rel_err(Y.cpu().numpy(), X64.T @ G64) < TOL


def test_gemm_epilogues(torch_dev, rdm):
    torch, dev = torch_dev
    ctx = rdm.Context(device=0)
    rng = np.random.default_rng(3)
    rows, k, m = 1500, 130, 41
    X = rng.standard_normal((rows, k)).astype(np.float32)
    W = rng.standard_normal((k, m)).astype(np.float32)
    M = rng.standard_normal((rows, m)).astype(np.float32)
    Xd, Md = _padded(torch, dev, X), _padded(torch, dev, M)
    Wd = torch.from_numpy(W).to(dev)
    C = torch.zeros_like(Md)
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m, rdm.EPI_RELU)
    ctx.sync()
    ref = X.astype(np.float64) @ W
    assert og.max_rel_err(C[:, :m].cpu().numpy(), np.maximum(ref, 0)) < TOL
    C.zero_()
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m, rdm.EPI_MASK, mask=Md)
    ctx.sync()
    assert og.max_rel_err(C[:, :m].cpu().numpy(), ref * (M > 0)) < TOL


@pytest.mark.parametrize("P,n,f", [(2, 6, 8), (2, 1001, 41), (3, 1000, 130), (4, 997, 7),
                                   (8, 5, 3), (8, 2708, 1433), (8, 10007, 128), (5, 333, 47)])
def test_redistribution_virtual_group_bit_exact(torch_dev, rdm, P, n, f):
    """Row→col→row round trip bit-exact and equal to the oracle's slicing
    (Fig. 7); payload includes NaN / denormal bit patterns."""
    torch, dev = torch_dev
    ctx = rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    rng = np.random.default_rng(n + f)
    bits = rng.integers(0, 2 ** 32, size=(n, f), dtype=np.uint64).astype(np.uint32)
    bits[0, 0] = 0x7FC00123      # NaN with payload
    if n > 1 and f > 1:
        bits[1, 1] = 0x00000001  # denormal
    M = bits.view(np.float32)
    rows, cols = [], []
    for p in range(P):
        lo, hi, ld = rdm.partition(P, rdm.ROW, n, f, p)
        r = torch.zeros((hi - lo, ld), dtype=torch.int32, device=dev)
        r[:, :f] = torch.from_numpy(bits[lo:hi].view(np.int32)).to(dev)
        rows.append(r.view(torch.float32))
        clo, chi, cld = rdm.partition(P, rdm.COL, n, f, p)
        cols.append(torch.zeros((n, cld), dtype=torch.float32, device=dev))
    ctx.redistribute(rdm.ROW, rows, cols, n, f)
    ctx.sync()
    ref_cols = ordist.col_slices(M, P)
    for p in range(P):
        w = ref_cols[p].shape[1]
        got = cols[p].view(torch.int32).cpu().numpy()
        assert np.array_equal(got[:, :w], ref_cols[p].view(np.int32))
        assert np.all(got[:, w:] == 0)
    back = [torch.zeros_like(r) for r in rows]
    ctx.redistribute(rdm.COL, cols, back, n, f)
    ctx.sync()
    for p in range(P):
        assert torch.equal(back[p].view(torch.int32), rows[p].view(torch.int32))
    c = ctx.counters()
    assert c["a2a_elems_payload"] == 2 * ordist.total_elements(n, f, P)


def test_adam_matches_oracle(torch_dev, rdm):
    torch, dev = torch_dev
    ctx = rdm.Context(device=0)
    rng = np.random.default_rng(2)
    p0 = rng.standard_normal((602, 128)).astype(np.float32)
    grads = [rng.standard_normal((602, 128)).astype(np.float32) for _ in range(3)]
    p = torch.from_numpy(p0.copy()).to(dev)
    m, v = torch.zeros_like(p), torch.zeros_like(p)
    rp, rm, rv = p0.astype(np.float64), 0.0, 0.0
    for t, gr in enumerate(grads, start=1):
        ctx.adam_step([p], [torch.from_numpy(gr).to(dev)], [m], [v], t)
        rp, rm, rv = og.adam(rp, gr, rm, rv, t)
    ctx.sync()
    assert og.max_rel_err(p.cpu().numpy(), rp) < 1e-6


@pytest.mark.parametrize("w", [4, 16, 41, 128, 130])
@pytest.mark.parametrize("K", [128, 1024])
def test_spmm_hub_core_matches_oracle(torch_dev, w, K, monkeypatch):
    """Dense hub core (tensor cores) + residual CSR == the plain product, with
    epilogues; forced core sizes (RDM_CORE_K) so small graphs exercise it."""
    torch, dev = torch_dev
    import paper_conf_ipps_kurtysps23_b200 as rdm
    monkeypatch.setenv("RDM_CORE_K", str(K))
    monkeypatch.setenv("RDM_NO_TILES", "1")   # the fp32 dense core, not the binary tiles
    g = synth.rmat(6000, 150000, seed=13)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val)
    gi = ctx.graph_info()
    assert gi["core_K"] == K and gi["core_nnz"] > 0
    rng = np.random.default_rng(w)
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    M = rng.standard_normal((g.n, w)).astype(np.float32)
    xd, md = _padded(torch, dev, X), _padded(torch, dev, M)
    out = torch.zeros_like(xd)
    ctx.spmm(0, xd, out, w, rdm.EPI_RELU | rdm.EPI_MASK, mask=md)
    ctx.sync()
    ref = np.maximum(og.spmm(g, X), 0) * (M > 0)
    assert og.max_rel_err(out[:, :w].cpu().numpy(), ref) < TOL
    assert np.all(out[:, w:].cpu().numpy() == 0)


@pytest.mark.parametrize("w", [1, 4, 16, 41, 128, 130, 256, 301])
@pytest.mark.parametrize("min_nnz,k2", [(1, 0), (40, 0), (1, 1024)])
@pytest.mark.parametrize("pieces", ["auto", "auto-paired", "2", "3"])
def test_spmm_hub_tiles_matches_oracle(torch_dev, w, min_nnz, k2, pieces, monkeypatch):
    """Binary hub tiles (tensor cores on 0/1 tiles against s ⊙ X as three int8
    digits on kind::i8 (auto), two column-scaled fp16 or three bf16 pieces on
    kind::f16) + residual CSR == the plain product, with epilogues.  min_nnz forces the tile selection (every block with at least
    that many entries), k2 limits the rank range (0 = all)."""
    torch, dev = torch_dev
    import paper_conf_ipps_kurtysps23_b200 as rdm
    monkeypatch.setenv("RDM_TILE_MIN_NNZ", str(min_nnz))
    if pieces == "auto-paired":   # int8 digits, two row blocks per panel load
        monkeypatch.setenv("RDM_TILE_PAIRS", "1")
    elif pieces != "auto":   # 2 column-scaled fp16 pieces / 3 bf16 pieces at every width
        monkeypatch.setenv("RDM_TILE_PIECES", pieces)
    if k2:
        monkeypatch.setenv("RDM_TILE_K2", str(k2))
    g = synth.rmat(6000, 150000, seed=13)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val)
    gi = ctx.graph_info()
    assert gi["n_tiles"] > 0 and gi["core_K"] == 0 and gi["core_nnz"] > 0
    assert gi["tile_ranks"] % 128 == 0 and gi["tile_ranks"] <= (k2 or g.n)
    rng = np.random.default_rng(w)
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    M = rng.standard_normal((g.n, w)).astype(np.float32)
    xd, md = _padded(torch, dev, X), _padded(torch, dev, M)
    out = torch.zeros_like(xd)
    ctx.spmm(0, xd, out, w)
    ctx.sync()
    assert og.max_rel_err(out[:, :w].cpu().numpy(), og.spmm(g, X)) < TOL
    out.zero_()
    ctx.spmm(0, xd, out, w, rdm.EPI_RELU | rdm.EPI_MASK, mask=md)
    ctx.sync()
    ref = np.maximum(og.spmm(g, X), 0) * (M > 0)
    assert og.max_rel_err(out[:, :w].cpu().numpy(), ref) < TOL
    assert np.all(out[:, w:].cpu().numpy() == 0)


@pytest.mark.parametrize("pieces", ["auto", "2", "3"])
def test_spmm_hub_tiles_wide_range_values(torch_dev, pieces, monkeypatch):
    """Inputs spanning 2^±30 per row and exact zeros: the int8 digits (auto:
    23-bit fixed point per column), the column-scaled fp16 pieces and the bf16
    pieces keep the fp32 gate (normwise per tensor, reading R26) — no
    overflow, no lost columns."""
    torch, dev = torch_dev
    import paper_conf_ipps_kurtysps23_b200 as rdm
    monkeypatch.setenv("RDM_TILE_MIN_NNZ", "1")
    monkeypatch.setenv("RDM_TILE_PIECES", pieces)
    g = synth.rmat(6000, 150000, seed=14)
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val)
    assert ctx.graph_info()["n_tiles"] > 0
    rng = np.random.default_rng(0)
    w = 64
    X = (rng.standard_normal((g.n, w)) * np.exp2(rng.integers(-30, 30, (g.n, 1)))).astype(np.float32)
    X[rng.random((g.n, w)) < 0.1] = 0
    xd = _padded(torch, dev, X)
    out = torch.zeros_like(xd)
    ctx.spmm(0, xd, out, w)
    ctx.sync()
    assert og.max_rel_err(out[:, :w].cpu().numpy(), og.spmm(g, X)) < TOL


def test_spmm_hub_tiles_need_factorised_values(torch_dev, monkeypatch):
    """Values that are not s_i·s_j (here: perturbed by 1e-3 relative) build no
    binary tiles (the fp32 dense core or plain CSR instead); unit values do."""
    torch, dev = torch_dev
    import paper_conf_ipps_kurtysps23_b200 as rdm
    monkeypatch.setenv("RDM_TILE_MIN_NNZ", "1")
    g = synth.rmat(6000, 150000, seed=15)
    rng = np.random.default_rng(1)
    bad = (g.val * (1 + 1e-3 * rng.standard_normal(g.nnz))).astype(np.float32)
    ones = np.ones_like(g.val)
    w = 41
    X = rng.standard_normal((g.n, w)).astype(np.float32)
    xd = _padded(torch, dev, X)
    for vals, tiled in ((bad, False), (ones, True)):
        ctx = rdm.Context(device=0)
        ctx.set_graph(g.rowptr, g.col, vals)
        assert (ctx.graph_info()["n_tiles"] > 0) == tiled
        out = torch.zeros_like(xd)
        ctx.spmm(0, xd, out, w)
        ctx.sync()
        g2 = synth.CSR(g.n, g.rowptr, g.col, vals)
        assert og.max_rel_err(out[:, :w].cpu().numpy(), og.spmm(g2, X)) < TOL


@pytest.mark.parametrize("norm", ["row", "col", "weighted"])
def test_spmm_hub_tiles_general_rank1_values(torch_dev, norm, monkeypatch):
    """Tiles factor any rank-1 scaling a_ij = r_i c_j of the 0/1 pattern, not only
    the symmetric s_i s_j: the row-normalised D^-1 (A+I), the column-normalised
    (A+I) D^-1 and random positive r, c all build tiles and match the oracle."""
    torch, dev = torch_dev
    import paper_conf_ipps_kurtysps23_b200 as rdm
    monkeypatch.setenv("RDM_TILE_MIN_NNZ", "1")
    g = synth.rmat(6000, 150000, seed=16)
    deg = np.diff(g.rowptr).astype(np.float64)
    rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    rng = np.random.default_rng(4)
    if norm == "row":
        v = 1.0 / deg[rows]
    elif norm == "col":
        v = 1.0 / deg[g.col]
    else:
        r, c = rng.uniform(0.1, 10, g.n), rng.uniform(0.1, 10, g.n)
        v = r[rows] * c[g.col]
    g2 = synth.CSR(g.n, g.rowptr, g.col, v.astype(np.float32))
    ctx = rdm.Context(device=0)
    ctx.set_graph(g2.rowptr, g2.col, g2.val, symmetric=False)   # values are not symmetric
    assert ctx.graph_info()["n_tiles"] > 0
    for w in (41, 128):
        X = rng.standard_normal((g.n, w)).astype(np.float32)
        xd = _padded(torch, dev, X)
        out = torch.zeros_like(xd)
        ctx.spmm(0, xd, out, w)
        ctx.sync()
        assert og.max_rel_err(out[:, :w].cpu().numpy(), og.spmm(g2, X)) < TOL
        out.zero_()
        ctx.spmm(1, xd, out, w)          # Aᵀ·X from the transpose's own tiles
        ctx.sync()
        assert og.max_rel_err(out[:, :w].cpu().numpy(), og.spmm_t(g2, X)) < TOL
