"""GPU parity of the CTA-pair GEMM (cluster of 2, tcgen05 cta_group::2, M = 256
per pair: each CTA holds 128 rows of A and half of the W panel) against the
fp64 oracle's products (eq. 1 Z = T·W, eq. 3 G·Wᵀ — PAPER.md L71-79), forced
on with RDM_PAIR=1 at sizes with ragged pair tiles (M mod 256 in both CTA
halves, a pair whose second CTA is entirely past M), in both A placements
(RDM_PAIR_ASMEM=0: A in TMEM, bit-identical to the single-CTA kernel — the pair
changes which SM loads which half of B, not the order of any sum;
RDM_PAIR_ASMEM=1: A split in smem, the k steps' MMAs alternating between two
partial accumulators summed in the epilogue — a different summation order,
held to the oracle gate)."""
import numpy as np
import pytest

from oracle import gcn as og

pytestmark = pytest.mark.gpu

TOL = 1e-4

SHAPES = [(1000, 602, 128), (257, 128, 41), (129, 7, 128), (4097, 256, 256), (3000, 128, 602),
          (300, 100, 256), (1, 128, 47), (5000, 41, 128), (640, 1433, 64), (383, 130, 33)]


@pytest.fixture(scope="module")
def env():
    import torch
    import paper_conf_ipps_kurtysps23_b200 as rdm
    return torch, torch.device("cuda:0"), rdm


def _padded(torch, dev, X):
    n, w = X.shape
    t = torch.zeros((n, (w + 3) // 4 * 4), dtype=torch.float32, device=dev)
    t[:, :w] = torch.from_numpy(np.ascontiguousarray(X, np.float32)).to(dev)
    return t


def _run(env, monkeypatch, pair, rows, k, m, epi=0, prec="fp32", bias=None, mask=None, seed=0, asmem=0):
    torch, dev, rdm = env
    monkeypatch.setenv("RDM_PAIR", "1" if pair else "0")
    monkeypatch.setenv("RDM_PAIR_ASMEM", str(asmem))
    ctx = rdm.Context(device=0)
    ctx.set_precision(prec)
    rng = np.random.default_rng(seed + rows + 7 * k + 13 * m)
    X = rng.standard_normal((rows, k)).astype(np.float32)
    W = rng.standard_normal((k, m)).astype(np.float32)
    G = rng.standard_normal((rows, m)).astype(np.float32)
    Xd, Gd = _padded(torch, dev, X), _padded(torch, dev, G)
    Wd = torch.from_numpy(W).to(dev)
    C = torch.zeros((rows, (m + 3) // 4 * 4), device=dev)
    kw = {}
    if bias is not None:
        kw["bias"] = torch.from_numpy(bias).to(dev)
    if mask is not None:
        kw["mask"] = _padded(torch, dev, mask)
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m, epi, **kw)
    D = torch.zeros((rows, (k + 3) // 4 * 4), device=dev)
    ctx.gemm(rdm.GEMM_NT, Gd, Wd, D, rows, k, m)
    ctx.sync()
    return X, W, G, C[:, :m].cpu().numpy(), D[:, :k].cpu().numpy()


@pytest.mark.parametrize("asmem", [0, 1])
@pytest.mark.parametrize("rows,k,m", SHAPES)
def test_pair_gemm_matches_oracle_and_single_cta(env, monkeypatch, rows, k, m, asmem):
    X, W, G, C, D = _run(env, monkeypatch, True, rows, k, m, asmem=asmem)
    X64, W64, G64 = X.astype(np.float64), W.astype(np.float64), G.astype(np.float64)
    assert og.max_rel_err(C, X64 @ W64) < TOL
    assert og.max_rel_err(D, G64 @ W64.T) < TOL
    if asmem == 0:
        _, _, _, C1, D1 = _run(env, monkeypatch, False, rows, k, m)
        assert np.array_equal(C.view(np.uint32), C1.view(np.uint32))
        assert np.array_equal(D.view(np.uint32), D1.view(np.uint32))


@pytest.mark.parametrize("asmem", [0, 1])
@pytest.mark.parametrize("rows,k,m", [(1000, 602, 128), (2500, 130, 41), (700, 256, 256)])
def test_pair_gemm_epilogues(env, monkeypatch, rows, k, m, asmem):
    torch, dev, rdm = env
    rng = np.random.default_rng(5)
    b = rng.standard_normal(m).astype(np.float32)
    Mk = rng.standard_normal((rows, m)).astype(np.float32)
    X, W, _, C, _ = _run(env, monkeypatch, True, rows, k, m, rdm.EPI_RELU | rdm.EPI_BIAS, bias=b, asmem=asmem)
    ref = X.astype(np.float64) @ W + b
    assert og.max_rel_err(C, np.maximum(ref, 0)) < TOL
    X, W, _, C, _ = _run(env, monkeypatch, True, rows, k, m, rdm.EPI_MASK, mask=Mk, asmem=asmem)
    assert og.max_rel_err(C, (X.astype(np.float64) @ W) * (Mk > 0)) < TOL
    if asmem == 0:
        _, _, _, C1, _ = _run(env, monkeypatch, False, rows, k, m, rdm.EPI_MASK, mask=Mk)
        assert np.array_equal(C.view(np.uint32), C1.view(np.uint32))


@pytest.mark.parametrize("asmem", [0, 1])
@pytest.mark.parametrize("rows,k,m", [(1000, 602, 128), (3000, 128, 602), (257, 100, 256)])
def test_pair_gemm_fast_variant(env, monkeypatch, rows, k, m, asmem):
    X, W, G, C, D = _run(env, monkeypatch, True, rows, k, m, prec="fast", asmem=asmem)
    assert og.max_rel_err(C, X.astype(np.float64) @ W) < 2e-2
    assert og.max_rel_err(D, G.astype(np.float64) @ W.T.astype(np.float64)) < 2e-2
    if asmem == 0:
        _, _, _, C1, D1 = _run(env, monkeypatch, False, rows, k, m, prec="fast")
        assert np.array_equal(C.view(np.uint32), C1.view(np.uint32))
        assert np.array_equal(D.view(np.uint32), D1.view(np.uint32))
