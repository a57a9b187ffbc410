"""GPU parity of the weight-gradient GEMM (TN, eq. 4 Y = Hᵀ·(A·G), PAPER.md
L79) on CTA pairs (RDM_TN_PAIR=1 forced: M = 256 per pair, each CTA loading its
128 rows of Xᵀ and half of U's 32-wide MN-major chunks) against the fp64
oracle product at the 1e-4 gate — ragged M (a pair's second CTA partly or
wholly past M), N of one or several chunks, split-K chains — and against the
single-CTA kernel (other split count: agreement at fp32 rounding level)."""
import numpy as np
import pytest

from oracle import gcn as og

pytestmark = pytest.mark.gpu

SHAPES = [(5000, 602, 128), (3000, 256, 256), (4097, 300, 41), (2000, 256, 47), (1000, 130, 64),
          (6000, 257, 100)]


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


def _tn(env, monkeypatch, pair, rows, k, m, prec="fp32"):
    torch, dev, rdm = env
    monkeypatch.setenv("RDM_TN_PAIR", "1" if pair else "0")
    ctx = rdm.Context(device=0)
    ctx.set_precision(prec)
    rng = np.random.default_rng(rows + 3 * k + 7 * m)
    X = rng.standard_normal((rows, k)).astype(np.float32)
    U = rng.standard_normal((rows, m)).astype(np.float32)
    Y = torch.zeros((k, m), device=dev)
    ctx.gemm(rdm.GEMM_TN, _padded(torch, dev, X), _padded(torch, dev, U), Y, rows, k, m)
    ctx.sync()
    return X, U, Y.cpu().numpy()


@pytest.mark.parametrize("rows,k,m", SHAPES)
def test_tn_pair_matches_oracle(env, monkeypatch, rows, k, m):
    X, U, Y = _tn(env, monkeypatch, True, rows, k, m)
    ref = X.astype(np.float64).T @ U.astype(np.float64)
    assert og.max_rel_err(Y, ref) < 1e-4
    _, _, Y1 = _tn(env, monkeypatch, False, rows, k, m)
    assert og.max_rel_err(Y, Y1.astype(np.float64)) < 1e-5


@pytest.mark.parametrize("rows,k,m", [(5000, 602, 128), (3000, 256, 256)])
def test_tn_pair_fast_variant(env, monkeypatch, rows, k, m):
    X, U, Y = _tn(env, monkeypatch, True, rows, k, m, prec="fast")
    ref = X.astype(np.float64).T @ U.astype(np.float64)
    assert og.max_rel_err(Y, ref) < 2e-2
