"""GPU parity of the fast variant's kind::f16 GEMM (NN / NT: A rounded to bf16
pairs in TMEM, W as bf16 K-major panels with the 64-byte swizzle) — NEXT-3
(SURVEY §8(f)): within the fast gate (2e-2) of the fp64 oracle product, and
within fp32-accumulation error (1e-5) of the fp64 product of the
bf16-rounded operands, which pins the operand layout exactly (a wrong k
order, swizzle or pair packing moves the result by O(1))."""
import numpy as np
import pytest

from oracle import gcn as og

pytestmark = pytest.mark.gpu

SHAPES = [(1000, 602, 128), (257, 128, 41), (129, 7, 128), (4097, 256, 256), (3000, 128, 602),
          (300, 100, 256), (1, 128, 47), (5000, 41, 128), (640, 1433, 64), (383, 130, 33), (2000, 16, 16)]


def bf16_rne(x):
    """float32 → nearest-even bfloat16, returned as float64 (test-side rounding)."""
    u = np.ascontiguousarray(x, np.float32).view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32).astype(np.float64)


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


@pytest.mark.parametrize("rows,k,m", SHAPES)
def test_f16_gemm_nn_nt(env, monkeypatch, rows, k, m):
    torch, dev, rdm = env
    monkeypatch.setenv("RDM_F16_GEMM", "1")
    ctx = rdm.Context(device=0)
    ctx.set_precision("fast")
    rng = np.random.default_rng(rows + 3 * k + 5 * m)
    X = rng.standard_normal((rows, k)).astype(np.float32)
    W = rng.standard_normal((k, m)).astype(np.float32)
    G = rng.standard_normal((rows, m)).astype(np.float32)
    C = torch.zeros((rows, (m + 3) // 4 * 4), device=dev)
    D = torch.zeros((rows, (k + 3) // 4 * 4), device=dev)
    Wd = torch.from_numpy(W).to(dev)
    ctx.gemm(rdm.GEMM_NN, _padded(torch, dev, X), Wd, C, rows, k, m)
    ctx.gemm(rdm.GEMM_NT, _padded(torch, dev, G), Wd, D, rows, k, m)
    ctx.sync()
    C, D = C[:, :m].cpu().numpy(), D[:, :k].cpu().numpy()
    X64, W64, G64 = X.astype(np.float64), W.astype(np.float64), G.astype(np.float64)
    assert og.max_rel_err(C, X64 @ W64) < 2e-2
    assert og.max_rel_err(D, G64 @ W64.T) < 2e-2
    assert og.max_rel_err(C, bf16_rne(X) @ bf16_rne(W)) < 1e-5
    assert og.max_rel_err(D, bf16_rne(G) @ bf16_rne(W).T) < 1e-5


def test_f16_gemm_epilogues(env, monkeypatch):
    torch, dev, rdm = env
    monkeypatch.setenv("RDM_F16_GEMM", "1")
    ctx = rdm.Context(device=0)
    ctx.set_precision("fast")
    rng = np.random.default_rng(11)
    rows, k, m = 2500, 130, 41
    X = rng.standard_normal((rows, k)).astype(np.float32)
    W = rng.standard_normal((k, m)).astype(np.float32)
    b = rng.standard_normal(m).astype(np.float32)
    Mk = rng.standard_normal((rows, m)).astype(np.float32)
    Xd, Wd = _padded(torch, dev, X), torch.from_numpy(W).to(dev)
    C = torch.zeros((rows, 44), device=dev)
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m, rdm.EPI_RELU | rdm.EPI_BIAS, bias=torch.from_numpy(b).to(dev))
    ctx.sync()
    ref = bf16_rne(X) @ bf16_rne(W)
    assert og.max_rel_err(C[:, :m].cpu().numpy(), np.maximum(ref + b, 0)) < 1e-5
    C.zero_()
    ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m, rdm.EPI_MASK, mask=_padded(torch, dev, Mk))
    ctx.sync()
    assert og.max_rel_err(C[:, :m].cpu().numpy(), ref * (Mk > 0)) < 1e-5
