"""fp64 GCN oracle — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The plain definition the GNN-RDM hot path must reproduce.  RDM reorders
(associativity), reuses identical intermediates (L118–127) and
moves data (L140–142); "all three implementations compute identical outputs,
with small differences due to reordering of floating point operations" (L323).
So the oracle is the undistributed definition, in fp64:

Forward, eq. (1)(2) (L69–73), l = 1..L:
    Z^l = Aᵀ H^{l-1} W^l  (+ 1·b^lᵀ, reading R8)
    H^l = ReLU(Z^l) for l < L;  logits = Z^L           (reading R4)
Loss (L206; reading R5): mean softmax cross-entropy over the train mask.
Backward, eq. (3)(4) (L75–79) with G^l = ∂ℓ/∂Z^l (reading R1), l = L..1:
    S^l = A G^l;  Y^l = (H^{l-1})ᵀ S^l;  db^l = 1ᵀ G^l
    G^{l-1} = S^l (W^l)ᵀ ⊙ 1[Z^{l-1} > 0]   (l > 1)
    G^0     = S^1 (W^1)ᵀ                     (reading R2)
Adam (L297: lr 0.01; reading R10: PyTorch defaults β=(0.9,0.999), ε=1e-8).

Library primitives used as steps: numpy fp64 matmul (dense GEMM), the C
loops in oracle/spmm.c (sparse products by definition).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import lib as _lib

_vp = None


def _ptr(a):
    import ctypes
    return a.ctypes.data_as(ctypes.c_void_p)


def spmm(A, X: np.ndarray) -> np.ndarray:
    """A·X in fp64 (A: synth.CSR; X: N×f).  Used by eqs. (3)(4)."""
    X = np.ascontiguousarray(X, dtype=np.float64)
    Y = np.empty_like(X)
    _lib().oracle_spmm(A.n, _ptr(A.rowptr), _ptr(A.col), _ptr(A.val), _ptr(X), X.shape[1], _ptr(Y))
    return Y


def spmm_t(A, X: np.ndarray) -> np.ndarray:
    """Aᵀ·X in fp64 — the aggregation of eq. (1) (L69: "the transpose of adjacency matrix A")."""
    X = np.ascontiguousarray(X, dtype=np.float64)
    Y = np.empty_like(X)
    _lib().oracle_spmm_t(A.n, _ptr(A.rowptr), _ptr(A.col), _ptr(A.val), _ptr(X), X.shape[1], _ptr(Y))
    return Y


def spmm_rows(A, X: np.ndarray, rows: np.ndarray) -> np.ndarray:
    """Rows `rows` of A·X (X fp32, any leading dim) in fp64 — sampled parity at full size."""
    X = np.asarray(X, dtype=np.float32)
    assert X.strides[1] == 4
    ldx = X.strides[0] // 4
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    f = X.shape[1]
    Y = np.empty((len(rows), f), dtype=np.float64)
    _lib().oracle_spmm_rows(_ptr(A.rowptr), _ptr(A.col), _ptr(A.val), _ptr(X), ldx, f,
                            _ptr(rows), len(rows), _ptr(Y))
    return Y


def relu(x):
    return np.maximum(x, 0.0)


def layer_forward(A, H: np.ndarray, W: np.ndarray, order: str = "S", b=None) -> np.ndarray:
    """One eq. (1) product in either association (L116): 'S' = (AᵀH)W, 'D' = Aᵀ(HW).
    Bias, if any, is added after both products (reading R8)."""
    W = np.asarray(W, dtype=np.float64)
    if order == "S":
        Z = spmm_t(A, H) @ W
    else:
        Z = spmm_t(A, np.asarray(H, np.float64) @ W)
    if b is not None:
        Z = Z + np.asarray(b, np.float64)[None, :]
    return Z


def softmax_xent(logits: np.ndarray, labels: np.ndarray, mask: np.ndarray, n_train=None):
    """Mean softmax cross-entropy over mask rows (reading R5) and its gradient
    G^L = (softmax − onehot(y)) ⊙ m / n_train.  Max-subtracted log-sum-exp."""
    Z = np.asarray(logits, np.float64)
    m = np.asarray(mask).astype(bool)
    if n_train is None:
        n_train = int(m.sum())
    zmax = Z.max(axis=1, keepdims=True)
    e = np.exp(Z - zmax)
    s = e.sum(axis=1, keepdims=True)
    lse = (zmax + np.log(s))[:, 0]
    rows = np.arange(Z.shape[0])
    per_row = lse - Z[rows, labels]
    loss = float(per_row[m].sum() / n_train) if n_train else 0.0
    G = e / s
    G[rows, labels] -= 1.0
    G *= (m[:, None] / n_train) if n_train else 0.0
    return loss, G


@dataclass
class Result:
    H: list                 # H^0 .. H^{L-1} (fp64)
    Z: list                 # Z^1 .. Z^L (index 0 unused → None)
    loss: float
    G: list = field(default_factory=list)    # G^0 .. G^L
    Y: list = field(default_factory=list)    # Y^1 .. Y^L (index 0 None)
    db: list = field(default_factory=list)


def forward(A, H0, Ws, labels, mask, bs=None, orders=None) -> Result:
    """eqs. (1)(2) for all layers + loss.  `orders[l-1]` picks the association of
    layer l (default 'S'); results agree up to rounding (L116, L323)."""
    L = len(Ws)
    H = [np.asarray(H0, np.float64)]
    Z = [None]
    for l in range(1, L + 1):
        o = orders[l - 1] if orders else "S"
        Zl = layer_forward(A, H[l - 1], Ws[l - 1], o, None if bs is None else bs[l - 1])
        Z.append(Zl)
        if l < L:
            H.append(relu(Zl))
    loss, GL = softmax_xent(Z[L], labels, mask)
    res = Result(H=H, Z=Z, loss=loss)
    res._GL = GL
    return res


def backward(A, res: Result, Ws) -> Result:
    """eqs. (3)(4) with G^l = ∂ℓ/∂Z^l (reading R1), G^0 without Hadamard (R2).
    σ'(Z^l) = 1[Z^l > 0] is taken from this oracle's own forward `res.Z`."""
    L = len(Ws)
    G = [None] * (L + 1)
    Y = [None] * (L + 1)
    db = [None] * (L + 1)
    G[L] = res._GL
    for l in range(L, 0, -1):
        S = spmm(A, G[l])                       # A G^l
        Y[l] = res.H[l - 1].T @ S               # eq. (4)
        db[l] = G[l].sum(axis=0)
        D = S @ np.asarray(Ws[l - 1], np.float64).T   # A G^l (W^l)ᵀ
        if l > 1:
            G[l - 1] = D * (res.Z[l - 1] > 0)   # eq. (3), σ'(Z) = 1[Z > 0]
        else:
            G[0] = D
    res.G, res.Y, res.db = G, Y, db
    return res


def epoch(A, H0, Ws, labels, mask, bs=None):
    res = forward(A, H0, Ws, labels, mask, bs)
    return backward(A, res, Ws)


def adam(p, g, m, v, step, lr=0.01, b1=0.9, b2=0.999, eps=1e-8):
    """torch.optim.Adam update (no weight decay, no amsgrad), fp64.  Returns (p, m, v)."""
    p = np.asarray(p, np.float64)
    g = np.asarray(g, np.float64)
    m = b1 * np.asarray(m, np.float64) + (1.0 - b1) * g
    v = b2 * np.asarray(v, np.float64) + (1.0 - b2) * g * g
    mhat = m / (1.0 - b1 ** step)
    vhat = v / (1.0 - b2 ** step)
    p = p - lr * mhat / (np.sqrt(vhat) + eps)
    return p, m, v


def max_rel_err(x, ref) -> float:
    """Normwise max-relative error max|x−r| / max|r| (reading R26).

    Shapes must match exactly (no broadcasting); a non-finite entry in x gives
    inf; an empty pair gives 0; an all-zero reference gives the absolute error."""
    x = np.asarray(x, np.float64)
    ref = np.asarray(ref, np.float64)
    if x.shape != ref.shape:
        raise ValueError(f"max_rel_err: shape {x.shape} vs reference {ref.shape}")
    if ref.size == 0:
        return 0.0
    if not np.all(np.isfinite(x)):
        return float("inf")
    den = float(np.abs(ref).max())
    num = float(np.abs(x - ref).max())
    if den == 0.0:
        return num
    return num / den
