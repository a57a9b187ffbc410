"""Seeded synthetic inputs shared by the oracle (``oracle/``) and the CUDA path.

This module holds none of the GNN-RDM method's arithmetic: it draws graphs,
features, labels and initial weights (recipe in DESIGN.md "Input recipe").
Large draws go through ``synth/libsynth.so`` (C++/OpenMP, counter-based
hashes, deterministic for any thread count); the tiny hand-built graphs used
by the closed-form pins are constructed here directly.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsynth.so")
_lib = None

# Seeds recorded in every bench record: graph 1, H 2, W 3, labels 4.
SEED_GRAPH, SEED_H, SEED_W, SEED_LABELS = 1, 2, 3, 4


def _build():
    src = os.path.join(_HERE, "gen.cpp")
    subprocess.check_call(["g++", "-O3", "-fopenmp", "-fPIC", "-shared", "-std=c++17",
                           src, "-o", _LIB_PATH])


def lib():
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "gen.cpp")
        if (not os.path.exists(_LIB_PATH)) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            _build()
        L = ctypes.CDLL(_LIB_PATH)
        i64, u64, dbl, vp = ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p
        L.synth_rmat_csr.argtypes = [i64, i64, u64, dbl, dbl, dbl, ctypes.c_int, ctypes.c_int, vp, vp, vp]
        L.synth_rmat_csr.restype = ctypes.c_int
        L.synth_features.argtypes = [i64, i64, u64, vp]
        L.synth_features_rows.argtypes = [i64, i64, i64, u64, vp]
        L.synth_labels_rows.argtypes = [i64, i64, i64, u64, vp]
        L.synth_glorot.argtypes = [i64, i64, u64, vp]
        L.synth_labels.argtypes = [i64, i64, u64, vp]
        L.synth_mask.argtypes = [i64, dbl, u64, vp]
        L.synth_splitmix64.argtypes = [u64]
        L.synth_splitmix64.restype = u64
        L.synth_num_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


@dataclass
class CSR:
    """CSR adjacency: int64 rowptr[n+1], int32 col[nnz], fp32 val[nnz]."""
    n: int
    rowptr: np.ndarray
    col: np.ndarray
    val: np.ndarray

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.rowptr)


def rmat(n: int, n_edges: int, seed: int = SEED_GRAPH, abc=(0.57, 0.19, 0.19),
         permute: bool = True, normalize: bool = True) -> CSR:
    """Symmetric R-MAT graph with one self loop per vertex; nnz = 2*n_edges + n."""
    nnz = 2 * n_edges + n
    rowptr = np.empty(n + 1, dtype=np.int64)
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=np.float32)
    rc = lib().synth_rmat_csr(n, n_edges, seed, abc[0], abc[1], abc[2], int(permute),
                              int(normalize), _p(rowptr), _p(col), _p(val))
    if rc != 0:
        raise RuntimeError(f"synth_rmat_csr failed rc={rc}")
    return CSR(n, rowptr, col, val)


def erdos_renyi(n: int, n_edges: int, seed: int = SEED_GRAPH, normalize: bool = True) -> CSR:
    """Uniform random graph (R-MAT with a=b=c=d=1/4), same conventions as rmat()."""
    return rmat(n, n_edges, seed, abc=(0.25, 0.25, 0.25), permute=True, normalize=normalize)


def features(n: int, f: int, seed: int = SEED_H) -> np.ndarray:
    out = np.empty((n, f), dtype=np.float32)
    if n * f:
        lib().synth_features(n, f, seed, _p(out))
    return out


def features_rows(lo: int, hi: int, f: int, seed: int = SEED_H) -> np.ndarray:
    """Rows [lo, hi) of features(n, f, seed) (identical values)."""
    out = np.empty((hi - lo, f), dtype=np.float32)
    if (hi - lo) * f:
        lib().synth_features_rows(lo, hi, f, seed, _p(out))
    return out


def labels_rows(lo: int, hi: int, C: int, seed: int = SEED_LABELS) -> np.ndarray:
    """Entries [lo, hi) of labels(n, C, seed)."""
    out = np.empty(hi - lo, dtype=np.int32)
    if hi > lo:
        lib().synth_labels_rows(lo, hi, C, seed, _p(out))
    return out


def glorot(fin: int, fout: int, seed: int = SEED_W) -> np.ndarray:
    out = np.empty((fin, fout), dtype=np.float32)
    lib().synth_glorot(fin, fout, seed, _p(out))
    return out


def weights(f, seed: int = SEED_W):
    """Glorot-uniform W^l for l = 1..L (one sub-seed per layer)."""
    return [glorot(f[l - 1], f[l], seed * 1000 + l) for l in range(1, len(f))]


def labels(n: int, C: int, seed: int = SEED_LABELS) -> np.ndarray:
    out = np.empty(n, dtype=np.int32)
    lib().synth_labels(n, C, seed, _p(out))
    return out


def train_mask(n: int, frac: float = 1.0, seed: int = 5) -> np.ndarray:
    out = np.empty(n, dtype=np.uint8)
    lib().synth_mask(n, frac, seed, _p(out))
    return out


# ---------------------------------------------------------------- tiny graphs
def from_edges(n: int, rows, cols, vals=None) -> CSR:
    """CSR from explicit (row, col[, val]) triples (duplicates not merged; rows sorted)."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    vals = np.ones(len(rows), dtype=np.float32) if vals is None else np.asarray(vals, dtype=np.float32)
    order = np.lexsort((cols, rows))
    rows, cols, vals = rows[order], cols[order], vals[order]
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(rowptr, rows + 1, 1)
    rowptr = np.cumsum(rowptr).astype(np.int64)
    return CSR(n, rowptr, cols.astype(np.int32), vals)


def normalize_sym(g: CSR) -> CSR:
    """Â = D^{-1/2} A D^{-1/2} with D the row sums of the given 0/1 pattern (fp64 → fp32)."""
    deg = np.diff(g.rowptr).astype(np.float64)
    rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    v = 1.0 / np.sqrt(deg[rows] * deg[g.col])
    return CSR(g.n, g.rowptr.copy(), g.col.copy(), v.astype(np.float32))


def identity_graph(n: int) -> CSR:
    return from_edges(n, np.arange(n), np.arange(n))


def complete_graph(n: int) -> CSR:
    """K_n with self loops, normalized: Â = J / n exactly (up to fp32 rounding of 1/n)."""
    r, c = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    return normalize_sym(from_edges(n, r.ravel(), c.ravel()))


def star_graph(n: int) -> CSR:
    """Hub 0 connected to all others, plus self loops: one row of degree n."""
    hub = np.zeros(n - 1, dtype=np.int64)
    leaves = np.arange(1, n)
    rows = np.concatenate([hub, leaves, np.arange(n)])
    cols = np.concatenate([leaves, hub, np.arange(n)])
    return normalize_sym(from_edges(n, rows, cols))


def random_directed(n: int, nnz: int, seed: int = 11, empty_rows: int = 0) -> CSR:
    """Non-symmetric random CSR with arbitrary real values (A != Aᵀ); optional empty rows."""
    rng = np.random.default_rng(seed)
    rows = rng.integers(0, n, size=nnz)
    if empty_rows:
        dead = rng.choice(n, size=empty_rows, replace=False)
        keep = ~np.isin(rows, dead)
        rows = rows[keep]
    cols = rng.integers(0, n, size=len(rows))
    key = np.unique(rows * n + cols)
    rows, cols = key // n, key % n
    vals = rng.standard_normal(len(rows)).astype(np.float32)
    return from_edges(n, rows, cols, vals)


# --------------------------------------------------------- named workloads
@dataclass(frozen=True)
class Workload:
    name: str
    n: int
    n_edges: int          # undirected edges before self loops: nnz = 2*n_edges + n
    f: tuple              # (f_0, ..., f_L)
    graph: str = "rmat"   # "rmat" (Graph500 a,b,c,d) or "er" (uniform)
    permute: bool = True  # seeded vertex permutation (Graph500: worst-case locality)
    values: str = "sym"   # "sym": D^-1/2 (A+I) D^-1/2; "noise": sym x (1 + 2^-4 u_ij), u_ij = u_ji
                          # (symmetric, not a rank-1 scaling); "row": D^-1 (A+I) (not symmetric)

    @property
    def nnz(self) -> int:
        return 2 * self.n_edges + self.n

    @property
    def L(self) -> int:
        return len(self.f) - 1


# BASELINE.json configs (shapes from PAPER.md Table V; hidden sizes L297)
WORKLOADS = {
    "cora": Workload("cora-shaped 2L h128", 2708, 5278, (1433, 128, 7)),
    "reddit": Workload("reddit-shaped 2L h128", 232965, 57307946, (602, 128, 41)),
    "products": Workload("products-shaped 3L h256", 2449029, 61859140, (100, 256, 256, 47)),
    "papers": Workload("papers100M-shaped 2L h128", 111059956, 799470022, (128, 128, 172)),
    # controls for the input specialisations: uniform graph, values
    # that are not a rank-1 scaling of the pattern, row-normalised values, and
    # the un-permuted (locality-preserving) R-MAT order
    "reddit-er": Workload("reddit-shaped ER 2L h128", 232965, 57307946, (602, 128, 41), graph="er"),
    "reddit-noise": Workload("reddit-shaped, non-factorable values 2L h128", 232965, 57307946, (602, 128, 41),
                             values="noise"),
    "reddit-row": Workload("reddit-shaped, row-normalised 2L h128", 232965, 57307946, (602, 128, 41),
                           values="row"),
    "products-er": Workload("products-shaped ER 3L h256", 2449029, 61859140, (100, 256, 256, 47), graph="er"),
    "papers-local": Workload("papers100M-shaped, un-permuted 2L h128", 111059956, 799470022, (128, 128, 172),
                             permute=False),
}


def make_graph(w: Workload, seed: int = SEED_GRAPH) -> CSR:
    if w.graph == "er":
        g = erdos_renyi(w.n, w.n_edges, seed)
    else:
        g = rmat(w.n, w.n_edges, seed, permute=w.permute)
    if w.values == "noise":
        rows = np.repeat(np.arange(g.n, dtype=np.int64), np.diff(g.rowptr))
        lo = np.minimum(rows, g.col).astype(np.uint64)
        hi = np.maximum(rows, g.col).astype(np.uint64)
        h = (lo * np.uint64(0x9E3779B97F4A7C15)) ^ (hi * np.uint64(0xBF58476D1CE4E5B9))
        h ^= h >> np.uint64(29)
        h *= np.uint64(0x94D049BB133111EB)
        h ^= h >> np.uint64(32)
        u = (h >> np.uint64(40)).astype(np.float64) / 16777216.0
        g = CSR(g.n, g.rowptr, g.col, (g.val.astype(np.float64) * (1.0 + u / 16.0)).astype(np.float32))
    elif w.values == "row":
        deg = np.diff(g.rowptr).astype(np.float64)
        rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
        g = CSR(g.n, g.rowptr, g.col, (1.0 / deg[rows]).astype(np.float32))
    return g


def symmetric_values(w: Workload) -> bool:
    """Whether make_graph(w)'s values satisfy A = Aᵀ (rdm_set_graph's `symmetric`)."""
    return w.values != "row"
