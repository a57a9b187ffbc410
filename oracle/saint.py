"""GraphSAINT-RDM sampler oracle — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md §III-F (L169–173): "graph-sampling to create independently processed
subgraphs, e.g., GraphSaint GCN [17]"; "a random generated seed can be passed
to all processes and each process can generate its sparse mask
individually".  §V-C (L388–390): "each subgraph is parallelized using our RDM
scheme"; the weights are updated after each subgraph.

The paper does not state the sampler's parameters; DESIGN.md readings:
  R31  random-walk sampler (GraphSAINT [17], BASELINE config 4): `roots`
       walks of `walk_len` steps (4) over the stored CSR entries of Â (self
       loops included: a lazy walk); node set = sorted set of visited ids.
  R32  subgraph = the induced one on the node set, re-normalised as a fresh
       GCN graph: Â_s[i][j] = 1/sqrt(d_i d_j), d_i = kept entries of row i,
       entries in the original row order; GraphSAINT's α/λ estimators are
       not applied (accuracy is out of scope).
  R33  counter-based draws: key = splitmix64(seed + it·φ) with
       φ = 0x9E3779B97F4A7C15; u(i, j) = splitmix64(key ^ (i << 8 | j));
       root i = u(i, 0) mod N; step j: next = col[rowptr[v] + u(i, j) mod deg v].
  R34  the subgraph's loss is the mean over its train-mask vertices; one
       Adam step per subgraph (L390).

Everything here is a plain transcription: python integers for the hash,
explicit loops for the walk, numpy only as arrays.
"""
from __future__ import annotations

import numpy as np

M64 = (1 << 64) - 1
PHI = 0x9E3779B97F4A7C15


def splitmix64(x: int) -> int:
    """Vigna's SplitMix64 output function for state x (the generator's next()
    after `state += φ`).  R33."""
    z = (x + PHI) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def walks(rowptr, col, n: int, roots: int, walk_len: int, seed: int, it: int) -> np.ndarray:
    """Visited vertices, roots × (walk_len + 1): R31 + R33."""
    key = splitmix64((seed + it * PHI) & M64)
    out = np.empty((roots, walk_len + 1), dtype=np.int64)
    for i in range(roots):
        base = i << 8
        v = splitmix64(key ^ base) % n
        out[i, 0] = v
        for j in range(1, walk_len + 1):
            b, e = int(rowptr[v]), int(rowptr[v + 1])
            if e > b:
                v = int(col[b + splitmix64(key ^ (base | j)) % (e - b)])
            out[i, j] = v
    return out


def node_set(visits: np.ndarray) -> np.ndarray:
    """Sorted distinct visited vertices (new id = position).  R31."""
    return np.unique(visits.reshape(-1))


def induced(rowptr, col, nodes: np.ndarray):
    """Induced, re-normalised subgraph (R32): returns rowptr_s (int64),
    col_s (int32, new ids, original row order), val_s (float32)."""
    n = len(nodes)
    nodes = np.asarray(nodes, dtype=np.int64)
    new_id = np.full(len(rowptr) - 1, -1, dtype=np.int64)   # new id of every vertex, -1 = not sampled
    new_id[nodes] = np.arange(n)
    # every stored entry of every sampled row, in row order then original entry order
    starts, ends = rowptr[nodes], rowptr[nodes + 1]
    row_of = np.repeat(np.arange(n), ends - starts)
    entry = np.concatenate([np.arange(b, e) for b, e in zip(starts, ends)]) if n else np.zeros(0, np.int64)
    j = new_id[col[entry]]
    keep = j >= 0                                            # both ends sampled
    row_of, j = row_of[keep], j[keep]
    deg = np.bincount(row_of, minlength=n).astype(np.int64)  # d_i = kept entries of row i
    rp = np.zeros(n + 1, dtype=np.int64)
    rp[1:] = np.cumsum(deg)
    vals = (1.0 / np.sqrt(deg[row_of].astype(np.float64) * deg[j].astype(np.float64))).astype(np.float32)
    return rp, j.astype(np.int32), vals


def sample(g, roots: int, walk_len: int, seed: int, it: int):
    """Subgraph `it`: (nodes, rowptr_s, col_s, val_s)."""
    nodes = node_set(walks(g.rowptr, g.col, g.n, roots, walk_len, seed, it))
    rp, cs, vs = induced(g.rowptr, g.col, nodes)
    return nodes, rp, cs, vs
