"""Virtual-rank redistribution oracle — TEST INFRASTRUCTURE ONLY.

Row ("horizontal") and column ("vertical") slicing of an N×f dense matrix
over P processes, and the all-to-all personalized redistribution between them
(§III-D, Fig. 7 / L212: divide into P chunks → exchange →
merge).  Redistribution is pure data movement, so the oracle is the slicing of
the full matrix itself: the result on rank p must equal that slice.

Partition (reading R11 — the paper only draws even halves, Fig. 5/7):
  rows    lo_p = ⌊p·N/P⌋
  columns 4-float granules: g = ⌈f/4⌉, lo_p = min(f, 4·⌊p·g/P⌋)
"""
from __future__ import annotations

import numpy as np


def row_range(n: int, P: int, p: int):
    return (p * n) // P, ((p + 1) * n) // P


def col_range(f: int, P: int, p: int):
    g = -(-f // 4)

    def lo(q):
        return f if q >= P else min(f, 4 * ((q * g) // P))

    return lo(p), lo(p + 1) if p + 1 < P else f


def row_slices(M: np.ndarray, P: int):
    n = M.shape[0]
    return [M[slice(*row_range(n, P, p))].copy() for p in range(P)]


def col_slices(M: np.ndarray, P: int):
    f = M.shape[1]
    return [M[:, slice(*col_range(f, P, p))].copy() for p in range(P)]


def send_elements(n: int, f: int, P: int, p: int, q: int, direction: str) -> int:
    """Elements rank p sends to rank q in one redistribution of an n×f matrix.
    row→col: p owns rows_p, q needs cols_q → rows_p × w_q.
    col→row: p owns cols_p, q needs rows_q → rows_q × w_p."""
    if p == q:
        return 0
    r0, r1 = row_range(n, P, p if direction == "row2col" else q)
    c0, c1 = col_range(f, P, q if direction == "row2col" else p)
    return (r1 - r0) * (c1 - c0)


def total_elements(n: int, f: int, P: int) -> int:
    """Elements crossing ranks in one redistribution: ≈ (P−1)/P·N·f (L142), exact form."""
    return sum(send_elements(n, f, P, p, q, "row2col") for p in range(P) for q in range(P))


def redistribute_row2col(slices, P: int):
    """Assemble rank p's column slice from the P row slices (Fig. 7a)."""
    M = np.concatenate(slices, axis=0)
    return col_slices(M, P)


def redistribute_col2row(slices, P: int):
    """Assemble rank p's row slice from the P column slices (Fig. 7b)."""
    M = np.concatenate(slices, axis=1)
    return row_slices(M, P)
