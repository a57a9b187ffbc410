"""Cost model oracle — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Layout-tracking simulator of the paper's communication / sparse-operation
model, written from §IV and Tables II–IV:

* Communication-free SpMM needs column-sliced operands, communication-free
  GEMM row-sliced ones (§III-A; §III-D).
* A redistribution of an N×f matrix costs (P−1)/P·N·f (L142); the model
  counts it in units of (P−1)/P·N, i.e. by its width f (Table IV caption L224).
* SpMM cost nnz·f counted in units of nnz (L142, L224).
* Forward S-first: SpMM on H^{l-1} (width f_{l-1}) then col→row of the
  product (f_{l-1}); D-first: GEMM, row→col of the product (f_l), SpMM (f_l)
  (Table II).
* Consecutive layers leaving the operand in the wrong layout pay an extra
  redistribution of width f_l (L210).
* The loss needs rows whole: redistribute Z^L (width f_L) if column-sliced
  (L206; reading R17 — the printed "(P−1)/P·N" lacks the ×f_L).
* Backward is the mirror image (L208, Table III); a GEMM-first backward layer
  whose forward layer was not SpMM-first (no memo of AᵀH^{l-1}, L118–127)
  pays one extra SpMM of width min(f_{l-1}, f_l) and 2·min(...)
  redistribution (Table III N.M. rows; reading R20).
* H^0 is available in both layouts at no charge (reading R12).

Configuration ID for L = 2 (reading R18, Fig. 4 "ID 10 =
dense-sparse-dense-sparse"):  ID = 8·[bwd L2=D] + 4·[bwd L1=D] + 2·[fwd L1=D]
+ [fwd L2=D]; in general the ID bits MSB→LSB are [bwd L … bwd 1, fwd 1 … fwd L]
(reading R22).
"""
from __future__ import annotations

from itertools import product

S, D = 0, 1
ROW, COL = "R", "C"


def decode(cfg_id: int, L: int):
    """ID → (fwd[1..L], bwd[1..L]) with 1 = D (GEMM first), 0 = S (SpMM first)."""
    bits = [(cfg_id >> (2 * L - 1 - i)) & 1 for i in range(2 * L)]  # MSB first
    bwd_desc = bits[:L]          # bwd L, ..., bwd 1
    fwd_asc = bits[L:]           # fwd 1, ..., fwd L
    fwd = {l: fwd_asc[l - 1] for l in range(1, L + 1)}
    bwd = {l: bwd_desc[L - l] for l in range(1, L + 1)}
    return fwd, bwd


def encode(fwd: dict, bwd: dict, L: int) -> int:
    bits = [bwd[l] for l in range(L, 0, -1)] + [fwd[l] for l in range(1, L + 1)]
    v = 0
    for b in bits:
        v = (v << 1) | b
    return v


def name(cfg_id: int, L: int) -> str:
    fwd, bwd = decode(cfg_id, L)
    sd = "SD"
    return "F" + "".join(sd[fwd[l]] for l in range(1, L + 1)) + "/B" + "".join(
        sd[bwd[l]] for l in range(L, 0, -1))


def simulate(cfg_id: int, f) -> tuple:
    """(comm units, sparse units) of configuration `cfg_id` for widths f = (f_0..f_L)."""
    L = len(f) - 1
    fwd, bwd = decode(cfg_id, L)
    comm = 0
    sparse = 0
    H = {0: {ROW, COL}}
    memo = {}
    for l in range(1, L + 1):
        if fwd[l] == S:
            if COL not in H[l - 1]:
                comm += f[l - 1]
                H[l - 1].add(COL)
            sparse += f[l - 1]      # T = Aᵀ H^{l-1}
            comm += f[l - 1]        # T: col → row (kept as memo, L134)
            memo[l] = True
            H[l] = {ROW}
        else:
            if ROW not in H[l - 1]:
                comm += f[l - 1]
                H[l - 1].add(ROW)
            comm += f[l]            # T = H W: row → col
            sparse += f[l]          # Z = Aᵀ T
            memo[l] = False
            H[l] = {COL}
    if ROW not in H[L]:              # loss needs whole rows (L206)
        comm += f[L]
    G = {L: {ROW}}
    for l in range(L, 0, -1):
        if bwd[l] == S:
            if COL not in G[l]:
                comm += f[l]
                G[l].add(COL)
            sparse += f[l]          # U = A G^l
            comm += f[l]            # U: col → row
            G[l - 1] = {ROW}
        else:
            if ROW not in G[l]:
                comm += f[l]
                G[l].add(ROW)
            comm += f[l - 1]        # V = G W^T: row → col
            sparse += f[l - 1]      # A V
            G[l - 1] = {COL}
            if not memo[l]:         # Table III N.M. rows
                mn = min(f[l - 1], f[l])
                sparse += mn
                comm += 2 * mn
    return comm, sparse


def all_costs(f) -> dict:
    L = len(f) - 1
    return {i: simulate(i, f) for i in range(4 ** L)}


def pareto(costs: dict) -> list:
    """Non-dominated configs in (comm, sparse): dominated = ≥ in both and > in one.
    Configurations with equal costs are all kept (reading R23)."""
    front = []
    for i, (c, s) in costs.items():
        dominated = any((c2 <= c and s2 <= s and (c2 < c or s2 < s)) for j, (c2, s2) in costs.items())
        if not dominated:
            front.append(i)
    return sorted(front)


def pareto_front(f) -> list:
    return pareto(all_costs(f))


def table_iv_symbolic(cfg_id: int, fin, fh, fout) -> tuple:
    """Table IV as printed for rows 0–12, 14, with the
    derived values for the two rows whose printed entries are inconsistent
    (reading R19): row 13's comm is a copy of row 9's; row 15 matches no config."""
    mn1, mn2 = min(fin, fh), min(fh, fout)
    t = {
        0: (fin + 4 * fh + 2 * fout, fin + 2 * fh + fout),
        1: (fin + 2 * fh + 4 * fout, fin + fh + 2 * fout),
        2: (4 * fh + 2 * fout, 3 * fh + fout),
        3: (4 * fh + 4 * fout, 2 * fh + 2 * fout),
        4: (2 * fin + 2 * fh + 2 * fout, 2 * fin + fh + fout),
        5: (2 * fin + 4 * fout, 2 * fin + 2 * fout),
        6: (fin + 2 * fh + 2 * fout + 2 * mn1, fin + 2 * fh + fout + mn1),
        7: (fin + 2 * fh + 4 * fout + 2 * mn1, fin + fh + 2 * fout + mn1),
        8: (fin + 4 * fh, fin + 3 * fh),
        9: (fin + 2 * fh + 2 * fout + 2 * mn2, fin + 2 * fh + fout + mn2),
        10: (4 * fh, 4 * fh),
        11: (4 * fh + 2 * fout + 2 * mn2, 3 * fh + fout + mn2),
        12: (2 * fin + 4 * fh, 2 * fin + 2 * fh),
        13: (2 * fin + 2 * fh + 2 * fout + 2 * mn2, 2 * fin + fh + fout + mn2),
        14: (fin + 4 * fh + 2 * mn1, fin + 3 * fh + mn1),
        15: (fin + 4 * fh + 2 * fout + 2 * mn1 + 2 * mn2, fin + 2 * fh + fout + mn1 + mn2),
    }
    return t[cfg_id]


# ---------------------------------------------------------------- R_A < P
# §III-E (Fig. 6) and the "Comm. (R_A < P)" rows of
# Tables II/III (L185-202), §IV-A.4 (L214-216).  P GPUs form a grid of
# P/R_A row panels x R_A column groups; A's row panel i is held by the R_A GPUs
# of panel group i (R_A copies of A in total).  Dense operands of the SpMM are
# (P/R_A) x R_A tiles (panel rows x column slice).  Reading R35: every
# redistribution of width f moves (R_A-1)/R_A·N·f elements (inside a panel
# group, L214), and every SpMM of width f additionally broadcasts its input
# tiles inside the column group, (P/R_A-1)·N·f elements (L152, L216); the
# printed R_A rows of Table III, which mix f_{l-1} and f_l and drop the
# broadcast term of the GEMM-first row, are read by that same rule.

def comm_elements_ra(cfg_id: int, f, n: int, P: int, RA: int) -> float:
    """Elements moved per epoch by configuration `cfg_id` at R_A = RA (R35)."""
    assert 1 <= RA <= P and P % RA == 0
    comm, sparse = simulate(cfg_id, f)
    return n * ((RA - 1) / RA * comm + (P / RA - 1) * sparse)


def layer_comm_ra(f_in: int, n: int, P: int, RA: int) -> float:
    """Table II "Comm. (R_A < P)" entry for one forward layer whose SpMM and
    redistribution both have width f_in (as printed, L185-189)."""
    return (RA - 1) / RA * n * f_in + (P / RA - 1) * n * f_in


def max_replication(P: int, mem_bytes: float, h_all_bytes: float, g_bytes: float) -> int:
    """L160-167: R_A = P·(M − H_all)/G replicas fit, at most P ("when this
    number is larger than P we are going to use R_A = P").  Reading R36: the
    grid needs R_A | P, so the largest divisor of P not above that bound; 0 if
    not even one copy of A fits in the aggregate memory."""
    bound = P * (mem_bytes - h_all_bytes) / g_bytes if g_bytes > 0 else P
    cap = min(P, int(bound)) if bound >= 1 else 0
    for r in range(cap, 0, -1):
        if P % r == 0:
            return r
    return 0


def pareto_ra(f, n: int, P: int, RA: int) -> list:
    """Pareto front in (elements moved at R_A, sparse units)."""
    L = len(f) - 1
    costs = {i: (comm_elements_ra(i, f, n, P, RA), simulate(i, f)[1]) for i in range(4 ** L)}
    return pareto(costs)
