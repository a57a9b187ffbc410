"""CPU-only checks of the C-ABI library: it loads, exports every symbol
include/rdm.h declares, and its pure host functions (partition, cost model,
selector, executor plan, exchange plan) agree with the oracle."""
import os
import random
import re
import subprocess

import numpy as np
import pytest

import paper_conf_ipps_kurtysps23_b200 as rdm
from oracle import cost_model as ocm
from oracle import redistribution as ordist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    txt = open(os.path.join(ROOT, "include", "rdm.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(rdm_[a-z_0-9]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    declared = _header_functions()
    out = subprocess.run(["nm", "-D", "--defined-only", rdm.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r" T (rdm_\w+)", out))
    missing = [f for f in declared if f not in exported]
    assert not missing, missing
    assert set(rdm.EXPORTS) <= set(declared)
    assert len(declared) >= 30


def test_library_is_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", rdm.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_tensor_core_and_tma_in_sass():
    """The GEMM is tcgen05 (UTC*MMA) fed by TMA (UTMALDG), epilogue via LDTM."""
    out = subprocess.run(["cuobjdump", "-sass", rdm.LIB_PATH], capture_output=True, text=True).stdout
    assert re.search(r"UTC\w*MMA", out)
    assert "UTMALDG" in out
    assert "LDTM" in out


@pytest.mark.parametrize("n,f,P", [(10, 7, 8), (2708, 1433, 8), (5, 3, 8), (100, 41, 3),
                                   (232965, 602, 8), (1, 1, 2), (0, 4, 2)])
def test_partition_matches_oracle(n, f, P):
    for p in range(P):
        lo, hi, ld = rdm.partition(P, rdm.ROW, n, f, p)
        assert (lo, hi) == ordist.row_range(n, P, p) and ld == (f + 3) // 4 * 4
        lo, hi, ld = rdm.partition(P, rdm.COL, n, f, p)
        assert (lo, hi) == ordist.col_range(f, P, p) and ld == (hi - lo + 3) // 4 * 4


def test_config_id_roundtrip():
    for L in (1, 2, 3, 4):
        for i in range(4 ** L):
            c = rdm.config_from_id(L, i)
            assert rdm.config_to_id(c) == i
            fwd, bwd = ocm.decode(i, L)
            assert [c.fwd_D[l - 1] for l in range(1, L + 1)] == [fwd[l] for l in range(1, L + 1)]
            assert [c.bwd_D[l - 1] for l in range(1, L + 1)] == [bwd[l] for l in range(1, L + 1)]
    assert rdm.config_name(rdm.config_from_id(2, 10)) == "FDS/BDS"


def test_cost_model_matches_oracle_simulator():
    rnd = random.Random(3)
    for L in (1, 2, 3):
        for _ in range(60):
            f = [rnd.randint(1, 2000) for _ in range(L + 1)]
            for i in range(4 ** L):
                assert rdm.config_costs(f, i) == ocm.simulate(i, f)


@pytest.mark.parametrize("f", [(128, 128, 40), (128, 128, 349), (100, 128, 47), (602, 128, 41),
                               (256, 128, 100), (128, 128, 100), (256, 128, 25), (256, 128, 32),
                               (100, 256, 256, 47), (128, 128, 172), (1433, 128, 7)])
@pytest.mark.parametrize("P", [1, 2, 8])
def test_selector_front_and_pick(f, P):
    front, chosen, c, s = rdm.select_config(list(f), 232965, 114848857, P)
    assert front == ocm.pareto_front(f)
    assert chosen in front
    assert (c, s) == ocm.simulate(chosen, f)
    if P == 1:   # comm is free on one GPU → minimum sparse cost (reading R24)
        assert s == min(ocm.simulate(i, f)[1] for i in front)


@pytest.mark.parametrize("P", [1, 2, 4, 8])
@pytest.mark.parametrize("f", [(602, 128, 41), (1433, 128, 7), (100, 256, 256, 47)])
def test_executor_plan_charges_the_model(P, f):
    """The executor's redistribution widths equal the paper's comm units except
    the transfers the model ignores (reading R15/R14); SpMM widths equal the
    sparse units; exchanged elements follow the exact partition."""
    L = len(f) - 1
    n = 2708
    for i in range(4 ** L):
        info, desc = rdm.plan_info(list(f), i, P, n)
        mc, ms = ocm.simulate(i, f)
        assert (info["model_comm_units"], info["model_sparse_units"]) == (mc, ms)
        assert info["plan_sparse_units"] == ms
        if P == 1:
            assert info["plan_comm_units"] == 0 and "A2A" not in desc
            continue
        hidden = info["plan_hidden_comm_units"]
        fwd, bwd = ocm.decode(i, L)
        memo_all = all(not (bwd[l] and fwd[l]) for l in range(1, L + 1))
        if memo_all:
            assert info["plan_comm_units"] - hidden == mc, (i, info)
        if L == 2 and i not in (6, 9):
            assert hidden == 0
        widths = [int(w) for w in re.findall(r"A2A .* f=(\d+)", desc)]
        assert sum(widths) == info["plan_comm_units"]
        assert info["a2a_elems"] == sum(ordist.total_elements(n, w, P) for w in widths)


def test_hidden_mask_cost_only_ids_6_9():
    """Reading R15: only IDs 6 and 9 (L=2) need H^1 moved for the Hadamard."""
    for i in range(16):
        info, desc = rdm.plan_info([602, 128, 41], i, 4, 1000)
        assert ("hidden" in desc) == (i in (6, 9)), (i, desc)


def test_fig4_id10_plan_text():
    """Fig. 4's red path (L132-134): D,S forward with T_d saved, D,S backward."""
    _, desc = rdm.plan_info([602, 128, 41], 10, 8, 1000)
    fwd, bwd = desc.split("backward:")
    assert fwd.index("GEMM  NN H0.row") < fwd.index("SPMM  A^T T1.col")
    assert "A2A   T2.col -> T2.row" in fwd            # memo kept row-sliced
    assert "GEMM  TN T2.row^T G2.row -> Y2" in bwd      # reused for Y^2
    assert bwd.count("SPMM") == 2


@pytest.mark.parametrize("P", [2, 3, 8])
@pytest.mark.parametrize("n,f", [(1001, 41), (10, 7), (5, 130)])
def test_exchange_plan_is_consistent(P, n, f):
    """What p sends to q is exactly what q expects from p, in both directions."""
    for frm in (rdm.ROW, rdm.COL):
        plans = [rdm.redist_plan(P, p, frm, n, f) for p in range(P)]
        for p in range(P):
            for q in range(P):
                assert plans[p]["send_elems"][q] == plans[q]["recv_elems"][p]
                if p == q:
                    assert plans[p]["send_elems"][q] == 0
        payload = 0
        for p in range(P):
            for q in range(P):
                if p != q:
                    payload += ordist.send_elements(n, f, P, p, q,
                                                    "row2col" if frm == rdm.ROW else "col2row")
        wire = sum(sum(pl["send_elems"]) for pl in plans)
        assert wire >= payload
        assert payload == ordist.total_elements(n, f, P)


def test_error_codes_without_gpu():
    with pytest.raises(rdm.RdmError) as e:
        rdm.partition(0, rdm.ROW, 10, 10, 0)
    assert e.value.status == rdm.ERR_ARG
    with pytest.raises(rdm.RdmError):
        rdm.config_from_id(2, 16)


# ------------------------------------------------- R_A < P host functions (NEXT-4)
@pytest.mark.parametrize("seed", range(6))
def test_partition_tile_covers_matrix_once(seed):
    """Tiles of the P/R_A x R_A grid cover the N x f matrix exactly once, and
    every rank's row slice lies inside its row panel (so the row ↔ tile
    redistribution stays inside a panel group, L214)."""
    rng = random.Random(seed)
    P = rng.choice([1, 2, 4, 6, 8])
    RA = rng.choice([r for r in range(1, P + 1) if P % r == 0])
    n, f = rng.randint(0, 3000), rng.randint(1, 300)
    cover = np.zeros((n, f), np.int32)
    for p in range(P):
        r0, r1, c0, c1, ld = rdm.partition_tile(P, RA, n, f, p)
        cover[r0:r1, c0:c1] += 1
        assert ld % 4 == 0 and ld >= c1 - c0
        lo, hi, _ = rdm.partition(P, rdm.ROW, n, f, p)
        assert r0 <= lo and hi <= r1
        # R_A = P: a tile is the plain column slice
        if RA == P:
            assert (r0, r1) == (0, n)
            assert (c0, c1) == rdm.partition(P, rdm.COL, n, f, p)[:2]
    assert np.all(cover == 1)


def test_partition_tile_rejects_bad_grid():
    with pytest.raises(rdm.RdmError):
        rdm.partition_tile(8, 3, 100, 10, 0)


def test_max_replication_matches_oracle():
    rng = random.Random(3)
    for _ in range(500):
        P = rng.choice([1, 2, 3, 4, 6, 8, 16])
        M = rng.uniform(1, 200) * 1e9
        H = rng.uniform(0, 1.2) * M
        G = rng.uniform(0.1, 400) * 1e9
        assert rdm.max_replication(P, M, H, G) == ocm.max_replication(P, M, H, G)


@pytest.mark.parametrize("seed", range(4))
def test_select_config_ra_front_matches_oracle(seed):
    """The library's R_A < P front (elements moved, sparse units) equals the
    oracle's (reading R35), and R_A = P gives the full-replication front."""
    rng = random.Random(100 + seed)
    for _ in range(25):
        L = rng.choice([2, 3])
        f = [rng.randint(1, 700) for _ in range(L + 1)]
        n, nnz = rng.randint(100, 10 ** 7), rng.randint(100, 10 ** 9)
        P = rng.choice([2, 4, 6, 8])
        RA = rng.choice([r for r in range(1, P + 1) if P % r == 0])
        front, chosen, elems, sparse = rdm.select_config_ra(f, n, nnz, P, RA)
        assert front == ocm.pareto_ra(f, n, P, RA)
        assert chosen in front
        assert elems == pytest.approx(ocm.comm_elements_ra(chosen, f, n, P, RA))
        assert sparse == ocm.simulate(chosen, f)[1]
        if RA == P:
            assert front == rdm.select_config(f, n, nnz, P)[0]


def test_low_memory_workspace_papers_p8():
    """BASELINE configs[4] (papers100M-shaped 2L h128) at P = 8 fits one B200
    (~70 GB/GPU of live tensors with liveness-based reuse):
    rank 0's activation workspace under RDM_GCN_LOW_MEMORY, plus the
    replicated CSR and the redistribution staging, stays below 170 GB."""
    import synth
    wl = synth.WORKLOADS["papers"]
    P = 8
    pareto, chosen, _, _ = rdm.select_config(list(wl.f), wl.n, wl.nnz, P)
    assert chosen == 10 and pareto == [10]
    full, _ = rdm.plan_info(list(wl.f), chosen, P, wl.n)
    low, _ = rdm.plan_info(list(wl.f), chosen, P, wl.n, low_memory=True)
    rows0 = wl.n // P + 1
    staging = 2 * rows0 * max(wl.f) * 4            # pack send + unpack recv staging
    csr = 8 * wl.nnz + 8 * (wl.n + 1)
    assert low["workspace_bytes"] < 0.7 * full["workspace_bytes"]
    assert low["workspace_bytes"] + staging + csr < 170e9, low["workspace_bytes"] / 1e9
    # identical plan otherwise
    for k in ("model_comm_units", "model_sparse_units", "plan_comm_units", "a2a_elems"):
        assert low[k] == full[k]


@pytest.mark.parametrize("f,P", [([1433, 128, 7], 1), ([602, 128, 41], 4), ([100, 256, 256, 47], 8)])
def test_low_memory_never_larger(f, P):
    """Sharing only ever removes allocations, for every configuration."""
    L = len(f) - 1
    for cid in range(4 ** L):
        a, _ = rdm.plan_info(f, cid, P, 10007)
        b, _ = rdm.plan_info(f, cid, P, 10007, low_memory=True)
        assert 0 < b["workspace_bytes"] <= a["workspace_bytes"]


def test_feature_row_slices_match_whole_draw():
    """synth.features_rows / labels_rows (one rank's slice of a matrix too large
    to draw whole on the host) equal the corresponding rows of the whole draw."""
    import synth
    H = synth.features(3001, 17)
    assert np.array_equal(H[1234:2999], synth.features_rows(1234, 2999, 17))
    y = synth.labels(3001, 41)
    assert np.array_equal(y[7:3001], synth.labels_rows(7, 3001, 41))


@pytest.mark.parametrize("f,P", [([1433, 128, 7], 1), ([602, 128, 41], 4), ([100, 256, 256, 47], 8)])
def test_bias_plan(f, P):
    """RDM_GCN_BIAS (reading R8): in every configuration each layer's bias is
    fused into exactly one producer of Z^l — the last product of the layer
    (GEMM for order S, SpMM for order D) — and db^l is summed exactly once from
    G^l after its Hadamard mask; nothing else in the plan changes."""
    L = len(f) - 1
    for cid in range(4 ** L):
        a, da = rdm.plan_info(f, cid, P, 10007)
        b, db = rdm.plan_info(f, cid, P, 10007, bias=True)
        for k in ("plan_comm_units", "plan_sparse_units", "a2a_elems", "workspace_bytes"):
            assert a[k] == b[k], (cid, k)
        cfg = rdm.config_from_id(L, cid)
        fwd, bwd = db.split("backward:")
        for l in range(1, L + 1):
            adds = [s for s in fwd.splitlines() if s.endswith(f" +b{l}")]
            assert len(adds) == 1, (cid, l, fwd)
            kind = "SPMM" if cfg.fwd_D[l - 1] else "GEMM"
            assert adds[0].strip().startswith(kind), (cid, l, adds)
            assert f"-> {'Z0' if l == L else f'H{l}'}." in adds[0], adds   # Z^L is stored as Z0
            sums = [i for i, s in enumerate(bwd.splitlines()) if s.strip().endswith(f"-> db{l}")]
            assert len(sums) == 1, (cid, l, bwd)
        # with the bias lines removed the plan is the bias-free plan
        clean = "\n".join(s for s in db.splitlines() if "BSUM" not in s)
        for l in range(1, L + 1):
            clean = clean.replace(f" +b{l}", "")
        assert clean == da.rstrip("\n") or clean + "\n" == da, cid
