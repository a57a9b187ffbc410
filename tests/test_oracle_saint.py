"""Pins of the GraphSAINT sampler oracle (oracle/saint.py) against things other
than itself (CPU only): the published SplitMix64 sequence, walk validity
against the dense adjacency, uniformity of the step draw (chi-square), the
induced subgraph against scipy slicing + dense normalisation, and closed
forms on the complete and star graphs."""
import numpy as np
import pytest
import scipy.sparse as sp

import synth
from oracle import saint


def test_splitmix64_published_sequence():
    """SplitMix64 seeded with 0 (Vigna, splitmix64.c): next() #k returns
    mix((k+1)·φ) = splitmix64(k·φ) in the oracle's convention."""
    want = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F, 0xF88BB8A8724C81EC]
    got = [saint.splitmix64((k * saint.PHI) & saint.M64) for k in range(4)]
    assert got == want


@pytest.fixture(scope="module")
def small():
    return synth.rmat(300, 1500, seed=9)


def test_walks_follow_edges(small):
    g = small
    dense = sp.csr_matrix((np.ones(g.nnz), g.col, g.rowptr), shape=(g.n, g.n)).toarray()
    V = saint.walks(g.rowptr, g.col, g.n, 200, 6, seed=3, it=2)
    assert V.shape == (200, 7)
    for row in V:
        for a, b in zip(row[:-1], row[1:]):
            assert dense[a, b] != 0


def test_roots_and_node_set(small):
    g = small
    V = saint.walks(g.rowptr, g.col, g.n, 50, 3, seed=1, it=0)
    key = saint.splitmix64(1)
    roots = [saint.splitmix64(key ^ (i << 8)) % g.n for i in range(50)]
    assert list(V[:, 0]) == roots
    nodes = saint.node_set(V)
    assert np.all(np.diff(nodes) > 0)
    assert set(nodes.tolist()) == set(V.ravel().tolist())


def test_step_draw_is_uniform():
    """Complete graph K_7 (self loops included): one step from any vertex is
    uniform over the 7 vertices (chi-square, 6 dof, 21,000 draws)."""
    g = synth.complete_graph(7)
    V = saint.walks(g.rowptr, g.col, g.n, 21000, 1, seed=5, it=0)
    cnt = np.bincount(V[:, 1], minlength=7)
    exp = len(V) / 7
    chi2 = float(((cnt - exp) ** 2 / exp).sum())
    assert chi2 < 30.0, (cnt, chi2)   # p ≈ 4e-5 at the bound
    rc = np.bincount(V[:, 0], minlength=7)
    assert float(((rc - exp) ** 2 / exp).sum()) < 30.0


def test_induced_matches_scipy(small):
    g = small
    rng = np.random.default_rng(4)
    nodes = np.sort(rng.choice(g.n, 120, replace=False))
    rp, cs, vs = saint.induced(g.rowptr, g.col, nodes)
    A = sp.csr_matrix((np.ones(g.nnz), g.col, g.rowptr), shape=(g.n, g.n))
    As = A[nodes][:, nodes].toarray()
    deg = As.sum(axis=1)
    with np.errstate(divide="ignore"):
        dinv = np.where(deg > 0, 1.0 / np.sqrt(deg), 0.0)
    ref = dinv[:, None] * As * dinv[None, :]
    got = sp.csr_matrix((vs.astype(np.float64), cs, rp), shape=(len(nodes), len(nodes))).toarray()
    assert np.array_equal(got != 0, As != 0)
    np.testing.assert_allclose(got, ref, rtol=1e-6, atol=0)
    # entries keep the original row order
    for i, v in enumerate(nodes):
        orig = [u for u in g.col[g.rowptr[v]:g.rowptr[v + 1]] if u in set(nodes.tolist())]
        assert list(nodes[cs[rp[i]:rp[i + 1]]]) == orig


def test_induced_complete_graph_closed_form():
    g = synth.complete_graph(9)
    nodes = np.array([1, 4, 5, 8])
    rp, cs, vs = saint.induced(g.rowptr, g.col, nodes)
    assert list(rp) == [0, 4, 8, 12, 16]
    np.testing.assert_allclose(vs, 0.25, rtol=0, atol=0)


def test_induced_star_leaves_only():
    """Leaves of a star without the hub keep only their self loops: Â_s = I."""
    g = synth.star_graph(6)
    rp, cs, vs = saint.induced(g.rowptr, g.col, np.array([1, 2, 5]))
    assert list(rp) == [0, 1, 2, 3] and list(cs) == [0, 1, 2]
    assert np.all(vs == 1.0)
