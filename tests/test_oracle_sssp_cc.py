"""Pins for oracle.sssp (Dijkstra) and oracle.cc (union-find)."""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import connected_components, dijkstra

import gen
import oracle
from brute import closure_min_labels, floyd_warshall

INF = 0xFFFFFFFF


def _fw_u32(g):
    D = floyd_warshall(g)
    return D


@pytest.mark.parametrize("n,p,seed,wmax", [(20, 0.2, 1, 64), (48, 0.08, 2, 64), (64, 0.05, 3, 5), (64, 0.3, 4, 64),
                                           (30, 0.04, 5, 64)])
def test_sssp_vs_floyd_warshall(n, p, seed, wmax):
    g = gen.with_weights(gen.random_simple(n, p, seed), seed=seed, wmax=wmax)
    D = floyd_warshall(g)
    for s in range(0, n, 5):
        d = oracle.sssp(g, s)
        exp = np.where(np.isfinite(D[s]), D[s], INF).astype(np.uint64)
        assert np.array_equal(d.astype(np.uint64), exp)


def test_sssp_weights_symmetric_in_range():
    g = gen.with_weights(gen.rmat(12, 16), seed=1)
    w = g.weights
    assert w.min() >= 1 and w.max() <= 64
    deg = g.degrees()
    src = np.repeat(np.arange(g.n), deg)
    key = dict(zip(zip(src.tolist(), g.col_idx.tolist()), w.tolist()))
    for (a, b), x in list(key.items())[:5000]:
        assert key[(b, a)] == x


def test_sssp_unit_weights_is_bfs():
    g = gen.rmat(13, 16, permute=True)
    g.weights = np.ones(g.nnz, np.uint8)
    for s in gen.sources(g, 3):
        assert np.array_equal(oracle.sssp(g, int(s)), oracle.bfs(g, int(s)))


def test_sssp_path_prefix_sums():
    g = gen.with_weights(gen.path(200), seed=7)
    deg = g.degrees()
    src = np.repeat(np.arange(g.n), deg)
    fwd = g.weights[g.col_idx == src + 1]          # w(i, i+1) in order of i
    exp = np.concatenate([[0], np.cumsum(fwd.astype(np.uint64))]).astype(np.uint32)
    assert np.array_equal(oracle.sssp(g, 0), exp)


def test_sssp_vs_library_dijkstra_rmat():
    """Special case reducing to a library routine: scipy's Dijkstra on the same weights."""
    g = gen.with_weights(gen.rmat(14, 16, permute=True), seed=3)
    A = sp.csr_matrix((g.weights.astype(np.float64), g.col_idx, g.row_ptr), shape=(g.n, g.n))
    for s in gen.sources(g, 2):
        ref = dijkstra(A, directed=True, indices=int(s))
        exp = np.where(np.isfinite(ref), ref, INF).astype(np.uint64)
        assert np.array_equal(oracle.sssp(g, int(s)).astype(np.uint64), exp)


def check_sssp_invariants(g, s, d):
    deg = g.degrees()
    src = np.repeat(np.arange(g.n), deg)
    du, dv = d[src].astype(np.int64), d[g.col_idx].astype(np.int64)
    w = g.weights.astype(np.int64)
    assert d[s] == 0
    ok = du != INF
    assert (dv[ok] <= du[ok] + w[ok]).all()                       # nothing relaxable
    tight = np.zeros(g.n, bool)
    m = ok & (dv == du + w)
    tight[g.col_idx[m]] = True
    reached = d != INF
    assert tight[reached & (np.arange(g.n) != s)].all()          # every reached v has a tight arc


def test_sssp_invariants():
    g = gen.with_weights(gen.rmat(15, 16), seed=1)
    for s in [0] + list(gen.sources(g, 2)):
        check_sssp_invariants(g, int(s), oracle.sssp(g, int(s)))


# ----------------------------------------------------------------------------- CC
@pytest.mark.parametrize("n,p,seed", [(10, 0.1, 1), (40, 0.03, 2), (40, 0.06, 3), (64, 0.02, 4), (25, 0.5, 5)])
def test_cc_vs_transitive_closure(n, p, seed):
    g = gen.random_simple(n, p, seed)
    assert np.array_equal(oracle.cc(g), closure_min_labels(g))


def check_cc_invariants(g, lab):
    deg = g.degrees()
    src = np.repeat(np.arange(g.n), deg)
    assert (lab[src] == lab[g.col_idx]).all()
    v = np.arange(g.n)
    assert (lab <= v).all()
    assert (lab[lab] == lab).all()
    A = sp.csr_matrix((np.ones(g.nnz, np.int8), g.col_idx, g.row_ptr), shape=(g.n, g.n))
    ncomp, comp = connected_components(A, directed=False)
    assert len(np.unique(lab)) == ncomp
    # min id per library component
    mins = np.full(ncomp, g.n)
    np.minimum.at(mins, comp, v)
    assert np.array_equal(lab, mins[comp])


def test_cc_invariants_and_library():
    for g in (gen.gnm(200_000, 100_000, seed=2), gen.rmat(14, 4, permute=True), gen.lattice(200, 300, 0.5)):
        check_cc_invariants(g, oracle.cc(g))


def test_cc_closed_forms():
    assert (oracle.cc(gen.path(50)) == 0).all()
    assert np.array_equal(oracle.cc(gen.empty_graph(7)), np.arange(7, dtype=np.int32))
    # two disjoint cycles 0..9 and 10..19 plus isolated 20
    u = list(range(10)) + list(range(10, 20))
    v = [(i + 1) % 10 for i in range(10)] + [10 + (i + 1) % 10 for i in range(10)]
    lab = oracle.cc(gen.from_edges(21, u, v))
    assert np.array_equal(lab, np.array([0] * 10 + [10] * 10 + [20], np.int32))
