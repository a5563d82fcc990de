"""Pins for oracle.bfs (queue BFS) — independent brute force, closed forms, invariants."""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import connected_components

import gen
import oracle
from brute import all_graphs, bfs_levels_matpow

INF = 0xFFFFFFFF


def test_exhaustive_5_vertices():
    """All 1,024 labelled graphs on 5 vertices x all 5 sources vs boolean matrix powers."""
    for edges in all_graphs(5):
        u = [e[0] for e in edges]
        v = [e[1] for e in edges]
        g = gen.from_edges(5, u, v)
        for s in range(5):
            assert np.array_equal(oracle.bfs(g, s), bfs_levels_matpow(g, s)), (edges, s)


@pytest.mark.parametrize("n,p,seed", [(16, 0.1, 1), (33, 0.08, 2), (64, 0.05, 3), (64, 0.2, 4), (40, 0.03, 5)])
def test_random_small_vs_matpow(n, p, seed):
    g = gen.random_simple(n, p, seed)
    for s in range(0, n, 7):
        assert np.array_equal(oracle.bfs(g, s), bfs_levels_matpow(g, s))


def test_closed_forms():
    n = 100
    assert np.array_equal(oracle.bfs(gen.path(n), 0), np.arange(n, dtype=np.uint32))
    i = np.arange(n)
    assert np.array_equal(oracle.bfs(gen.cycle(n), 0), np.minimum(i, n - i).astype(np.uint32))
    lv = oracle.bfs(gen.star(n), 5)
    exp = np.full(n, 2, np.uint32); exp[0] = 1; exp[5] = 0
    assert np.array_equal(lv, exp)
    lv = oracle.bfs(gen.complete(30), 7)
    exp = np.ones(30, np.uint32); exp[7] = 0
    assert np.array_equal(lv, exp)
    R, C = 37, 53
    lv = oracle.bfs(gen.grid(R, C), 0)
    r, c = np.divmod(np.arange(R * C), C)
    assert np.array_equal(lv, (r + c).astype(np.uint32))
    s = 11 * C + 20
    lv = oracle.bfs(gen.grid(R, C), s)
    assert np.array_equal(lv, (np.abs(r - 11) + np.abs(c - 20)).astype(np.uint32))
    d = 12
    v = np.arange(1 << d)
    for s in (0, 1234):
        pc = np.array([bin(x ^ s).count("1") for x in v], dtype=np.uint32)
        assert np.array_equal(oracle.bfs(gen.hypercube(d), s), pc)


def test_isolated_and_empty():
    g = gen.empty_graph(10)
    lv = oracle.bfs(g, 3)
    assert lv[3] == 0 and (np.delete(lv, 3) == INF).all()
    g = gen.rmat(10, 16)
    iso = np.nonzero(g.degrees() == 0)[0][0]
    lv = oracle.bfs(g, int(iso))
    assert lv[iso] == 0 and (lv == INF).sum() == g.n - 1


def check_bfs_invariants(g, s, lv):
    deg = g.degrees()
    src = np.repeat(np.arange(g.n), deg)
    dst = g.col_idx
    assert lv[s] == 0
    a, b = lv[src].astype(np.int64), lv[dst].astype(np.int64)
    both = (a != INF) & (b != INF)
    assert (np.abs(a[both] - b[both]) <= 1).all()
    # an arc never joins reached and unreached
    assert ((a == INF) == (b == INF)).all()
    # every reached v != s has a neighbour at level[v]-1
    has_parent = np.zeros(g.n, bool)
    m = both & (a + 1 == b)
    has_parent[dst[m]] = True
    reached = lv != INF
    assert has_parent[reached & (np.arange(g.n) != s)].all()
    # reached set = connected component of s (library routine)
    A = sp.csr_matrix((np.ones(g.nnz, np.int8), g.col_idx, g.row_ptr), shape=(g.n, g.n))
    _, lab = connected_components(A, directed=False)
    assert np.array_equal(reached, lab == lab[s])


def test_invariants_rmat():
    g = gen.rmat(15, 16, permute=True)
    for s in gen.sources(g, 4):
        check_bfs_invariants(g, int(s), oracle.bfs(g, int(s)))


def test_invariants_lattice():
    g = gen.lattice(120, 150, 0.6)
    for s in gen.sources(g, 3, stream=6):
        check_bfs_invariants(g, int(s), oracle.bfs(g, int(s)))


def test_advance_step_set_semantics_reproduce_levels():
    """Iterating the one-step set definition (Table 2 advance + Listing 1 compute) from {s}
    yields exactly the level sets of the pinned queue BFS."""
    g = gen.rmat(12, 16, permute=True)
    s = int(gen.sources(g, 1)[0])
    lv = oracle.bfs(g, s)
    frontier = np.zeros(g.n, bool)
    frontier[s] = True
    visited = frontier.copy()
    d = 0
    while frontier.any():
        assert np.array_equal(frontier, lv == d)
        out = oracle.bfs_advance_step(g, frontier, visited)
        visited |= out
        frontier = out
        d += 1
    assert d == int(lv[lv != INF].max()) + 1


def test_jacobi_step_bounds_final_values():
    """Iterating the Jacobi relax step to a fixed point reaches Dijkstra's distances and CC labels."""
    g = gen.with_weights(gen.rmat(11, 8, permute=True), seed=2)
    s = int(gen.sources(g, 1)[0])
    val = np.full(g.n, INF, np.int64)
    val[s] = 0
    front = np.zeros(g.n, bool)
    front[s] = True
    while front.any():
        new = oracle.jacobi_relax_step(g, front, val, g.weights)
        front = new < val
        val = new
    assert np.array_equal(val.astype(np.uint32), oracle.sssp(g, s))
    lab = np.arange(g.n, dtype=np.int64)
    front = np.ones(g.n, bool)
    while front.any():
        new = oracle.jacobi_relax_step(g, front, lab)
        front = new < lab
        lab = new
    assert np.array_equal(lab.astype(np.int32), oracle.cc(g))


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_jacobi_single_step_vs_brute_force(seed):
    """One Jacobi step, pinned on its own (not through the fixed point): for every v,
    new[v] = min(value[v], min over frontier neighbours u of value[u] + w(u,v)), computed here by a
    pure-Python pull over v's row (the oracle pushes over source rows).  A step that ignored the
    frontier restriction, dropped the weight, or took max instead of min fails."""
    g = gen.with_weights(gen.rmat(7, 6, seed=seed, permute=True), seed=seed)
    rng = np.random.default_rng(seed)
    value = rng.integers(0, 500, g.n).astype(np.int64)
    value[rng.random(g.n) < 0.2] = INF
    front = rng.random(g.n) < 0.3
    for weights in (g.weights, None):
        got = oracle.jacobi_relax_step(g, front, value, weights)
        for v in range(g.n):
            best = int(value[v])
            for e in range(int(g.row_ptr[v]), int(g.row_ptr[v + 1])):
                u = int(g.col_idx[e])
                if front[u]:
                    c = int(value[u]) + (int(weights[e]) if weights is not None else 0)
                    best = min(best, c)
            assert got[v] == best, (v, got[v], best)
        # the frontier restriction matters on this input
        assert not np.array_equal(got, oracle.jacobi_relax_step(g, np.ones(g.n, bool), value, weights))
