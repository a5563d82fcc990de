"""Generator determinism / CSR well-formedness, and the oracle's 2LB layout vs the hand-worked fixture."""
import numpy as np

import gen
import oracle
from golden import twolayer_example


def _check_csr(g):
    rp, ci = g.row_ptr, g.col_idx
    assert rp[0] == 0 and rp[-1] == len(ci) and (np.diff(rp) >= 0).all()
    rows = np.repeat(np.arange(g.n), np.diff(rp))
    assert (ci != rows).all()                                   # no self-loops
    assert ((ci >= 0) & (ci < g.n)).all()
    d = np.diff(ci.astype(np.int64))
    starts = np.zeros(len(ci) + 1, bool)
    starts[rp[1:-1]] = True
    assert ((d > 0) | starts[1:-1]).all()                        # rows strictly ascending => simple
    k1 = rows.astype(np.int64) * g.n + ci
    k2 = ci.astype(np.int64) * g.n + rows
    assert np.array_equal(np.sort(k1), np.sort(k2))             # symmetric


def test_generators_wellformed_and_deterministic():
    for mk in (lambda: gen.rmat(12, 16), lambda: gen.rmat(12, 32, permute=True),
               lambda: gen.gnm(50_000, 300_000), lambda: gen.lattice(90, 110, 0.6),
               lambda: gen.hypercube(8), lambda: gen.grid(5, 7)):
        a, b = mk(), mk()
        _check_csr(a)
        assert a.sha256() == b.sha256()


def test_rmat_shape_matches_survey_scratch():
    # scale 10 EF16 -> ~10.5K undirected edges, hub = vertex 0
    g = gen.rmat(10, 16)
    assert 10_000 < g.nnz // 2 < 11_000
    assert int(np.argmax(g.degrees())) == 0
    assert 400 < g.degrees().max() < 600


def test_lattice_degree_and_sources():
    g = gen.lattice(100, 100, 0.6)
    assert g.degrees().max() <= 4
    assert abs(g.nnz / 2 / (2 * 100 * 99) - 0.6) < 0.02
    s = gen.sources(g, 64, stream=6)
    assert len(set(s.tolist())) == 64 and (g.degrees()[s] > 0).all()


def test_c5_sources_in_largest_component():
    """Reading C15: config-5 sources come from the largest component (checked with the oracle's
    union-find labels, independent of the scipy routine that builds the mask)."""
    g = gen.lattice(120, 180, 0.6)
    lab = oracle.cc(g)
    big = np.bincount(lab).argmax()
    mask = gen.largest_component_mask(g)
    assert np.array_equal(mask.astype(bool), lab == big)
    s = gen.sources(g, 64, stream=6, eligible=mask)
    assert len(set(s.tolist())) == 64 and (lab[s] == big).all()
    # the unrestricted draw on the same stream hits small clusters (so the restriction matters)
    s_any = gen.sources(g, 64, stream=6)
    assert (lab[s_any] != big).any()


def test_weights_symmetric():
    g = gen.with_weights(gen.rmat(11, 16), seed=5)
    rows = np.repeat(np.arange(g.n), g.degrees())
    fwd = dict(zip(zip(rows.tolist(), g.col_idx.tolist()), g.weights.tolist()))
    assert all(fwd[(b, a)] == w for (a, b), w in fwd.items())


def test_two_layer_bitmap_fixture():
    n, active, words, summ = twolayer_example()
    mask = np.zeros(n, bool)
    mask[active] = True
    w = oracle.bitmap_words(mask)
    assert np.array_equal(w, words)
    assert np.array_equal(oracle.summary_words(w), summ)
    assert np.array_equal(oracle.words_to_mask(w, n), mask)


def test_orient_makes_a_directed_subgraph():
    """gen.orient keeps each arc of a symmetric graph by a hash bit: every kept arc is an arc of
    the input, rows stay sorted, and both / one / no direction survive about 1/4, 1/2, 1/4."""
    g = gen.with_weights(gen.rmat(12, 16, permute=True), seed=3)
    d = gen.orient(g, seed=5)
    rows = np.repeat(np.arange(g.n), g.degrees())
    full = set(zip(rows.tolist(), g.col_idx.tolist()))
    drows = np.repeat(np.arange(d.n), d.degrees())
    arcs = set(zip(drows.tolist(), d.col_idx.tolist()))
    assert arcs <= full
    both = sum(1 for (u, v) in arcs if u < v and (v, u) in arcs)
    edges = len(full) // 2
    assert abs(both / edges - 0.25) < 0.03 and abs(len(arcs) / len(full) - 0.5) < 0.03
    starts = np.zeros(d.nnz + 1, bool)
    starts[d.row_ptr[:-1]] = True
    assert ((np.diff(d.col_idx.astype(np.int64)) > 0) | starts[1:-1]).all()
    w = dict(zip(zip(rows.tolist(), g.col_idx.tolist()), g.weights.tolist()))
    assert all(w[(u, v)] == x for (u, v), x in zip(zip(drows.tolist(), d.col_idx.tolist()), d.weights.tolist()))
