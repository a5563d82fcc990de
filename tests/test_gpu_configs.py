"""GPU parity at the full BASELINE.json sizes (configs 2-5), in the launch configuration bench.py
uses (default options, graph-driven BFS).  Every output element is compared with the oracle
(BFS / SSSP / CC bit-exact, BC within 1e-9 relative); where the oracle would take minutes, a
sample of the workload's sources is used (stated per test)."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
INF = 0xFFFFFFFF


@pytest.fixture(scope="module")
def sg():
    import torch
    import paper_conf_icpp_carocc25_b200 as m
    torch.cuda.set_device(0)
    return m


def test_config2_sssp_rmat20(sg):
    g = gen.make_config_graph(2)
    assert g.n == 1 << 20 and g.nnz > 30_000_000
    G = sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights)
    for s in list(gen.config_sources(2, g)) + list(gen.sources(g, 2)):
        d, st = sg.run_sssp(G, int(s))
        assert np.array_equal(sg.as_u32(d), oracle.sssp(g, int(s)))


def test_config3_cc_gnm_21M(sg):
    g = gen.make_config_graph(3)
    assert g.n == 21_000_000 and g.nnz > 529_000_000
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    lab, st = sg.run_cc(G)
    ref = oracle.cc(g)
    assert np.array_equal(lab.cpu().numpy(), ref)
    del G


def test_config3b_cc_many_components(sg):
    g = gen.gnm(21_000_000, 10_500_000, seed=1)
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    lab, _ = sg.run_cc(G)
    ref = oracle.cc(g)
    assert len(np.unique(ref)) > 1_000_000
    assert np.array_equal(lab.cpu().numpy(), ref)


@pytest.fixture(scope="module")
def c4(sg):
    g = gen.make_config_graph(4)
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    return g, G


def test_config4_bfs_kron24_two_roots(sg, c4):
    """Sample: 2 of the 64 roots (the oracle needs ~5 s per root); all 2^24 levels compared."""
    g, G = c4
    roots = gen.config_sources(4, g)
    assert len(roots) == 64
    for s in roots[:2]:
        lv, st = sg.run_bfs(G, int(s))
        ref = oracle.bfs(g, int(s))
        assert np.array_equal(sg.as_u32(lv), ref)
        assert st.pull_steps > 0 and st.push_steps > 0        # direction optimisation engaged
        assert st.reached == int((ref != INF).sum())


def test_config4_push_only_matches(sg, c4):
    g, G = c4
    s = int(gen.config_sources(4, g)[5])
    a, sa = sg.run_bfs(G, s, direction=sg.SG_DIR_PUSH)             # heavy levels: segmented advance
    c, sc = sg.run_bfs(G, s, direction=sg.SG_DIR_PUSH, scsr=1)     # word path only
    b, _ = sg.run_bfs(G, s)
    ref = oracle.bfs(g, s)
    assert np.array_equal(sg.as_u32(a), ref) and np.array_equal(sg.as_u32(b), ref)
    assert np.array_equal(sg.as_u32(c), ref)
    assert sa.arcs_pushed == sc.arcs_pushed                       # both inspect every reached vertex's arcs


def test_config4_all_roots_bfs_invariants(sg, c4):
    """All 64 roots at full size through invariants that hold at any size: level[s] = 0,
    |level[u] - level[v]| <= 1 on every arc, every reached v != s has a parent one level up,
    reached set identical for all roots in the giant component."""
    import torch
    g, G = c4
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    src = torch.repeat_interleave(torch.arange(g.n, device="cuda"), torch.diff(rp))
    for s in gen.config_sources(4, g):
        lv, _ = sg.run_bfs(G, int(s))
        l64 = lv.to(torch.int64) & 0xFFFFFFFF
        assert int(l64[int(s)]) == 0
        a, b = l64[src], l64[ci.to(torch.int64)]
        fin = (a != INF) & (b != INF)
        assert bool(((a == INF) == (b == INF)).all())
        assert int((a[fin] - b[fin]).abs().max()) <= 1
        has_parent = torch.zeros(g.n, dtype=torch.bool, device="cuda")
        has_parent[ci.to(torch.int64)[fin & (a + 1 == b)]] = True
        reached = l64 != INF
        reached[int(s)] = False
        assert bool(has_parent[reached].all())


def test_config5_bc_lattice_two_sources(sg):
    """Sample: 2 of the 64 sources on the full 4000x6000 p=0.6 lattice (sigma far beyond
    DBL_MAX along ~10^4 levels); every vertex's score compared with the long-double oracle."""
    g = gen.make_config_graph(5)
    assert g.n == 24_000_000
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    srcs = gen.config_sources(5, g)[:2]
    bc, st = sg.run_bc(G, srcs)
    ref = oracle.bc(g, srcs)
    got = bc.cpu().numpy()
    assert np.all(np.abs(got - ref) <= 1e-9 * np.maximum(np.abs(ref), 1.0))
