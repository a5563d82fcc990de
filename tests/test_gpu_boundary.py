"""C-ABI boundary cases (include/sygraph.h): the functor-level advance entry
points a user drives directly (Table 2), graph_load_csr's validation and borrow
modes (§3.1; readings C8, C9), and their error paths."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

INF = 0xFFFFFFFF


@pytest.fixture(scope="module")
def sg():
    import torch
    import paper_conf_icpp_carocc25_b200 as m
    torch.cuda.set_device(0)
    return m


def test_advance_without_output_frontier(sg):
    """advance::frontier(G, In, F): no output frontier; the BFS functor still writes
    level[] and visited for exactly the set {v : exists u in In, (u,v) in E, v not visited}."""
    import torch
    g = gen.rmat(12, 16, permute=True)
    G = sg.graph_load_csr(g.row_ptr, g.col_idx, validate=True)
    s = int(gen.sources(g, 1)[0])
    lvl = oracle.bfs(g, s)
    fin = sg.frontier_init(G)
    level = torch.full((g.n,), -1, dtype=torch.int32, device="cuda")
    visited = torch.zeros((g.n + 63) // 64, dtype=torch.int64, device="cuda")
    for d in range(int(lvl[lvl != INF].max()) + 1):
        vis = lvl <= d
        visited.copy_(torch.from_numpy(oracle.bitmap_words(vis).view(np.int64)))
        level.copy_(torch.from_numpy(np.where(vis, lvl, INF).astype(np.uint32).view(np.int32)))
        sg.frontier_clear(fin)
        sg.frontier_insert(fin, np.nonzero(lvl == d)[0].astype(np.int32))
        sg.advance(G, fin, None, sg.SG_FN_BFS, dict(level=level, visited=visited, depth=d))
        exp = oracle.bfs_advance_step(g, lvl == d, vis)
        got_vis = oracle.words_to_mask(visited.cpu().numpy().view(np.uint64), g.n)
        assert np.array_equal(got_vis, vis | exp)
        got_lv = sg.as_u32(level)
        assert np.array_equal(got_lv, np.where(vis | exp, np.where(vis, lvl, d + 1), INF).astype(np.uint32))


def _sigma_forward(sg, g, s, with_exp=True):
    """User-driven Brandes forward pass through advance(SG_FN_BC_SIGMA)."""
    import torch
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    level = torch.full((g.n,), -1, dtype=torch.int32, device="cuda")
    level[s] = 0
    sigma = torch.zeros(g.n, dtype=torch.float64, device="cuda")
    sigma[s] = 1.0
    expo = torch.zeros(g.n + 2, dtype=torch.int32, device="cuda") if with_exp else None
    visited = torch.zeros((g.n + 63) // 64, dtype=torch.int64, device="cuda")
    fin = sg.frontier_init(G)
    sg.frontier_insert(fin, np.array([s], np.int32))
    sg.frontier_or_into(fin, visited)
    d = 0
    while True:
        fout = sg.frontier_init(G)
        st = dict(level=level, visited=visited, sigma=sigma, depth=d)
        if with_exp:
            st["exp2_per_level"] = expo
        sg.advance(G, fin, fout, sg.SG_FN_BC_SIGMA, st)
        sg.frontier_or_into(fout, visited)
        if sg.frontier_count(fout) == 0:
            break
        fin = fout
        d += 1
    return sg.as_u32(level), sigma.cpu().numpy(), expo.cpu().numpy() if with_exp else None, d


@pytest.mark.parametrize("make,s", [(lambda: gen.grid(600, 600), 0), (lambda: gen.rmat(12, 16, permute=True), None),
                                    (lambda: gen.lattice(150, 200, 0.6, seed=3), None)])
def test_advance_bc_sigma_with_level_exponents(sg, make, s):
    """sigma through the ABI entry itself, on a 600x600 grid where sigma reaches ~2^1193 > DBL_MAX:
    stored sigma * 2^E[level] must equal the oracle's path counts (compared in log2, rel 1e-9), and
    each level's maximum is scaled into [1, 2) (reading C20)."""
    g = make()
    if s is None:
        s = int(gen.sources(g, 1)[0])
    lv, sig, expo, depth = _sigma_forward(sg, g, s)
    ref_lv, _, ref_lsig, _ = oracle.bc_single(g, s)
    assert np.array_equal(lv, ref_lv)
    r = ref_lv != INF
    got_l2 = np.log2(sig[r]) + expo[lv[r]]
    assert np.all(np.abs(got_l2 - ref_lsig[r]) <= 1.5e-9 * np.maximum(1.0, np.abs(ref_lsig[r])))
    for L in range(1, depth + 1):
        m = sig[lv == L].max()
        assert 1.0 <= m < 2.0, (L, m)


def test_advance_bc_sigma_needs_exponents_and_output(sg):
    import torch
    g = gen.path(10)
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    fin, fout = sg.frontier_init(G), sg.frontier_init(G)
    sg.frontier_insert(fin, np.array([0], np.int32))
    st = dict(level=torch.zeros(10, dtype=torch.int32, device="cuda"),
              visited=torch.zeros(1, dtype=torch.int64, device="cuda"),
              sigma=torch.zeros(10, dtype=torch.float64, device="cuda"), depth=0)
    with pytest.raises(sg.SgError) as e:
        sg.advance(G, fin, fout, sg.SG_FN_BC_SIGMA, st)
    assert e.value.code == sg.SG_ERR_STATE
    st["exp2_per_level"] = torch.zeros(12, dtype=torch.int32, device="cuda")
    with pytest.raises(sg.SgError) as e:
        sg.advance(G, fin, None, sg.SG_FN_BC_SIGMA, st)
    assert e.value.code == sg.SG_ERR_STATE


# ------------------------------------------------------------------ graph_load_csr contract
def _csr_from_rows(rows):
    rp = np.zeros(len(rows) + 1, np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    ci = np.array([c for r in rows for c in r], np.int32)
    return rp, ci


@pytest.mark.parametrize("rows,what", [
    ([[1, 2], [0], [0]], None),                      # valid star
    ([[2, 1], [0], [0]], "unsorted"),
    ([[1, 1], [0, 0], []], "duplicate"),
    ([[0, 1], [0], []], "self-loop"),
    ([[1, 2], [0], []], "asymmetric"),
    ([[1], [0, 3], [], [1]], None),
])
def test_validate_rejects_each_violation(sg, rows, what):
    rp, ci = _csr_from_rows(rows)
    if what is None:
        sg.graph_load_csr(rp, ci, validate=True).free()
        return
    with pytest.raises(sg.SgError) as e:
        sg.graph_load_csr(rp, ci, validate=True)
    assert e.value.code == sg.SG_ERR_INVALID
    G = sg.graph_load_csr(rp, ci)   # without SG_F_VALIDATE only malformed row_ptr / ids are refused
    G.free()


def test_validate_rejects_malformed_row_ptr_and_ids(sg):
    rp, ci = _csr_from_rows([[1], [0]])
    for bad_rp, bad_ci in ((np.array([0, 2, 1], np.int64), ci), (rp, np.array([1, 5], np.int32)),
                           (rp, np.array([1, -1], np.int32))):
        with pytest.raises(sg.SgError) as e:
            sg.graph_load_csr(bad_rp, bad_ci)
        assert e.value.code == sg.SG_ERR_INVALID


def _shuffle_rows(g, seed):
    rng = np.random.default_rng(seed)
    ci = g.col_idx.copy()
    for v in range(g.n):
        a, b = int(g.row_ptr[v]), int(g.row_ptr[v + 1])
        if b - a > 1:
            ci[a:b] = rng.permutation(ci[a:b])
    return ci


@pytest.mark.parametrize("host_loop", [False, True])
def test_unsorted_rows_disable_sorted_only_tiers(sg, monkeypatch, host_loop):
    """Rows out of order (allowed without SG_F_VALIDATE): the hub-segmented tier, the segment-major
    sweep and the label-blocked CC pull binary-search sorted rows, so they are switched off for the
    graph instead of indexing shared memory out of range; every forced-on mode still gives the
    oracle's results."""
    monkeypatch.setenv("SG_CC_LBLOCK_KB", "4")
    g = gen.rmat(13, 16, permute=True)
    ci = _shuffle_rows(g, 1)
    G = sg.graph_load_csr(g.row_ptr, ci)
    with pytest.raises(sg.SgError):
        sg.graph_load_csr(g.row_ptr, ci, validate=True)
    for s in list(gen.sources(g, 2)) + [int(np.argmax(g.degrees()))]:
        ref = oracle.bfs(g, s)
        for kw in (dict(segmented=2, direction=sg.SG_DIR_PUSH), dict(scsr=2, direction=sg.SG_DIR_PUSH),
                   dict(segmented=2), dict(direction=sg.SG_DIR_PULL)):
            lv, _ = sg.run_bfs(G, int(s), host_loop=host_loop, **kw)
            assert np.array_equal(sg.as_u32(lv), ref), kw
    ref = oracle.cc(g)
    for d in (sg.SG_DIR_PULL, sg.SG_DIR_AUTO):
        lab, _ = sg.run_cc(G, direction=d)
        assert np.array_equal(lab.cpu().numpy(), ref)


def test_borrowed_device_csr(sg):
    """SG_F_BORROW: the graph keeps the caller's device tensors (no copy) and gives the same results;
    misaligned col_idx is refused."""
    import torch
    g = gen.with_weights(gen.rmat(12, 16, permute=True), seed=4)
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    w = torch.from_numpy(g.weights).cuda()
    G = sg.graph_load_csr(rp, ci, w, borrow=True, validate=True)
    _, _, rp_dev, ci_dev, _ = sg.graph_info(G)
    assert rp_dev == rp.data_ptr() and ci_dev == ci.data_ptr()
    s = int(gen.sources(g, 1)[0])
    lv, _ = sg.run_bfs(G, s)
    assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, s))
    d, _ = sg.run_sssp(G, s)
    assert np.array_equal(sg.as_u32(d), oracle.sssp(g, s))
    big = torch.zeros(g.nnz + 64, dtype=torch.int32, device="cuda")
    big[1:g.nnz + 1] = ci
    with pytest.raises(sg.SgError) as e:
        sg.graph_load_csr(rp, big[1:g.nnz + 1], borrow=True)
    assert e.value.code == sg.SG_ERR_INVALID
    with pytest.raises(sg.SgError):
        sg.graph_load_csr(g.row_ptr, g.col_idx, borrow=True)   # host arrays cannot be borrowed


@pytest.mark.parametrize("make", [lambda: gen.rmat(14, 16, permute=True), lambda: gen.lattice(100, 130, 0.7, seed=2),
                                  lambda: gen.rmat(12, 4, permute=True)])
def test_directed_graphs_pull_through_the_transpose(sg, make):
    """SG_F_DIRECTED ("CSR and CSC", P:299 directed datasets): push follows out-arcs,
    pull steps scan in-neighbours from the library-built CSC; BFS in every direction / loop mode and
    SSSP equal the oracle's directed BFS / Dijkstra; CC and BC refuse a directed graph."""
    g = gen.with_weights(gen.orient(make(), seed=9), seed=4)
    G = sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights, validate=True, directed=True)
    with pytest.raises(sg.SgError):          # the same arcs are not a valid symmetric graph
        sg.graph_load_csr(g.row_ptr, g.col_idx, validate=True)
    deg = g.degrees()
    for s in list(gen.sources(g, 3)) + [int(np.argmax(deg))]:
        ref = oracle.bfs(g, int(s))
        for d in (sg.SG_DIR_AUTO, sg.SG_DIR_PUSH, sg.SG_DIR_PULL):
            for hl in (False, True):
                lv, _ = sg.run_bfs(G, int(s), direction=d, host_loop=hl)
                assert np.array_equal(sg.as_u32(lv), ref), (s, d, hl)
        dist, _ = sg.run_sssp(G, int(s))
        assert np.array_equal(sg.as_u32(dist), oracle.sssp(g, int(s)))
    for fn in (lambda: sg.run_cc(G), lambda: sg.run_bc(G, [0])):
        with pytest.raises(sg.SgError) as e:
            fn()
        assert e.value.code == sg.SG_ERR_UNSUPPORTED
