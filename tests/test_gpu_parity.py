"""GPU parity: the CUDA path (through the C ABI) against the pinned oracle, element by element.

BFS levels, SSSP distances and CC labels must be bit-exact; BC within
|g - o| <= 1e-9 * max(|o|, 1) (north_star; reading C21).  Sizes span several tiles
and ragged tails; tier-forcing options must not change any result."""
import numpy as np
import pytest

import gen
import oracle
from golden import twolayer_example

pytestmark = pytest.mark.gpu

INF = 0xFFFFFFFF


@pytest.fixture(scope="module")
def sg():
    import torch
    import paper_conf_icpp_carocc25_b200 as m
    torch.cuda.set_device(0)
    return m


def load(sg, g):
    return sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights, validate=True)


def bc_close(got, ref, tol=1e-9):
    return np.all(np.abs(got - ref) <= tol * np.maximum(np.abs(ref), 1.0))


# ------------------------------------------------------------------ frontier / 2LB layout
def test_frontier_layout_matches_handworked_fixture(sg):
    import torch
    n, active, words, summ = twolayer_example()
    g = gen.empty_graph(n)
    G = load(sg, g)
    f = sg.frontier_init(G)
    sg.frontier_insert(f, active.astype(np.int32))
    bits, sm = sg.frontier_view(f)
    torch.cuda.synchronize()
    assert np.array_equal(bits.cpu().numpy().view(np.uint64), words)
    assert np.array_equal(sm.cpu().numpy().view(np.uint64), summ)
    assert sg.frontier_count(f) == len(active)


@pytest.mark.parametrize("n", [1, 63, 64, 65, 4095, 4096, 4097, 100_003])
def test_fill_all_tail_and_count(sg, n):
    g = gen.empty_graph(n)
    G = load(sg, g)
    f = sg.frontier_init(G)
    sg.frontier_fill_all(f)
    bits, summ = sg.frontier_view(f)
    mask = np.ones(n, bool)
    w = oracle.bitmap_words(mask) if n <= 5000 else None
    b = bits.cpu().numpy().view(np.uint64)
    if w is not None:
        assert np.array_equal(b, w)
        assert np.array_equal(summ.cpu().numpy().view(np.uint64), oracle.summary_words(w))
    assert sg.frontier_count(f) == n
    sg.frontier_clear(f)
    assert sg.frontier_count(f) == 0


def test_frontier_set_ops(sg):
    n = 20_000
    rng = np.random.default_rng(5)
    a = rng.random(n) < 0.1
    b = rng.random(n) < 0.05
    G = load(sg, gen.empty_graph(n))
    for op, fn in enumerate([np.logical_or, np.logical_and, lambda x, y: x & ~y, np.logical_xor]):
        fa, fb = sg.frontier_init(G), sg.frontier_init(G)
        sg.frontier_insert(fa, np.nonzero(a)[0].astype(np.int32))
        sg.frontier_insert(fb, np.nonzero(b)[0].astype(np.int32))
        sg.frontier_op(fa, fb, op)
        bits, summ = sg.frontier_view(fa)
        exp = oracle.bitmap_words(fn(a, b))
        assert np.array_equal(bits.cpu().numpy().view(np.uint64), exp)
        assert np.array_equal(summ.cpu().numpy().view(np.uint64), oracle.summary_words(exp))


# ------------------------------------------------------------------------------- BFS
DIRS = ["push", "pull", "auto"]


def _dir(sg, d):
    return {"push": sg.SG_DIR_PUSH, "pull": sg.SG_DIR_PULL, "auto": sg.SG_DIR_AUTO}[d]


@pytest.mark.parametrize("host_loop", [False, True])
@pytest.mark.parametrize("direction", DIRS)
def test_bfs_config1(sg, direction, host_loop):
    g = gen.rmat(10, 16)
    G = load(sg, g)
    lv, st = sg.run_bfs(G, 0, direction=_dir(sg, direction), host_loop=host_loop)
    ref = oracle.bfs(g, 0)
    assert np.array_equal(sg.as_u32(lv), ref)
    # one superstep per level; the last level is expanded (finding nothing) unless the device
    # proves it a dead end first (every vertex visited, or a tiny last frontier whose arcs all
    # lead to visited vertices: bfs_decide / bfs_lookahead)
    L = int(ref[ref != INF].max())
    assert st.iterations in (L, L + 1)


@pytest.mark.parametrize("host_loop", [False, True])
def test_bfs_stops_when_everything_is_visited(sg, host_loop):
    """The BFS runs one superstep per level and skips the empty one after the last level when it
    can prove the last frontier a dead end: every vertex visited (path, grid, a 5,000-leaf star),
    or a tiny last frontier (<= 64 words and arcs) whose arcs all lead to visited vertices (a
    path with a second component).  A wide last level next to an unreached component (the star
    plus one extra edge) is expanded.  Levels equal the oracle in every case."""
    leaves = list(range(1, 5001))
    cases = [(gen.path(300), 299), (gen.grid(20, 30), 48), (gen.from_edges(10, [0, 1, 5], [1, 2, 6]), 2),
             (gen.from_edges(5001, [0] * 5000, leaves), 1),
             (gen.from_edges(5003, [0] * 5000 + [5001], leaves + [5002]), 2)]
    for g, want in cases:
        G = load(sg, g)
        lv, st = sg.run_bfs(G, 0, host_loop=host_loop)
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, 0))
        assert st.iterations == want, (g.n, st.iterations, want)


def test_bfs_graph_and_host_loop_agree_on_stats(sg):
    """The CUDA-graph driven loop (device-side direction policy) and the host loop take the same
    direction decisions, so levels and per-direction step counts agree."""
    g = gen.rmat(15, 16, permute=True)
    G = load(sg, g)
    for s in gen.sources(g, 4):
        a, sa = sg.run_bfs(G, int(s))
        b, sb = sg.run_bfs(G, int(s), host_loop=True)
        assert np.array_equal(sg.as_u32(a), sg.as_u32(b))
        assert (sa.iterations, sa.push_steps, sa.pull_steps) == (sb.iterations, sb.push_steps, sb.pull_steps)
        assert sa.reached == sb.reached == int((sg.as_u32(a) != INF).sum())


def test_bfs_graph_reuse_across_sources_and_buffers(sg):
    import torch
    g = gen.rmat(12, 16, permute=True)
    G = load(sg, g)
    bufs = [torch.empty(g.n, dtype=torch.int32, device="cuda") for _ in range(2)]
    for i, s in enumerate(gen.sources(g, 6)):
        lv, _ = sg.run_bfs(G, int(s), level=bufs[i % 2])
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s)))


def test_bfs_iteration_cap(sg):
    G = load(sg, gen.path(100))
    for hl in (False, True):
        with pytest.raises(sg.SgError):
            sg.run_bfs(G, 0, max_iters=10, host_loop=hl)


@pytest.mark.parametrize("opts", [dict(), dict(heavy_degree=1), dict(heavy_degree=40), dict(small_degree=-1),
                                  dict(small_degree=100000, heavy_degree=100000), dict(small_degree=3, heavy_degree=7)])
def test_bfs_tier_forcing_invariant(sg, opts):
    g = gen.rmat(14, 16, permute=True)
    G = load(sg, g)
    for s in gen.sources(g, 3):
        lv, _ = sg.run_bfs(G, int(s), direction=sg.SG_DIR_PUSH, **opts)
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s))), (opts, s)


@pytest.mark.parametrize("kw", [dict(one_layer=True), dict(one_layer=True, coarsening=1, small_degree=-1),
                                dict(coarsening=7), dict(coarsening=1, heavy_degree=1 << 30)])
def test_bfs_ablation_knobs_do_not_change_results(sg, kw):
    """Fig. 7 ablation switches (plain one-layer bitmap, coarsening factor) keep levels exact."""
    g = gen.rmat(15, 12)
    G = load(sg, g)
    for s in gen.sources(g, 3):
        for d in (sg.SG_DIR_PUSH, sg.SG_DIR_AUTO):
            lv, _ = sg.run_bfs(G, int(s), direction=d, host_loop=True, **kw)
            assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s))), (kw, d)


@pytest.mark.parametrize("host_loop", [False, True])
@pytest.mark.parametrize("make", [lambda: gen.rmat(14, 16, permute=True), lambda: gen.rmat(21, 8, permute=True),
                                  lambda: gen.rmat(20, 16)])
def test_bfs_segmented_hub_tier(sg, make, host_loop):
    """Hubs (deg >= 256) through the destination-segmented tier (visited slice in shared memory),
    forced on every superstep; RMAT-21 spans 3 segments of 802,816 vertices."""
    g = make()
    G = load(sg, g)
    for s in list(gen.sources(g, 2)) + [int(np.argmax(g.degrees()))]:
        for d in (sg.SG_DIR_PUSH, sg.SG_DIR_AUTO):
            lv, _ = sg.run_bfs(G, int(s), direction=d, segmented=2, host_loop=host_loop)
            assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s))), (s, d)


@pytest.mark.parametrize("deg", [255, 256, 257, 4097, 900_000])
def test_bfs_segmented_degree_boundaries(sg, deg):
    n = deg + 1 + 50
    u = np.concatenate([np.zeros(deg, np.int64), np.arange(deg, n - 1)])
    v = np.concatenate([np.arange(1, deg + 1), np.arange(deg + 1, n)])
    g = gen.from_edges(n, u, v)
    G = load(sg, g)
    for s in (0, 1, n - 1):
        lv, _ = sg.run_bfs(G, s, direction=sg.SG_DIR_PUSH, segmented=2)
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, s)), (deg, s)


@pytest.mark.parametrize("make", [lambda: gen.path(5000), lambda: gen.cycle(4097), lambda: gen.grid(97, 131),
                                  lambda: gen.hypercube(16), lambda: gen.complete(300), lambda: gen.star(70_000),
                                  lambda: gen.lattice(300, 400, 0.6)])
@pytest.mark.parametrize("direction", DIRS)
def test_bfs_closed_form_families(sg, make, direction):
    g = make()
    G = load(sg, g)
    for s in [0, g.n // 2, g.n - 1]:
        lv, _ = sg.run_bfs(G, s, direction=_dir(sg, direction))
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, s))


@pytest.mark.parametrize("deg", [1, 31, 32, 33, 2047, 2048, 2049, 4095, 4096, 4097, 65536, 200_001])
def test_bfs_degree_tier_boundaries(sg, deg):
    # a hub of degree `deg` plus a tail path so several levels exist
    n = deg + 1 + 50
    u = np.concatenate([np.zeros(deg, np.int64), np.arange(deg, n - 1)])
    v = np.concatenate([np.arange(1, deg + 1), np.arange(deg + 1, n)])
    g = gen.from_edges(n, u, v)
    G = load(sg, g)
    for s in (0, 1, n - 1):
        for d in (sg.SG_DIR_PUSH, sg.SG_DIR_AUTO):
            lv, _ = sg.run_bfs(G, s, direction=d)
            assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, s)), (deg, s, d)


@pytest.mark.parametrize("n", [4096 * 3 + 77, 4096 * 5, 64 * 70 + 1])
@pytest.mark.parametrize("direction", ["pull", "auto"])
def test_bfs_pull_fully_visited_words(sg, n, direction):
    """Pull steps over frontiers where whole layer-2 words (4,096 vertices) and single layer-1
    words are already visited (the pull's skip paths), next to words with a few unvisited
    vertices left: a dense random core over the first half (visited after 2-3 levels), a long
    path through the rest, small components scattered into otherwise visited words, isolated
    vertices and a ragged tail."""
    rng = np.random.default_rng(n)
    h = n // 2
    cu = rng.integers(0, h, 24 * h)
    cv = rng.integers(0, h, 24 * h)
    pu = np.arange(h - 1, n - 200)   # path from the core's last vertex through the second half
    iso = rng.choice(np.arange(1, h), 40, replace=False)   # pairs / triangles inside the core words
    tu = np.concatenate([iso[0:40:2]])
    tv = np.concatenate([iso[1:40:2]])
    keep = ~(np.isin(cu, iso) | np.isin(cv, iso))
    g = gen.from_edges(n, np.concatenate([cu[keep], pu, tu]), np.concatenate([cv[keep], pu + 1, tv]))
    G = load(sg, g)
    for s in (0, 5, h + 1000, n - 201):
        lv, st = sg.run_bfs(G, s, direction=_dir(sg, direction))
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, s)), (n, s)
        lv2, _ = sg.run_bfs(G, s, direction=_dir(sg, direction), host_loop=True)
        assert np.array_equal(sg.as_u32(lv2), oracle.bfs(g, s)), (n, s)


def test_bfs_isolated_source_and_empty_graph(sg):
    g = gen.rmat(10, 16)
    iso = int(np.nonzero(g.degrees() == 0)[0][0])
    G = load(sg, g)
    lv, st = sg.run_bfs(G, iso)
    exp = np.full(g.n, INF, np.uint32)
    exp[iso] = 0
    assert np.array_equal(sg.as_u32(lv), exp) and st.iterations == 1
    G0 = load(sg, gen.empty_graph(1))
    lv, _ = sg.run_bfs(G0, 0)
    assert sg.as_u32(lv)[0] == 0


def test_bfs_rejects_bad_source(sg):
    G = load(sg, gen.path(10))
    with pytest.raises(sg.SgError):
        sg.run_bfs(G, 10)
    with pytest.raises(sg.SgError):
        sg.run_bfs(G, -1)


@pytest.mark.parametrize("direction", DIRS)
def test_bfs_rmat16_many_sources(sg, direction):
    g = gen.rmat(16, 32, permute=True)
    G = load(sg, g)
    for s in gen.sources(g, 5):
        lv, _ = sg.run_bfs(G, int(s), direction=_dir(sg, direction))
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s)))


# ------------------------------------------- destination-segmented (SCSR) push advance
@pytest.mark.parametrize("sw", [0, 1, 3, 64])
@pytest.mark.parametrize("host_loop", [False, True])
def test_bfs_scsr_forced(sg, monkeypatch, sw, host_loop):
    """Every push superstep through the segment-major arc copy (scsr=2) with segments of 64*sw
    vertices (sw=0: the default 24,576 words, one segment here; sw=1: 256 segments of 64
    vertices; sw=3: ragged last segment), push-only and direction-optimising."""
    if sw:
        monkeypatch.setenv("SG_SCSR_WORDS", str(sw))
    for g in (gen.rmat(14, 16, permute=True), gen.rmat(12, 8)):
        G = load(sg, g)
        for s in list(gen.sources(g, 2)) + [int(np.argmax(g.degrees()))]:
            for d in (sg.SG_DIR_PUSH, sg.SG_DIR_AUTO):
                lv, _ = sg.run_bfs(G, int(s), direction=d, scsr=2, host_loop=host_loop)
                assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s))), (sw, s, d)


@pytest.mark.parametrize("deg", [254, 255, 256, 511, 70_000])
@pytest.mark.parametrize("sw", [0, 8])
def test_bfs_scsr_part_length_escapes(sg, monkeypatch, deg, sw):
    """Part lengths >= 255 arcs (a hub's neighbours inside one segment) take the exact offset
    table: a star of degree `deg` plus a tail path, segments of 64*sw vertices."""
    if sw:
        monkeypatch.setenv("SG_SCSR_WORDS", str(sw))
    n = deg + 1 + 50
    u = np.concatenate([np.zeros(deg, np.int64), np.arange(deg, n - 1)])
    v = np.concatenate([np.arange(1, deg + 1), np.arange(deg + 1, n)])
    g = gen.from_edges(n, u, v)
    G = load(sg, g)
    for s in (0, 1, n - 1):
        for hl in (False, True):
            lv, _ = sg.run_bfs(G, s, direction=sg.SG_DIR_PUSH, scsr=2, host_loop=hl)
            assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, s)), (deg, sw, s, hl)


def test_bfs_scsr_auto_matches_word_path_multi_segment(sg, monkeypatch):
    """Auto policy (sweep on supersteps with m_f >= nnz/8) with 8 segments (RMAT-17, 64*256-vertex
    segments): scsr auto / off / always give identical levels and step counts."""
    monkeypatch.setenv("SG_SCSR_WORDS", "256")
    monkeypatch.setenv("SG_SWEEP_MIN_M", "0")
    monkeypatch.setenv("SG_SWEEP_FRAC64", "8")
    g = gen.rmat(17, 16, permute=True)
    G = load(sg, g)
    for s in gen.sources(g, 3):
        ref = oracle.bfs(g, int(s))
        stats = []
        for mode in (0, 1, 2):
            lv, st = sg.run_bfs(G, int(s), scsr=mode)
            assert np.array_equal(sg.as_u32(lv), ref), mode
            stats.append((st.iterations, st.push_steps, st.pull_steps, st.reached))
        assert stats[0] == stats[1] == stats[2]


# ---------------------------------------------------------------------- one advance step
def test_single_bfs_advance_step_set_semantics(sg):
    import torch
    g = gen.rmat(13, 16, permute=True)
    G = load(sg, g)
    s = int(gen.sources(g, 1)[0])
    lvl = oracle.bfs(g, s)
    fin, fout = sg.frontier_init(G), sg.frontier_init(G)
    level = torch.full((g.n,), -1, dtype=torch.int32, device="cuda")
    visited = torch.zeros((g.n + 63) // 64, dtype=torch.int64, device="cuda")
    for d in range(int(lvl[lvl != INF].max()) + 1):
        frontier = lvl == d
        vis = lvl <= d
        # state before step d: visited = levels <= d, level set for those
        visited.copy_(torch.from_numpy(oracle.bitmap_words(vis).view(np.int64)))
        lv_host = np.where(vis, lvl, INF).astype(np.uint32)
        level.copy_(torch.from_numpy(lv_host.view(np.int32)))
        sg.frontier_clear(fin)
        sg.frontier_clear(fout)
        sg.frontier_insert(fin, np.nonzero(frontier)[0].astype(np.int32))
        sg.advance(G, fin, fout, sg.SG_FN_BFS, dict(level=level, visited=visited, depth=d))
        bits, summ = sg.frontier_view(fout)
        exp = oracle.bfs_advance_step(g, frontier, vis)
        ew = oracle.bitmap_words(exp)
        assert np.array_equal(bits.cpu().numpy().view(np.uint64), ew)
        assert np.array_equal(summ.cpu().numpy().view(np.uint64), oracle.summary_words(ew))
        got_lv = sg.as_u32(level)
        assert np.array_equal(got_lv[exp], np.full(exp.sum(), d + 1, np.uint32))


def test_single_relax_step_invariants(sg):
    """SSSP/CC steps are non-unique under asynchronous updates (reading C12): check
    out == {v: value decreased}, final >= fixed point, and <= the Jacobi step bound."""
    import torch
    g = gen.with_weights(gen.rmat(12, 16, permute=True), seed=4)
    G = load(sg, g)
    s = int(gen.sources(g, 1)[0])
    ref = oracle.sssp(g, s).astype(np.int64)
    dist = np.full(g.n, INF, np.int64)
    dist[s] = 0
    front = np.zeros(g.n, bool)
    front[s] = True
    fin, fout = sg.frontier_init(G), sg.frontier_init(G)
    dd = torch.empty(g.n, dtype=torch.int32, device="cuda")
    for _ in range(200):
        if not front.any():
            break
        dd.copy_(torch.from_numpy(dist.astype(np.uint32).view(np.int32)))
        sg.frontier_clear(fin)
        sg.frontier_clear(fout)
        sg.frontier_insert(fin, np.nonzero(front)[0].astype(np.int32))
        sg.advance(G, fin, fout, sg.SG_FN_SSSP, dict(dist=dd))
        new = sg.as_u32(dd).astype(np.int64)
        bits, _ = sg.frontier_view(fout)
        out = oracle.words_to_mask(bits.cpu().numpy().view(np.uint64), g.n)
        assert np.array_equal(out, new < dist)
        assert (new >= ref).all()
        assert (new <= oracle.jacobi_relax_step(g, front, dist, g.weights)).all()
        dist, front = new, out
    assert np.array_equal(dist, ref)


# ------------------------------------------------------------------------------ SSSP
@pytest.mark.parametrize("scale,ef,perm", [(10, 16, False), (14, 16, True), (16, 8, False)])
def test_sssp_rmat(sg, scale, ef, perm):
    g = gen.with_weights(gen.rmat(scale, ef, permute=perm), seed=1)
    G = load(sg, g)
    for s in [0] + list(gen.sources(g, 3)):
        d, _ = sg.run_sssp(G, int(s))
        assert np.array_equal(sg.as_u32(d), oracle.sssp(g, int(s)))


@pytest.mark.parametrize("opts", [dict(heavy_degree=1), dict(small_degree=-1), dict(small_degree=5000, heavy_degree=5000)])
def test_sssp_tiers(sg, opts):
    g = gen.with_weights(gen.rmat(13, 16), seed=2)
    G = load(sg, g)
    d, _ = sg.run_sssp(G, 0, **opts)
    assert np.array_equal(sg.as_u32(d), oracle.sssp(g, 0))


def test_sssp_lattice_and_unit_weights(sg):
    g = gen.with_weights(gen.lattice(200, 300, 0.7), seed=9)
    G = load(sg, g)
    s = int(gen.sources(g, 1, stream=6)[0])
    d, _ = sg.run_sssp(G, s)
    assert np.array_equal(sg.as_u32(d), oracle.sssp(g, s))
    g2 = gen.rmat(12, 16)
    g2.weights = np.ones(g2.nnz, np.uint8)
    G2 = load(sg, g2)
    d, _ = sg.run_sssp(G2, 0)
    assert np.array_equal(sg.as_u32(d), oracle.bfs(g2, 0))


@pytest.mark.parametrize("delta", [1, 7, 64, 100_000])
@pytest.mark.parametrize("make", [lambda: gen.with_weights(gen.rmat(14, 16, permute=True), seed=3),
                                  lambda: gen.with_weights(gen.lattice(150, 200, 0.7), seed=5)])
def test_sssp_delta_stepping(sg, make, delta):
    """Near-far delta-stepping (f4) reaches the same distances as Dijkstra for any bucket width."""
    g = make()
    G = load(sg, g)
    for s in gen.sources(g, 2, stream=6):
        d, st = sg.run_sssp(G, int(s), sssp_delta=delta)
        assert np.array_equal(sg.as_u32(d), oracle.sssp(g, int(s))), (delta, s)


def test_sssp_requires_weights(sg):
    G = load(sg, gen.path(10))
    with pytest.raises(sg.SgError):
        sg.run_sssp(G, 0)


# -------------------------------------------------------------------------------- CC
@pytest.mark.parametrize("make", [lambda: gen.gnm(300_000, 150_000, seed=3), lambda: gen.gnm(100_000, 1_200_000),
                                  lambda: gen.rmat(15, 8, permute=True), lambda: gen.lattice(300, 300, 0.5),
                                  lambda: gen.empty_graph(1000), lambda: gen.path(3000)])
def test_cc(sg, make):
    g = make()
    G = load(sg, g)
    lab, _ = sg.run_cc(G)
    assert np.array_equal(lab.cpu().numpy(), oracle.cc(g))


def test_cc_tiers(sg):
    g = gen.rmat(13, 16)
    G = load(sg, g)
    ref = oracle.cc(g)
    for opts in (dict(heavy_degree=1), dict(small_degree=-1), dict(small_degree=100000, heavy_degree=100000)):
        lab, _ = sg.run_cc(G, direction=sg.SG_DIR_PUSH, **opts)
        assert np.array_equal(lab.cpu().numpy(), ref)


@pytest.mark.parametrize("make", [lambda: gen.gnm(200_000, 1_000_000), lambda: gen.rmat(14, 8, permute=True),
                                  lambda: gen.lattice(200, 300, 0.55), lambda: gen.gnm(100_003, 40_000, seed=7)])
def test_cc_directions_agree(sg, make):
    """push-only, pull-only and auto (pull on dense supersteps) reach the same min labels."""
    g = make()
    G = load(sg, g)
    ref = oracle.cc(g)
    for d in (sg.SG_DIR_PUSH, sg.SG_DIR_PULL, sg.SG_DIR_AUTO):
        lab, st = sg.run_cc(G, direction=d)
        assert np.array_equal(lab.cpu().numpy(), ref), d


@pytest.mark.parametrize("kb", [4, 64, 1000])
@pytest.mark.parametrize("make", [lambda: gen.gnm(200_000, 1_000_000), lambda: gen.rmat(15, 16, permute=True),
                                  lambda: gen.lattice(300, 300, 0.55), lambda: gen.gnm(100_003, 40_000, seed=7)])
def test_cc_label_blocked_pull(sg, monkeypatch, make, kb):
    """Label-blocked pull (one pass per label block of kb KB; block boundaries inside rows, ragged
    last block, up to 64 blocks) reaches the union-find labels, for pull-only and auto."""
    monkeypatch.setenv("SG_CC_LBLOCK_KB", str(kb))
    g = make()
    G = load(sg, g)
    ref = oracle.cc(g)
    for d in (sg.SG_DIR_PULL, sg.SG_DIR_AUTO):
        lab, _ = sg.run_cc(G, direction=d)
        assert np.array_equal(lab.cpu().numpy(), ref), (d, kb)


# -------------------------------------------------------------------------------- BC
@pytest.mark.parametrize("make,k", [(lambda: gen.random_simple(60, 0.08, 3), 60), (lambda: gen.path(300), 10),
                                    (lambda: gen.hypercube(10), 5), (lambda: gen.rmat(12, 16, permute=True), 8),
                                    (lambda: gen.lattice(80, 120, 0.6, seed=2), 6)])
@pytest.mark.parametrize("per_source", [False, True])
def test_bc(sg, make, k, per_source):
    """Default = source-batched (32 sources per graph launch); per_source = one BFS pair per source."""
    g = make()
    G = load(sg, g)
    srcs = gen.sources(g, k) if k < g.n else np.arange(g.n, dtype=np.int32)
    bc, _ = sg.run_bc(G, srcs, host_loop=per_source)
    assert bc_close(bc.cpu().numpy(), oracle.bc(g, srcs))


def test_bc_batches_of_32_with_ragged_tail_and_duplicates(sg):
    g = gen.lattice(60, 70, 0.7, seed=4)
    G = load(sg, g)
    srcs = np.concatenate([gen.sources(g, 70, stream=6), gen.sources(g, 3, stream=6)])   # 73 = 32+32+9, dups
    bc, st = sg.run_bc(G, srcs)
    assert bc_close(bc.cpu().numpy(), oracle.bc(g, srcs))
    bc2, _ = sg.run_bc(G, srcs, host_loop=True)
    assert bc_close(bc.cpu().numpy(), bc2.cpu().numpy(), 1e-12)


def test_bc_sigma_beyond_fp64_range(sg):
    """Full 600x600 grid from a corner: sigma reaches ~2^1193 > DBL_MAX (reading C20); the
    per-level exponent scaling must keep BC exact to 1e-9."""
    g = gen.grid(600, 600)
    G = load(sg, g)
    srcs = np.array([0, 600 * 600 - 1], np.int32)
    bc, _ = sg.run_bc(G, srcs)
    assert bc_close(bc.cpu().numpy(), oracle.bc(g, srcs))


def test_bc_duplicates_and_isolated(sg):
    g = gen.from_edges(8, [0, 1, 2, 3], [1, 2, 3, 4])
    G = load(sg, g)
    srcs = [0, 0, 7, 2]
    bc, _ = sg.run_bc(G, srcs)
    assert bc_close(bc.cpu().numpy(), oracle.bc(g, srcs))


@pytest.mark.parametrize("make", [lambda: gen.rmat(14, 16, permute=True), lambda: gen.path(300),
                                  lambda: gen.lattice(90, 120, 0.6, seed=3), lambda: gen.rmat(12, 4, permute=True)])
def test_bfs_fused_sparse_supersteps(sg, monkeypatch, make):
    """SG_SPARSE=1: small push supersteps run in the fused persistent loop (sparse.cu: direct output
    insertion, the input zeroed as consumed, dirty output buffers cleared first, 256-arc items for
    long lists, several supersteps per launch ending on either buffer parity); levels and step
    counts equal the default path's and the oracle's."""
    g = make()
    G = load(sg, g)
    for s in list(gen.sources(g, 3)) + [int(np.argmax(g.degrees()))]:
        ref = oracle.bfs(g, int(s))
        monkeypatch.setenv("SG_SPARSE", "0")
        _, st0 = sg.run_bfs(G, int(s))
        for arcs in ("65536", "300", "0"):
            monkeypatch.setenv("SG_SPARSE", "1")
            monkeypatch.setenv("SG_SPARSE_ARCS", arcs)
            for d in (sg.SG_DIR_AUTO, sg.SG_DIR_PUSH):
                lv, st = sg.run_bfs(G, int(s), direction=d)
                assert np.array_equal(sg.as_u32(lv), ref), (s, arcs, d)
            _, st = sg.run_bfs(G, int(s))
            assert (st.iterations, st.push_steps, st.pull_steps) == (st0.iterations, st0.push_steps, st0.pull_steps)


@pytest.mark.parametrize("make", [lambda: gen.with_weights(gen.rmat(14, 16, permute=True), seed=2),
                                  lambda: gen.with_weights(gen.lattice(120, 150, 0.6, seed=5), seed=3),
                                  lambda: gen.with_weights(gen.gnm(50_000, 30_000, seed=4), seed=4)])
def test_sssp_cc_graph_driven_equals_host_loop(sg, monkeypatch, make):
    """The device-driven SSSP / CC loops (CUDA graph, val_decide) give the oracle's values, as the
    host loop does, for every direction and with label-blocked CC pulls.  (Superstep counts are
    not compared: with asynchronous relaxation, reading C12, a superstep's frontier depends on
    the order its atomics land in.)"""
    g = make()
    G = load(sg, g)
    for s in gen.sources(g, 2):
        d, st = sg.run_sssp(G, int(s))
        d2, st2 = sg.run_sssp(G, int(s), host_loop=True)
        ref = oracle.sssp(g, int(s))
        assert np.array_equal(sg.as_u32(d), ref) and np.array_equal(sg.as_u32(d2), ref)
    ref = oracle.cc(g)
    for kb in ("32768", "8"):
        monkeypatch.setenv("SG_CC_LBLOCK_KB", kb)
        for dr in (sg.SG_DIR_AUTO, sg.SG_DIR_PUSH, sg.SG_DIR_PULL):
            lab, st = sg.run_cc(G, direction=dr)
            lab2, st2 = sg.run_cc(G, direction=dr, host_loop=True)
            assert np.array_equal(lab.cpu().numpy(), ref) and np.array_equal(lab2.cpu().numpy(), ref)
            assert st.iterations >= 1 and st.push_steps + st.pull_steps == st.iterations


@pytest.mark.parametrize("bits", [32, 64])
@pytest.mark.parametrize("make", [lambda: gen.rmat(13, 16, permute=True), lambda: gen.path(200),
                                  lambda: gen.lattice(70, 90, 0.6, seed=2), lambda: gen.empty_graph(100)])
def test_word_width_ablation_bfs(sg, make, bits):
    """sg_ablation_bfs (f3): the 32- and 64-bit-word push-only 2LB BFS reach the oracle's levels."""
    g = make()
    G = load(sg, g)
    for s in list(gen.sources(g, 2)) + [0, g.n - 1]:
        lv, st = sg.ablation_bfs(G, int(s), bits)
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s))), (bits, s)


@pytest.mark.parametrize("word_max", ["0", "4", "64"])
@pytest.mark.parametrize("host_loop", [False, True])
def test_bfs_pull_word_mode_threshold(sg, monkeypatch, word_max, host_loop):
    """The CTA pull's word mode (a thread per layer-1 word, pull.cu) is a runtime threshold:
    off (0), narrow (4) and forced on dense words (64) all give the oracle's levels, with and
    without the late warp-owned pulls (SG_PULL_WARP_FRAC=0 keeps every pull on the CTA kernel)."""
    g = gen.rmat(15, 16, permute=True)
    G = load(sg, g)
    monkeypatch.setenv("SG_PULL_WORD_MAX", word_max)
    for frac in ("0", "8"):
        monkeypatch.setenv("SG_PULL_WARP_FRAC", frac)
        for s in gen.sources(g, 3):
            ref = oracle.bfs(g, int(s))
            for d in (sg.SG_DIR_PULL, sg.SG_DIR_AUTO):
                lv, _ = sg.run_bfs(G, int(s), direction=d, host_loop=host_loop)
                assert np.array_equal(sg.as_u32(lv), ref), (word_max, frac, d)


@pytest.mark.parametrize("name,defines", [
    ("pull128", ("SG_PULL_THREADS=128",)),
    ("pullnoq", ("SG_PULL_QUEUE=0",)),
    ("pullq2", ("SG_PULLQ_SHORT=2", "SG_PULLQ2_CAP=4")),
])
def test_bfs_pull_build_variants(sg, name, defines):
    """Compile-time layouts of the CTA pull, each built as its own library and run in a
    subprocess: 128-thread CTAs (a measured round-1 variant), the per-thread list scan without
    the miss queue, and the queue with a 2-arc stage A and a 4-row stage-B queue (so stage B and
    its overflow path, the thread scanning the rest itself, both run).  Pull-only and auto BFS
    equal the oracle."""
    import os
    import subprocess
    import sys
    from paper_conf_icpp_carocc25_b200 import _build
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    lib = _build.build(defines=defines, lib=os.path.join(root, "build", "variants", name, "libsygraph.so"))
    code = ("import numpy as np, gen, oracle, paper_conf_icpp_carocc25_b200 as sg\n"
            "for g in (gen.rmat(14, 16, permute=True), gen.rmat(16, 4, permute=True)):\n"
            "    G = sg.graph_load_csr(g.row_ptr, g.col_idx)\n"
            "    for s in gen.sources(g, 3):\n"
            "        for d in (sg.SG_DIR_PULL, sg.SG_DIR_AUTO):\n"
            "            lv, _ = sg.run_bfs(G, int(s), direction=d)\n"
            "            assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s)))\n"
            "print('ok')\n")
    env = dict(os.environ, SYGRAPH_LIB=lib, PYTHONPATH=root)
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, cwd=root)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-2000:]


def _deg8_decoded(d):
    """The library's 8-bit degree code (exact below 32, 3 mantissa bits above) decoded: the m_f
    unit of the direction policy (frontier.cu k_deg8 / common.cuh deg8_decode)."""
    d = np.asarray(d, dtype=np.int64)
    out = d.copy()
    big = d >= 32
    e = np.floor(np.log2(np.maximum(d, 1))).astype(np.int64)
    m = (d >> np.maximum(e - 3, 0)) & 7
    code = np.minimum(32 + (e - 5) * 8 + m, 255)
    e2 = ((code - 32) >> 3) + 5
    m2 = (code - 32) & 7
    out[big] = (((8 + m2) << (e2 - 3)) + (1 << (e2 - 4)))[big]
    return out


@pytest.mark.parametrize("direction", DIRS)
def test_bfs_trace_frontier_statistics(sg, direction):
    """n_f and m_f of every BFS frontier as the output kernels sum them (quad_mf: the dp4a path
    for degrees < 32, the table path for coded ones) equal the level sizes and the decoded degree
    sums of the oracle's levels, on a graph with hubs and low-degree vertices mixed in quads."""
    g = gen.rmat(14, 16, permute=True)
    G = load(sg, g)
    dec = _deg8_decoded(g.degrees())
    for s in gen.sources(g, 2):
        ref = oracle.bfs(g, int(s))
        lv, st = sg.run_bfs(G, int(s), direction=_dir(sg, direction))
        assert np.array_equal(sg.as_u32(lv), ref)
        for t in sg.bfs_trace(G):
            at = ref == t["step"]
            assert t["nf"] == int(at.sum()), t
            assert t["mf"] == int(dec[at].sum()), t
