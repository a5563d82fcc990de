"""The 1-D partitioned BFS on one GPU: P simulated ranks, each a push block loaded through the
C ABI, advanced with the real kernels over the replicated frontier; the all-gather is emulated
by OR-ing the disjoint owned slices (what ncclAllGather delivers).  Must equal the oracle."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu
INF = 0xFFFFFFFF


@pytest.mark.parametrize("P", [1, 2, 3, 4])
def test_partitioned_bfs_equals_oracle(P):
    import torch
    import paper_conf_icpp_carocc25_b200 as sg
    from paper_conf_icpp_carocc25_b200.partition import partition_ranges, push_block

    g = gen.rmat(15, 16, permute=True)
    s = int(gen.sources(g, 1)[0])
    ranges = partition_ranges(g.row_ptr, P)
    ranks = []
    for lo, hi in ranges:
        rp, ci, _ = push_block(g.row_ptr, g.col_idx, None, lo, hi)
        G = sg.graph_load_csr(rp, ci)
        fi, fo = sg.frontier_init(G), sg.frontier_init(G)
        sg.frontier_insert(fi, np.array([s], np.int32))
        ranks.append(dict(G=G, fi=fi, fo=fo, lo=lo, hi=hi,
                          level=torch.full((g.n,), -1, dtype=torch.int32, device="cuda"),
                          visited=torch.zeros((g.n + 63) // 64, dtype=torch.int64, device="cuda")))
    bit = 1 << (s & 63)
    for r in ranks:
        r["visited"][s >> 6] = bit - (1 << 64) if bit >= 1 << 63 else bit
        if r["lo"] <= s < r["hi"]:
            r["level"][s] = 0
    depth = 0
    while True:
        for r in ranks:
            sg.advance(r["G"], r["fi"], r["fo"], sg.SG_FN_BFS, dict(level=r["level"], visited=r["visited"], depth=depth))
        views = [sg.frontier_view(r["fo"]) for r in ranks]
        bits = views[0][0].view(torch.int64).clone()
        summ = views[0][1].view(torch.int64).clone()
        for b, sm in views[1:]:
            bits |= b.view(torch.int64)
            summ |= sm.view(torch.int64)
        for (b, sm), r in zip(views, ranks):           # "all-gather": every rank sees every slice
            b.view(torch.int64).copy_(bits)
            sm.view(torch.int64).copy_(summ)
            sg.frontier_or_into(r["fo"], r["visited"])
        if int(torch.count_nonzero(bits)) == 0:
            break
        depth += 1
        for r in ranks:
            sg.frontier_clear(r["fi"])
            r["fi"], r["fo"] = r["fo"], r["fi"]
    level = np.full(g.n, INF, np.uint32)
    for r in ranks:
        lv = sg.as_u32(r["level"])
        level[r["lo"]:r["hi"]] = lv[r["lo"]:r["hi"]]
    assert np.array_equal(level, oracle.bfs(g, s))


def test_dist_bfs_world1():
    """The production driver (partition.dist_bfs) at world size 1 through the C ABI."""
    import torch
    import paper_conf_icpp_carocc25_b200 as sg
    from paper_conf_icpp_carocc25_b200.partition import DistGraph, SliceExchange, dist_bfs

    g = gen.rmat(14, 16, permute=True)
    dg = DistGraph(g.row_ptr, g.col_idx, None, 0, 1)
    ex = SliceExchange(dg.layout, 0, 1, torch.device("cuda"))
    for s in gen.sources(g, 3):
        lv = dist_bfs(dg, int(s), ex)
        assert np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s)))


def test_dist_sssp_and_cc_world1():
    """The production SSSP / CC drivers (partition.dist_sssp / dist_cc) at world size 1."""
    import torch
    import paper_conf_icpp_carocc25_b200 as sg
    from paper_conf_icpp_carocc25_b200.partition import DistGraph, SliceExchange, dist_cc, dist_sssp

    g = gen.with_weights(gen.rmat(14, 16, permute=True), seed=5)
    dg = DistGraph(g.row_ptr, g.col_idx, g.weights, 0, 1)
    ex = SliceExchange(dg.layout, 0, 1, torch.device("cuda"))
    for s in gen.sources(g, 3):
        d = dist_sssp(dg, int(s), ex)
        assert np.array_equal(sg.as_u32(d), oracle.sssp(g, int(s)))
    lab = dist_cc(dg, ex)
    assert np.array_equal(lab.cpu().numpy(), oracle.cc(g))


@pytest.mark.parametrize("P", [2, 3])
def test_partitioned_sssp_and_cc_equal_oracle(P):
    """P simulated ranks on one GPU through the real kernels: each rank advances its push block
    over the replicated frontier and values; the all-gathers are emulated by copying each rank's
    owned slices into every rank's replicas (what ncclAllGather delivers)."""
    import torch
    import paper_conf_icpp_carocc25_b200 as sg
    from paper_conf_icpp_carocc25_b200.partition import partition_ranges, push_block

    g = gen.with_weights(gen.rmat(14, 16, permute=True), seed=7)
    ranges = partition_ranges(g.row_ptr, P)
    Gs = [sg.graph_load_csr(*push_block(g.row_ptr, g.col_idx, g.weights, lo, hi)) for lo, hi in ranges]

    def run(functor, key, init, seed_frontier):
        vals = [init() for _ in Gs]
        fr = [(sg.frontier_init(G), sg.frontier_init(G)) for G in Gs]
        for fi, _ in fr:
            seed_frontier(fi)
        for _ in range(g.n + 1):
            for G, (fi, fo), v in zip(Gs, fr, vals):
                sg.advance(G, fi, fo, functor, {key: v})
            views = [sg.frontier_view(fo) for _, fo in fr]
            bits = sum_or = views[0][0].view(torch.int64).clone()
            summ = views[0][1].view(torch.int64).clone()
            for b, sm in views[1:]:
                bits |= b.view(torch.int64)
                summ |= sm.view(torch.int64)
            full = vals[0].clone()
            for (lo, hi), v in zip(ranges, vals):
                full[lo:hi] = v[lo:hi]
            for (b, sm), v in zip(views, vals):
                b.view(torch.int64).copy_(bits)
                sm.view(torch.int64).copy_(summ)
                v.copy_(full)
            if int(torch.count_nonzero(sum_or)) == 0:
                return full
            for (fi, fo), i in zip(fr, range(len(fr))):
                sg.frontier_clear(fi)
                fr[i] = (fo, fi)
        raise AssertionError("no fixed point")

    s = int(gen.sources(g, 1)[0])

    def init_dist():
        d = torch.full((g.n,), -1, dtype=torch.int32, device="cuda")
        d[s] = 0
        return d

    dist = run(sg.SG_FN_SSSP, "dist", init_dist, lambda f: sg.frontier_insert(f, np.array([s], np.int32)))
    assert np.array_equal(sg.as_u32(dist), oracle.sssp(g, s))
    lab = run(sg.SG_FN_CC, "label", lambda: torch.arange(g.n, dtype=torch.int32, device="cuda"),
              lambda f: sg.frontier_fill_all(f))
    assert np.array_equal(lab.cpu().numpy(), oracle.cc(g))
