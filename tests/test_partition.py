"""Multi-GPU host logic on CPU: 1-D destination partition, push blocks, and the owned-slice
all-gather protocol run with a real collective (gloo, world size 2).  The per-rank advance is
emulated on the CPU with the oracle's one-step set semantics restricted to owned destinations
(test-side code), so what is checked is the partition + exchange protocol itself: it must
reproduce the single-process BFS / label propagation exactly."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle
from paper_conf_icpp_carocc25_b200.partition import ALIGN, Layout, SliceExchange, partition_ranges, push_block

INF = 0xFFFFFFFF


def test_partition_ranges_aligned_covering_balanced():
    g = gen.rmat(16, 16, permute=True)
    for P in (1, 2, 3, 4, 8):
        rs = partition_ranges(g.row_ptr, P)
        assert rs[0][0] == 0 and rs[-1][1] == g.n
        for (a, b), (c, d) in zip(rs, rs[1:]):
            assert b == c and b % ALIGN == 0
        arcs = [int(g.row_ptr[b] - g.row_ptr[a]) for a, b in rs]
        assert max(arcs) - min(arcs) <= g.nnz / P * 0.25 + ALIGN * g.degrees().max()


def test_push_blocks_partition_the_arcs():
    g = gen.with_weights(gen.rmat(13, 16, permute=True), seed=2)
    rs = partition_ranges(g.row_ptr, 3)
    total = 0
    rows = np.repeat(np.arange(g.n), g.degrees())
    full = set(zip(rows.tolist(), g.col_idx.tolist()))
    seen = set()
    for lo, hi in rs:
        rp, ci, w = push_block(g.row_ptr, g.col_idx, g.weights, lo, hi)
        assert ((ci >= lo) & (ci < hi)).all()
        r = np.repeat(np.arange(g.n), np.diff(rp))
        pairs = set(zip(r.tolist(), ci.tolist()))
        assert not (pairs & seen)
        seen |= pairs
        total += len(ci)
        # rows sorted, weights follow their arcs
        d = np.diff(ci.astype(np.int64))
        starts = np.zeros(len(ci) + 1, bool)
        starts[rp[1:-1]] = True
        assert ((d > 0) | starts[1:-1]).all()
    assert seen == full and total == g.nnz


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _words_to_tensor(words):
    return torch.from_numpy(words.view(np.int64).copy())


def _worker(rank, world, port, scale, q):
    os.environ.setdefault("OMP_NUM_THREADS", "1")
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        g = gen.rmat(scale, 16, permute=True)
        s = int(gen.sources(g, 1)[0])
        ranges = partition_ranges(g.row_ptr, world, align=ALIGN)
        L = Layout(g.n, ranges)
        ex = SliceExchange(L, rank, world, torch.device("cpu"))
        lo, hi = ranges[rank]
        owned = np.zeros(g.n, bool)
        owned[lo:hi] = True
        # ---- BFS: replicated frontier/visited, owned-only writes, gather slices ----
        frontier = np.zeros(g.n, bool)
        frontier[s] = True
        visited = frontier.copy()
        level = np.full(g.n, -1, np.int64)
        if owned[s]:
            level[s] = 0
        d = 0
        while True:
            out_local = oracle.bfs_advance_step(g, frontier, visited) & owned       # emulated local advance
            level[out_local] = d + 1
            bits = _words_to_tensor(oracle.bitmap_words(out_local))
            summ = _words_to_tensor(oracle.summary_words(oracle.bitmap_words(out_local)))
            ex.gather_bitmap(bits, summ)
            out = oracle.words_to_mask(bits.numpy().view(np.uint64), g.n)
            # the gathered summary must be the summary of the gathered words
            assert np.array_equal(summ.numpy().view(np.uint64), oracle.summary_words(bits.numpy().view(np.uint64)))
            visited |= out
            if not out.any():
                break
            frontier = out
            d += 1
        lv = torch.from_numpy(level.astype(np.int32))
        ex.gather_values(lv)
        ok_bfs = np.array_equal(lv.numpy().view(np.uint32), oracle.bfs(g, s))
        # ---- CC label propagation with replicated labels and owned-slice gathers ----
        label = np.arange(g.n, dtype=np.int64)
        front = np.ones(g.n, bool)
        while front.any():
            new = oracle.jacobi_relax_step(g, front, label)
            new = np.where(owned, new, label)                 # a rank only writes owned labels
            t = torch.from_numpy(new.astype(np.int32))
            ex.gather_values(t)
            new = t.numpy().astype(np.int64)
            front = new < label
            label = new
        ok_cc = np.array_equal(label.astype(np.int32), oracle.cc(g))
        q.put((rank, ok_bfs, ok_cc, ex.collectives))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_two_rank_gloo_protocol_reproduces_bfs_and_cc(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, 14, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok_bfs, ok_cc, ncoll in res:
        assert ok_bfs, f"rank {rank}: distributed BFS differs from the oracle"
        assert ok_cc, f"rank {rank}: distributed CC differs from the oracle"
        assert ncoll > 0


@pytest.mark.parametrize("n,P", [(3000, 4), (4097, 3), (70000, 8), (1, 2), (8191, 8)])
def test_owned_slices_disjoint_and_covering(n, P):
    """Empty ranks (n not a multiple of the alignment, P large) own no layer-1 / layer-2 word:
    the owned word and summary slices are disjoint and cover the bitmap exactly."""
    rp = np.arange(n + 1, dtype=np.int64) * 3      # uniform degrees (values irrelevant to ownership)
    L = Layout(n, partition_ranges(rp, P))
    for get, total in ((L.word_range, L.nw1), (L.summ_range, L.nw2)):
        cover = np.zeros(total, np.int32)
        for r in range(P):
            a, b = get(r)
            assert 0 <= a <= b <= total
            cover[a:b] += 1
        assert (cover == 1).all(), (get.__name__, cover)
