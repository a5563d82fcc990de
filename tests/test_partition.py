"""Multi-GPU host logic on CPU: the 1-D destination partition rule (partition.py, the numpy mirror
of the library's), push blocks, and the communicator bootstrap over a real gloo process group
(world size 2-3).  The kernels + peer-memory exchange run in tests/test_gpu_partition.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle
from paper_conf_icpp_carocc25_b200.partition import ALIGN, Layout, partition_ranges, push_block

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


def _gloo_worker(rank, world, port, q):
    os.environ.setdefault("OMP_NUM_THREADS", "1")
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        import ctypes
        import paper_conf_icpp_carocc25_b200 as sg
        c = sg.comm_from_torch()                       # id made on rank 0, broadcast over gloo
        nr, rk = ctypes.c_int(), ctypes.c_int()
        sg.load().comm_info(c.handle, ctypes.byref(nr), ctypes.byref(rk))
        # the partition every rank derives from the same CSR is identical (what graph_load_csr
        # checks across ranks before keeping its blocks)
        g = gen.rmat(12, 16, permute=True)
        ranges = partition_ranges(g.row_ptr, world)
        obj = [None] * world
        dist.all_gather_object(obj, ranges)
        q.put((rank, nr.value, rk.value, all(o == ranges for o in obj)))
        c.free()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_bootstrap_of_the_partition_communicator(world):
    """Host side of the N > 1 path on CPU (gloo, world size 2-3): the library communicator is
    bootstrapped through torch.distributed (comm_from_torch: rank 0's id broadcast), every rank
    joins with its own rank, and every rank derives the same partition."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gloo_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res == [(r, world, r, True) for r in range(world)]


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
