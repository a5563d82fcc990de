"""1-D destination partitioning across GPUs (§6 "static graph
partitioning ... each GPU handles a local subgraph").

Rank r owns the vertex range [lo_r, hi_r): ranges are aligned to 4,096 vertices (one layer-2
word, so every rank owns whole layer-1 *and* layer-2 words) and balanced by degree (the graph is
symmetric, so out-degree = in-degree = the arcs a rank receives).  Each rank stores the *push
block*: all arcs (u -> v) with v owned, as a CSR over all n sources.  A superstep is

    local advance over the replicated input frontier   (only owned bits / values are written)
    ncclAllGather of the owned layer-1 + layer-2 slices (2 MB + 32 KB at n = 2^24)
    [SSSP / CC: ncclAllGather of the owned value slice]

so no cross-GPU atomics are needed and every rank sees the same next frontier (same direction
and termination decisions without an extra collective).  The exchange runs through
torch.distributed (NCCL on GPUs, gloo in the CPU tests); the advance is the C ABI's.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

ALIGN = 4096          # vertices per layer-2 word


def partition_ranges(row_ptr: np.ndarray, parts: int, align: int = ALIGN) -> list[tuple[int, int]]:
    """Contiguous, `align`-aligned vertex ranges with ~equal arc counts (last range ends at n)."""
    n = len(row_ptr) - 1
    nnz = int(row_ptr[-1])
    bounds = [0]
    for r in range(1, parts):
        target = nnz * r // parts
        v = int(np.searchsorted(row_ptr, target, side="left"))
        v = min(max((v + align // 2) // align * align, bounds[-1]), n)
        bounds.append(v)
    bounds.append(n)
    return [(bounds[i], bounds[i + 1]) for i in range(parts)]


def push_block(row_ptr: np.ndarray, col_idx: np.ndarray, weights, lo: int, hi: int):
    """CSR over all sources holding only the arcs whose destination lies in [lo, hi).
    Rows stay sorted (a sub-range of each sorted row)."""
    n = len(row_ptr) - 1
    keep = (col_idx >= lo) & (col_idx < hi)
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(row_ptr))
    counts = np.bincount(src[keep], minlength=n)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    ci = np.ascontiguousarray(col_idx[keep])
    w = np.ascontiguousarray(weights[keep]) if weights is not None else None
    return rp, ci, w


@dataclass
class Layout:
    n: int
    ranges: list

    @property
    def nw1(self):
        return (self.n + 63) // 64

    @property
    def nw2(self):
        return (self.nw1 + 63) // 64

    def word_range(self, r):      # owned layer-1 words (empty vertex range -> empty word range)
        lo, hi = self.ranges[r]
        if hi <= lo:
            return lo // 64, lo // 64
        return lo // 64, min((hi + 63) // 64, self.nw1)

    def summ_range(self, r):      # owned layer-2 words
        a, b = self.word_range(r)
        if b <= a:
            return a // 64, a // 64
        return a // 64, min((b + 63) // 64, self.nw2)


class SliceExchange:
    """All-gather of owned slices with equal-size (padded) chunks, as ncclAllGather requires."""

    def __init__(self, layout: Layout, rank: int, world: int, device, group=None):
        import torch
        self.L, self.rank, self.world, self.device, self.group = layout, rank, world, device, group
        self.torch = torch
        self.w_max = max(b - a for a, b in (layout.word_range(r) for r in range(world)))
        self.s_max = max(b - a for a, b in (layout.summ_range(r) for r in range(world)))
        self.v_max = max(hi - lo for lo, hi in layout.ranges)
        self.collectives = 0

    def _gather(self, full, ranges, chunk):
        """full: 1-D tensor; ranges[r] = (a, b) slice owned by rank r; writes every slice in place."""
        torch = self.torch
        if self.world == 1:
            return full
        a, b = ranges[self.rank]
        send = torch.zeros(chunk, dtype=full.dtype, device=full.device)
        send[: b - a] = full[a:b]
        recv = torch.empty(chunk * self.world, dtype=full.dtype, device=full.device)
        torch.distributed.all_gather_into_tensor(recv, send, group=self.group)
        self.collectives += 1
        for r, (ra, rb) in enumerate(ranges):
            if r != self.rank and rb > ra:   # empty ranks own nothing (never overwrite a real slice)
                full[ra:rb] = recv[r * chunk: r * chunk + (rb - ra)]
        return full

    def gather_bitmap(self, bits, summ):
        """bits: int64[nw1], summ: int64[nw2] views of a 2LB frontier."""
        self._gather(bits, [self.L.word_range(r) for r in range(self.world)], self.w_max)
        self._gather(summ, [self.L.summ_range(r) for r in range(self.world)], self.s_max)

    def gather_values(self, values):
        """values: per-vertex tensor (int32 / float64); owned slices replicated everywhere."""
        self._gather(values, self.L.ranges, self.v_max)


# ------------------------------------------------------------------------------------------
# Distributed drivers on top of the C ABI (one process per GPU).
class DistGraph:
    """This rank's push block loaded through graph_load_csr, plus the partition layout."""

    def __init__(self, row_ptr, col_idx, weights, rank, world, stream=None):
        import paper_conf_icpp_carocc25_b200 as sg
        self.sg = sg
        self.n = len(row_ptr) - 1
        self.ranges = partition_ranges(row_ptr, world)
        self.layout = Layout(self.n, self.ranges)
        lo, hi = self.ranges[rank]
        rp, ci, w = push_block(row_ptr, col_idx, weights, lo, hi)
        self.G = sg.graph_load_csr(rp, ci, w, stream=stream)
        self.rank, self.world = rank, world


def dist_bfs(dg: DistGraph, src: int, exchange: SliceExchange, max_iters: int | None = None):
    """Level-synchronous push BFS over the 1-D partition; returns the full level array (int32
    storage of uint32 levels, replicated on every rank)."""
    import torch
    sg = dg.sg
    n = dg.n
    dev = torch.device("cuda", torch.cuda.current_device())
    level = torch.full((n,), -1, dtype=torch.int32, device=dev)
    visited = torch.zeros(dg.layout.nw1, dtype=torch.int64, device=dev)
    fin, fout = sg.frontier_init(dg.G), sg.frontier_init(dg.G)
    sg.frontier_insert(fin, np.array([src], dtype=np.int32))
    lo, hi = dg.ranges[dg.rank]
    if lo <= src < hi:
        level[src] = 0
    bit = 1 << (src & 63)
    visited[src >> 6] = bit - (1 << 64) if bit >= 1 << 63 else bit
    depth = 0
    cap = max_iters or n + 1
    while True:
        sg.advance(dg.G, fin, fout, sg.SG_FN_BFS, dict(level=level, visited=visited, depth=depth))
        bits, summ = sg.frontier_view(fout)
        exchange.gather_bitmap(bits.view(torch.int64), summ.view(torch.int64))
        sg.frontier_or_into(fout, visited)
        if sg.frontier_count(fout) == 0:
            break
        depth += 1
        if depth > cap:
            raise RuntimeError("iteration cap reached")
        sg.frontier_clear(fin)
        fin, fout = fout, fin
    exchange.gather_values(level)
    return level


def _exchange_frontier(sg, exchange, fout):
    import torch
    bits, summ = sg.frontier_view(fout)
    exchange.gather_bitmap(bits.view(torch.int64), summ.view(torch.int64))


def dist_sssp(dg: DistGraph, src: int, exchange: SliceExchange, max_iters: int | None = None):
    """Bellman-Ford by frontier over the 1-D partition: each rank relaxes the arcs of its
    push block (only owned distances change, no cross-GPU atomics), then the owned slices of the
    output frontier and of dist are all-gathered.  Returns the full dist array (int32 storage of
    uint32 distances, UINT32_MAX = unreached), replicated on every rank."""
    import torch
    sg = dg.sg
    n = dg.n
    dev = torch.device("cuda", torch.cuda.current_device())
    dist = torch.full((n,), -1, dtype=torch.int32, device=dev)
    dist[src] = 0
    fin, fout = sg.frontier_init(dg.G), sg.frontier_init(dg.G)
    sg.frontier_insert(fin, np.array([src], dtype=np.int32))
    cap = max_iters or n + 1
    it = 0
    while True:
        sg.advance(dg.G, fin, fout, sg.SG_FN_SSSP, dict(dist=dist))
        _exchange_frontier(sg, exchange, fout)
        exchange.gather_values(dist)
        if sg.frontier_count(fout) == 0:
            break
        it += 1
        if it > cap:
            raise RuntimeError("iteration cap reached")
        sg.frontier_clear(fin)
        fin, fout = fout, fin
    return dist


def dist_cc(dg: DistGraph, exchange: SliceExchange, max_iters: int | None = None):
    """Label propagation over the 1-D partition: all vertices start active
    (advance::vertices); each rank lowers the labels of its owned vertices from the arcs
    of its push block, then the owned label slices and output-frontier slices are all-gathered.
    Returns the full label array (component minimum ids), replicated on every rank."""
    import torch
    sg = dg.sg
    n = dg.n
    dev = torch.device("cuda", torch.cuda.current_device())
    label = torch.arange(n, dtype=torch.int32, device=dev)
    fin, fout = sg.frontier_init(dg.G), sg.frontier_init(dg.G)
    sg.frontier_fill_all(fin)
    cap = max_iters or n + 1
    it = 0
    while True:
        sg.advance(dg.G, fin, fout, sg.SG_FN_CC, dict(label=label))
        _exchange_frontier(sg, exchange, fout)
        exchange.gather_values(label)
        if sg.frontier_count(fout) == 0:
            break
        it += 1
        if it > cap:
            raise RuntimeError("iteration cap reached")
        sg.frontier_clear(fin)
        fin, fout = fout, fin
    return label
