"""1-D destination partitioning across GPUs (§6 "static graph
partitioning ... each GPU handles a local subgraph") — Python side.

The product path is native: ``graph_load_csr(..., comm=Comm)`` partitions the graph in the
library (csrc/partition.cu) and ``run_bfs / run_sssp / run_cc`` exchange the owned slices inside
their output kernels over peer memory (csrc/xchg.cuh).  This module holds

* ``partition_ranges`` / ``push_block`` / ``Layout``: the same partition rule written in numpy,
  used by the tests to check the library's bounds and to document the layout:
  rank r owns vertices [lo_r, hi_r), aligned to 4,096 vertices (one layer-2 word, so every rank
  owns whole layer-1 *and* layer-2 words) and balanced by arcs (the graph is symmetric, so
  out-degree = in-degree = the arcs a rank receives);
* ``dist_bc``: BC's multi-GPU form, which is not a partition: the sources are independent
  problems, sharded over ranks that each hold a full replica, with one all-reduce (sum) of the
  scores at the end.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

ALIGN = 4096          # vertices per layer-2 word


def partition_ranges(row_ptr: np.ndarray, parts: int, align: int = ALIGN) -> list[tuple[int, int]]:
    """Contiguous, `align`-aligned vertex ranges with ~equal arc counts (last range ends at n).
    Bound r = the first vertex whose row starts at or after nnz*r/parts, rounded to the nearest
    multiple of `align`, kept monotone and <= n (csrc/capi.cu partition_graph: the same rule)."""
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


def dist_bc(G, sources, group=None, **opts):
    """Brandes BC over ranks that each hold a full replica G (not a partitioned graph): rank r
    takes sources[r::world], runs run_bc locally, and the fp64 scores are summed over ranks
    (torch.distributed all-reduce; plumbing).  Returns the full score tensor on every rank."""
    import torch.distributed as dist
    import paper_conf_icpp_carocc25_b200 as sg
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    mine = np.asarray(sources, dtype=np.int32)[rank::world]
    bc, st = sg.run_bc(G, mine, **opts)
    dist.all_reduce(bc, op=dist.ReduceOp.SUM, group=group)
    return bc, st
