"""Parity oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_icpp_carocc25_b200``) never imports it and shares no code with it.

Whole-algorithm results come from ``oracle.c`` (plain single-threaded C: queue BFS,
binary-heap Dijkstra, union-find, Brandes in long double).  The per-superstep set
semantics of one advance and the Two-Layer-Bitmap invariants are written here in numpy,
each function citing the passage it follows.  Pins: tests/test_oracle_*.py (brute force,
closed forms, invariants).  Parity status of every function: pinned.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None
INF32 = np.uint32(0xFFFFFFFF)


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-fvisibility=hidden", "-o",
                               _LIB_PATH + ".tmp", src, "-lm"])
        os.replace(_LIB_PATH + ".tmp", _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
        lib.oracle_bfs.restype = i64
        lib.oracle_bfs.argtypes = [i64, vp, vp, i32, vp]
        lib.oracle_sssp.restype = i64
        lib.oracle_sssp.argtypes = [i64, vp, vp, vp, i32, vp]
        lib.oracle_cc.restype = i64
        lib.oracle_cc.argtypes = [i64, vp, vp, vp]
        lib.oracle_bc.restype = ctypes.c_int
        lib.oracle_bc.argtypes = [i64, vp, vp, vp, i64, vp]
        lib.oracle_bc_single.restype = ctypes.c_int
        lib.oracle_bc_single.argtypes = [i64, vp, vp, i32, vp, vp, vp, vp]
        _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data if a is not None and a.size else None


def _csr(g):
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
    return rp, ci


def bfs(g, src: int) -> np.ndarray:
    """Hop levels from ``src`` (Listing 1); UINT32_MAX = unreached (C6)."""
    rp, ci = _csr(g)
    level = np.empty(g.n, dtype=np.uint32)
    _load().oracle_bfs(g.n, _ptr(rp), _ptr(ci), int(src), _ptr(level))
    return level


def sssp(g, src: int, weights=None) -> np.ndarray:
    """Shortest-path distances (Bellman-Ford fixed point) by Dijkstra."""
    rp, ci = _csr(g)
    w = np.ascontiguousarray(g.weights if weights is None else weights, dtype=np.uint8)
    dist = np.empty(g.n, dtype=np.uint32)
    _load().oracle_sssp(g.n, _ptr(rp), _ptr(ci), _ptr(w), int(src), _ptr(dist))
    return dist


def cc(g) -> np.ndarray:
    """Min-id component labels (label-propagation fixed point) by union-find."""
    rp, ci = _csr(g)
    label = np.empty(g.n, dtype=np.int32)
    _load().oracle_cc(g.n, _ptr(rp), _ptr(ci), _ptr(label))
    return label


def bc(g, sources) -> np.ndarray:
    """Sum over sources of Brandes dependencies delta_s(v) (reading C14)."""
    rp, ci = _csr(g)
    src = np.ascontiguousarray(np.asarray(sources, dtype=np.int32))
    out = np.empty(g.n, dtype=np.float64)
    rc = _load().oracle_bc(g.n, _ptr(rp), _ptr(ci), _ptr(src), len(src), _ptr(out))
    if rc != 0:
        raise MemoryError("oracle_bc allocation failed")
    return out


def bc_single(g, s: int):
    """(level, sigma, log2 sigma, delta) for one Brandes source (forward + backward)."""
    rp, ci = _csr(g)
    n = g.n
    level = np.empty(n, dtype=np.uint32)
    sigma = np.empty(n, dtype=np.float64)
    lsig = np.empty(n, dtype=np.float64)
    delta = np.empty(n, dtype=np.float64)
    _load().oracle_bc_single(n, _ptr(rp), _ptr(ci), int(s), _ptr(level), _ptr(sigma), _ptr(lsig), _ptr(delta))
    return level, sigma, lsig, delta


# ----------------------------------------------------------------------------------
# One superstep (numpy; plain set definitions)
# ----------------------------------------------------------------------------------
def neighbours_of_set(g, active: np.ndarray) -> np.ndarray:
    """Boolean mask of vertices adjacent to some vertex of ``active`` (bool[n])."""
    deg = np.diff(g.row_ptr)
    src = np.repeat(np.arange(g.n), deg)
    hit = np.zeros(g.n, dtype=bool)
    sel = active[src]
    hit[g.col_idx[sel]] = True
    return hit


def bfs_advance_step(g, frontier: np.ndarray, visited: np.ndarray) -> np.ndarray:
    """advance::frontier with the BFS functor (Table 2; Listing 1 l.9-13):
    out = {v : exists u in frontier, (u,v) in E, v not visited}.  Bool masks in, bool out."""
    return neighbours_of_set(g, frontier) & ~visited


def jacobi_relax_step(g, frontier: np.ndarray, value: np.ndarray, weights=None) -> np.ndarray:
    """Jacobi bound for one SSSP/CC advance (reading C12): new[v] = min(value[v],
    min over active u of value[u] + w(u,v)) (w = 0 for CC label propagation)."""
    deg = np.diff(g.row_ptr)
    src = np.repeat(np.arange(g.n), deg)
    sel = frontier[src]
    val = value.astype(np.int64)
    cand = val[src[sel]] + (weights[sel].astype(np.int64) if weights is not None else 0)
    new = val.copy()
    np.minimum.at(new, g.col_idx[sel], cand)
    return new


# ----------------------------------------------------------------------------------
# Two-Layer Bitmap layout (PAPER.md:211-217 §4.1, :253 §4.3; readings C1-C3)
# ----------------------------------------------------------------------------------
def bitmap_words(mask: np.ndarray) -> np.ndarray:
    """Layer 1: word v>>6, bit v&63 (LSB first), ceil(n/64) uint64 words."""
    n = len(mask)
    nw = (n + 63) // 64
    words = np.zeros(nw, dtype=np.uint64)
    idx = np.nonzero(mask)[0]
    for w in np.unique(idx >> 6):
        sel = idx[(idx >> 6) == w]
        acc = 0
        for v in sel:
            acc |= 1 << int(v & 63)
        words[w] = np.uint64(acc)
    return words


def summary_words(words: np.ndarray) -> np.ndarray:
    """Layer 2: bit w of summary word w>>6 set iff layer-1 word w != 0."""
    nw = len(words)
    ns = (nw + 63) // 64
    summ = np.zeros(ns, dtype=np.uint64)
    for w in np.nonzero(words)[0]:
        summ[w >> 6] |= np.uint64(1 << int(w & 63))
    return summ


def words_to_mask(words: np.ndarray, n: int) -> np.ndarray:
    bits = np.unpackbits(words.astype("<u8").view(np.uint8), bitorder="little")
    return bits[:n].astype(bool)
