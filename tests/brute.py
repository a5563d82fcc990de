"""Brute-force and closed-form references used to PIN the oracle (independent methods).

None of these follow the oracle's algorithms: BFS levels come from boolean matrix powers,
SSSP from Floyd-Warshall, CC from transitive closure, BC from the pair-dependency
definition evaluated with exact rationals over all-pairs distances (pins).
"""
from __future__ import annotations

import itertools
from fractions import Fraction
from math import comb, factorial

import numpy as np

INF = 0xFFFFFFFF


def adjacency(g) -> np.ndarray:
    A = np.zeros((g.n, g.n), dtype=bool)
    deg = np.diff(g.row_ptr)
    src = np.repeat(np.arange(g.n), deg)
    A[src, g.col_idx] = True
    return A


def weight_matrix(g) -> np.ndarray:
    W = np.full((g.n, g.n), np.inf)
    deg = np.diff(g.row_ptr)
    src = np.repeat(np.arange(g.n), deg)
    W[src, g.col_idx] = g.weights.astype(np.float64)
    return W


def bfs_levels_matpow(g, s: int) -> np.ndarray:
    """level(v) = min k such that (A^k)[s][v] != 0 (boolean powers)."""
    A = adjacency(g).astype(np.int64)
    n = g.n
    level = np.full(n, INF, dtype=np.uint64)
    reach = np.zeros(n, dtype=bool)
    reach[s] = True
    level[s] = 0
    cur = np.zeros(n, dtype=np.int64)
    cur[s] = 1
    for k in range(1, n):          # every hop distance is <= n-1
        cur = (cur @ A > 0).astype(np.int64)   # vertices ending a walk of length exactly k
        new = (cur > 0) & ~reach
        level[new] = k
        reach |= cur > 0
    return level.astype(np.uint32)


def floyd_warshall(g) -> np.ndarray:
    D = weight_matrix(g)
    np.fill_diagonal(D, 0.0)
    for k in range(g.n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    return D


def hop_apsp(g) -> np.ndarray:
    A = adjacency(g)
    D = np.where(A, 1.0, np.inf)
    np.fill_diagonal(D, 0.0)
    for k in range(g.n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    return D


def closure_min_labels(g) -> np.ndarray:
    """Warshall transitive closure, then label = min reachable id (including itself)."""
    R = adjacency(g) | np.eye(g.n, dtype=bool)
    for k in range(g.n):
        R = R | (R[:, k:k + 1] & R[k:k + 1, :])
    return np.array([int(np.nonzero(R[v])[0].min()) for v in range(g.n)], dtype=np.int32)


def bc_pair_dependency(g, sources) -> list[Fraction]:
    """bc(v) = sum_{s in S} sum_{t != s, v} [D(s,v)+D(v,t) = D(s,t)] sigma_sv sigma_vt / sigma_st,
    sigma from DP over hop distances, exact rationals (definition, not Brandes' recursion)."""
    n = g.n
    D = hop_apsp(g)
    A = adjacency(g)
    # sigma[s][t]: number of shortest s-t paths, by DP in increasing distance
    sigma = [[0] * n for _ in range(n)]
    for s in range(n):
        order = sorted((t for t in range(n) if np.isfinite(D[s, t])), key=lambda t: D[s, t])
        sigma[s][s] = 1
        for t in order:
            if t == s:
                continue
            sigma[s][t] = sum(sigma[s][u] for u in range(n) if A[u, t] and D[s, u] + 1 == D[s, t])
    bc = [Fraction(0)] * n
    for s in sources:
        for v in range(n):
            if v == s or not np.isfinite(D[s, v]):
                continue
            acc = Fraction(0)
            for t in range(n):
                if t == s or t == v or not np.isfinite(D[s, t]) or not np.isfinite(D[v, t]):
                    continue
                if D[s, v] + D[v, t] == D[s, t]:
                    acc += Fraction(sigma[s][v] * sigma[v][t], sigma[s][t])
            bc[v] += acc
    return bc


def hypercube_delta(d: int, k: int) -> Fraction:
    """Single-source dependency on Q_d of a vertex at distance k: sum_j C(d-k,j) k! j!/(k+j)!."""
    return sum((Fraction(comb(d - k, j) * factorial(k) * factorial(j), factorial(k + j))
                for j in range(1, d - k + 1)), Fraction(0))


def all_graphs(n: int):
    """Every labelled simple graph on n vertices as an edge list."""
    pairs = list(itertools.combinations(range(n), 2))
    for mask in range(1 << len(pairs)):
        yield [p for i, p in enumerate(pairs) if mask >> i & 1]
