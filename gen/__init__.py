"""Seeded synthetic graph inputs shared by the oracle side and the CUDA side.

Input construction only: this module
draws graphs, weights and source lists.  It contains none of the method's arithmetic
(no traversal, relaxation, labels or bitmap frontier), so sharing it does not couple
the oracle to the CUDA path.  Heavy lifting is in ``gen.c`` (OpenMP, counter-based RNG,
bit-reproducible regardless of thread count).
"""
from __future__ import annotations

import ctypes
import hashlib
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsggen.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile gen.c into libsggen.so (gcc, OpenMP)."""
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-fPIC", "-shared",
                               "-fvisibility=hidden", "-o", _LIB_PATH + ".tmp", src])
        os.replace(_LIB_PATH + ".tmp", _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        vp, i64, u64, dbl, c_int = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_int
        lib.sgg_rmat.restype = vp
        lib.sgg_rmat.argtypes = [c_int, i64, dbl, dbl, dbl, u64, c_int]
        lib.sgg_gnm.restype = vp
        lib.sgg_gnm.argtypes = [i64, i64, u64]
        lib.sgg_lattice.restype = vp
        lib.sgg_lattice.argtypes = [i64, i64, dbl, u64]
        lib.sgg_from_edges.restype = vp
        lib.sgg_from_edges.argtypes = [i64, i64, vp, vp]
        lib.sgg_n.restype = i64
        lib.sgg_n.argtypes = [vp]
        lib.sgg_nnz.restype = i64
        lib.sgg_nnz.argtypes = [vp]
        lib.sgg_fill.restype = c_int
        lib.sgg_fill.argtypes = [vp, vp, vp]
        lib.sgg_free.restype = None
        lib.sgg_free.argtypes = [vp]
        lib.sgg_weights.restype = None
        lib.sgg_weights.argtypes = [i64, vp, vp, u64, ctypes.c_uint32, vp]
        lib.sgg_sources.restype = i64
        lib.sgg_sources.argtypes = [i64, vp, u64, u64, i64, vp, vp]
        lib.sgg_rnd.restype = u64
        lib.sgg_rnd.argtypes = [u64, u64, u64]
        _lib = lib
    return _lib


@dataclass
class CSR:
    """Symmetric simple graph in CSR form: rows ascending, no self-loops, no multi-edges."""
    n: int
    row_ptr: np.ndarray          # int64[n+1]
    col_idx: np.ndarray          # int32[nnz]
    name: str = ""
    weights: np.ndarray | None = None   # uint8[nnz] (SSSP), symmetric
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr)

    def sha256(self) -> str:
        h = hashlib.sha256()
        h.update(np.int64(self.n).tobytes())
        h.update(np.ascontiguousarray(self.row_ptr).tobytes())
        h.update(np.ascontiguousarray(self.col_idx).tobytes())
        if self.weights is not None:
            h.update(np.ascontiguousarray(self.weights).tobytes())
        return h.hexdigest()


def _materialise(handle, name, alloc=None) -> CSR:
    lib = _load()
    if not handle:
        raise MemoryError("generator failed (out of host memory?)")
    try:
        n = lib.sgg_n(handle)
        nnz = lib.sgg_nnz(handle)
        if alloc is None:
            row_ptr = np.empty(n + 1, dtype=np.int64)
            col_idx = np.empty(max(nnz, 0), dtype=np.int32)
        else:
            row_ptr, col_idx = alloc(n, nnz)
        rc = lib.sgg_fill(handle, row_ptr.ctypes.data, col_idx.ctypes.data if nnz else None)
        if rc != 0:
            raise RuntimeError("sgg_fill failed")
    finally:
        lib.sgg_free(handle)
    return CSR(n=int(n), row_ptr=row_ptr, col_idx=col_idx, name=name)


def rmat(scale: int, edge_factor: int, seed: int = 1, permute: bool = False,
         A: float = 0.57, B: float = 0.19, C: float = 0.19, alloc=None) -> CSR:
    """Graph500 R-MAT/Kronecker (reading C17); ``edge_factor`` counts generated undirected edges."""
    h = _load().sgg_rmat(scale, edge_factor, A, B, C, seed, int(permute))
    g = _materialise(h, f"rmat{scale}_ef{edge_factor}{'_perm' if permute else ''}_s{seed}", alloc)
    g.meta.update(kind="rmat", scale=scale, edge_factor=edge_factor, seed=seed, permute=permute)
    return g


def gnm(n: int, m: int, seed: int = 1, alloc=None) -> CSR:
    """Uniform G(n, m): m uniform endpoint pairs, self-loops and duplicates dropped."""
    h = _load().sgg_gnm(n, m, seed)
    g = _materialise(h, f"gnm_n{n}_m{m}_s{seed}", alloc)
    g.meta.update(kind="gnm", m=m, seed=seed)
    return g


def lattice(R: int, C: int, p: float = 1.0, seed: int = 1, alloc=None) -> CSR:
    """Bond-percolated R x C lattice (row-major ids); p = 1 gives the full grid."""
    h = _load().sgg_lattice(R, C, p, seed)
    g = _materialise(h, f"lattice_{R}x{C}_p{p}_s{seed}", alloc)
    g.meta.update(kind="lattice", R=R, C=C, p=p, seed=seed)
    return g


def from_edges(n: int, u, v, name: str = "edges") -> CSR:
    u = np.ascontiguousarray(np.asarray(u, dtype=np.int64).ravel())
    v = np.ascontiguousarray(np.asarray(v, dtype=np.int64).ravel())
    assert u.shape == v.shape
    h = _load().sgg_from_edges(n, len(u), u.ctypes.data if len(u) else None, v.ctypes.data if len(v) else None)
    return _materialise(h, name)


# ---- closed-form families (pins) ----
def path(n: int) -> CSR:
    i = np.arange(n - 1)
    return from_edges(n, i, i + 1, f"path{n}")


def cycle(n: int) -> CSR:
    i = np.arange(n)
    return from_edges(n, i, (i + 1) % n, f"cycle{n}")


def star(n: int) -> CSR:
    i = np.arange(1, n)
    return from_edges(n, np.zeros_like(i), i, f"star{n}")


def complete(n: int) -> CSR:
    u, v = np.triu_indices(n, 1)
    return from_edges(n, u, v, f"K{n}")


def grid(R: int, C: int) -> CSR:
    return lattice(R, C, 1.0, 1)


def hypercube(d: int) -> CSR:
    n = 1 << d
    v = np.arange(n, dtype=np.int64)
    us, vs = [], []
    for b in range(d):
        m = (v >> b) & 1 == 0
        us.append(v[m])
        vs.append(v[m] | (1 << b))
    return from_edges(n, np.concatenate(us), np.concatenate(vs), f"Q{d}")


def empty_graph(n: int) -> CSR:
    return from_edges(n, [], [], f"empty{n}")


def random_simple(n: int, p: float, seed: int) -> CSR:
    """Small Erdos-Renyi G(n, p) for brute-force pins (numpy RNG, test sizes only)."""
    rng = np.random.default_rng(seed)
    u, v = np.triu_indices(n, 1)
    keep = rng.random(len(u)) < p
    return from_edges(n, u[keep], v[keep], f"gnp{n}_{p}_{seed}")


def with_weights(g: CSR, seed: int = 1, wmax: int = 64) -> CSR:
    """Attach symmetric weights w(u,v) = 1 + rnd(seed, 3, min*n+max) mod wmax (reading C11)."""
    w = np.empty(g.nnz, dtype=np.uint8)
    if g.nnz:
        _load().sgg_weights(g.n, g.row_ptr.ctypes.data, g.col_idx.ctypes.data, seed, wmax, w.ctypes.data)
    g.weights = w
    return g


def _mix64(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser, vectorised (uint64, wrapping)."""
    z = z.astype(np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def orient(g: CSR, seed: int = 1, stream: int = 7) -> CSR:
    """A directed graph from a symmetric one (SURVEY f4 test input): edge {u < v} keeps the arc
    u -> v iff bit 0 of mix(mix(seed ^ stream << 56) + u*n + v) is set and v -> u iff bit 1 is
    (so ~1/4 of the edges keep both arcs, ~1/4 neither).  Rows stay sorted; weights follow."""
    rows = np.repeat(np.arange(g.n, dtype=np.int64), g.degrees())
    cols = g.col_idx.astype(np.int64)
    lo, hi = np.minimum(rows, cols), np.maximum(rows, cols)
    with np.errstate(over="ignore"):
        base = _mix64(np.array([np.uint64(seed) ^ (np.uint64(stream) << np.uint64(56))], dtype=np.uint64))[0]
        h = _mix64(base + (lo * g.n + hi).astype(np.uint64))
    bit = np.where(rows < cols, h & np.uint64(1), (h >> np.uint64(1)) & np.uint64(1)).astype(bool)
    counts = np.bincount(rows[bit], minlength=g.n)
    rp = np.zeros(g.n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    out = CSR(n=g.n, row_ptr=rp, col_idx=np.ascontiguousarray(g.col_idx[bit]), name=g.name + "-directed")
    if g.weights is not None:
        out.weights = np.ascontiguousarray(g.weights[bit])
    return out


def sources(g: CSR, k: int, seed: int = 1, stream: int = 5, eligible: np.ndarray | None = None) -> np.ndarray:
    """First k distinct rnd(seed, stream, i) mod n with degree > 0 (reading C15), restricted to
    eligible[v] != 0 when a mask is given."""
    out = np.empty(k, dtype=np.int32)
    if eligible is not None:
        eligible = np.ascontiguousarray(eligible, dtype=np.uint8)
        assert eligible.shape == (g.n,)
    got = _load().sgg_sources(g.n, g.row_ptr.ctypes.data, seed, stream, k, out.ctypes.data,
                              eligible.ctypes.data if eligible is not None else None)
    return out[:got].copy()


def largest_component_mask(g: CSR) -> np.ndarray:
    """uint8[n]: 1 on the vertices of the largest connected component (ties: the one holding the
    smallest vertex id).  Source selection only (reading C15); computed with scipy's
    connected_components, a library routine shared by neither the oracle nor the CUDA path."""
    import scipy.sparse as sp
    from scipy.sparse.csgraph import connected_components
    A = sp.csr_matrix((np.ones(g.nnz, dtype=np.int8), g.col_idx, g.row_ptr), shape=(g.n, g.n))
    _, lab = connected_components(A, directed=False)
    cnt = np.bincount(lab)
    big = int(np.argmax(cnt))          # argmax returns the first maximum: smallest label = smallest id
    return (lab == big).astype(np.uint8)


def rnd(seed: int, stream: int, i: int) -> int:
    return int(_load().sgg_rnd(seed, stream, i))


# ---- the BASELINE.json configurations (sizes per SURVEY.md §8(d)) ----
CONFIGS = {
    1: dict(workload="bfs", graph=("rmat", dict(scale=10, edge_factor=16, permute=False)), sources=[0]),
    2: dict(workload="sssp", graph=("rmat", dict(scale=20, edge_factor=16, permute=False)), sources=[0],
            weights=64),
    3: dict(workload="cc", graph=("gnm", dict(n=21_000_000, m=265_000_000))),
    4: dict(workload="bfs_do", graph=("rmat", dict(scale=24, edge_factor=32, permute=True)), n_sources=64,
            source_stream=5),
    5: dict(workload="bc", graph=("lattice", dict(R=4000, C=6000, p=0.6)), n_sources=64, source_stream=6,
            largest_component=True),   # reading C15
}


def make_config_graph(cfg: int, seed: int = 1, alloc=None) -> CSR:
    c = CONFIGS[cfg]
    kind, kw = c["graph"]
    fn = {"rmat": rmat, "gnm": gnm, "lattice": lattice}[kind]
    g = fn(seed=seed, alloc=alloc, **kw)
    if c.get("weights"):
        with_weights(g, seed=seed, wmax=c["weights"])
    return g


def config_sources(cfg: int, g: CSR, seed: int = 1) -> np.ndarray:
    c = CONFIGS[cfg]
    if "sources" in c:
        return np.asarray(c["sources"], dtype=np.int32)
    eligible = largest_component_mask(g) if c.get("largest_component") else None
    return sources(g, c["n_sources"], seed=seed, stream=c["source_stream"], eligible=eligible)
