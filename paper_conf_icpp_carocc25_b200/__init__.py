"""Python binding of libsygraph (include/sygraph.h) — argument marshalling only.

Every step of the path runs in the sm_100a kernels of ``csrc/``; this module converts torch
tensors / numpy arrays into pointers and calls the C ABI functions of the same names.  There is
no CPU fallback: if ``lib/libsygraph.so`` is missing, importing the library raises.
PyTorch is used for device memory and streams only.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SYGRAPH_LIB") or os.path.join(_PKG, "lib", "libsygraph.so")

SG_OK, SG_ERR_INVALID, SG_ERR_OOM, SG_ERR_CUDA, SG_ERR_NCCL, SG_ERR_UNSUPPORTED, SG_ERR_STATE = 0, -1, -2, -3, -4, -5, -6
SG_MEM_HOST, SG_MEM_DEVICE = 0, 1
SG_F_BORROW, SG_F_VALIDATE, SG_F_DIRECTED = 1, 2, 4
SG_FN_BFS, SG_FN_SSSP, SG_FN_CC, SG_FN_BC_SIGMA = 0, 1, 2, 3
SG_DIR_AUTO, SG_DIR_PUSH, SG_DIR_PULL = 0, 1, 2
INF32 = 0xFFFFFFFF


class SgError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"sygraph error {code}: {msg}")
        self.code = code


class SgOpts(ctypes.Structure):
    _fields_ = [("stream", ctypes.c_void_p), ("direction", ctypes.c_int), ("alpha", ctypes.c_double),
                ("beta", ctypes.c_double), ("max_iters", ctypes.c_int64), ("heavy_degree", ctypes.c_int32),
                ("small_degree", ctypes.c_int32), ("host_loop", ctypes.c_int32), ("segmented", ctypes.c_int32),
                ("one_layer", ctypes.c_int32), ("coarsening", ctypes.c_int32), ("sssp_delta", ctypes.c_int32),
                ("scsr", ctypes.c_int32), ("owned_only", ctypes.c_int32), ("reserved", ctypes.c_int32 * 1)]


class SgStats(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_int64), ("push_steps", ctypes.c_int64), ("pull_steps", ctypes.c_int64),
                ("arcs_pushed", ctypes.c_int64), ("arcs_pulled", ctypes.c_int64), ("reached", ctypes.c_int64),
                ("device_ms", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class SgBfsState(ctypes.Structure):
    _fields_ = [("level", ctypes.c_void_p), ("visited", ctypes.c_void_p), ("depth", ctypes.c_uint32)]


class SgSsspState(ctypes.Structure):
    _fields_ = [("dist", ctypes.c_void_p)]


class SgCcState(ctypes.Structure):
    _fields_ = [("label", ctypes.c_void_p)]


class SgBcState(ctypes.Structure):
    _fields_ = [("level", ctypes.c_void_p), ("visited", ctypes.c_void_p), ("sigma", ctypes.c_void_p),
                ("exp2_per_level", ctypes.c_void_p), ("depth", ctypes.c_uint32)]


class SgKprof(ctypes.Structure):
    _fields_ = [("ms", ctypes.c_double), ("bytes", ctypes.c_double), ("launches", ctypes.c_int64)]


SG_K_COMPACT, SG_K_STATS, SG_K_PUSH, SG_K_PULL, SG_K_BC, SG_K_SWEEP, SG_K_COUNT = 0, 1, 2, 3, 4, 5, 6
K_NAMES = ["compact", "stats", "advance_push", "advance_pull", "bc", "advance_sweep"]

# every symbol include/sygraph.h declares (checked by tests/test_abi.py)
EXPORTS = ["graph_load_csr", "graph_free", "graph_info", "frontier_init", "frontier_free", "frontier_insert",
           "frontier_fill_all", "frontier_clear", "frontier_count", "frontier_view", "frontier_op",
           "frontier_or_into", "advance", "run_bfs", "run_sssp", "run_cc", "run_bc", "sg_opts_default",
           "sg_last_error", "sg_version", "sg_profile", "sg_profile_read", "sg_launch_count", "frontier_filter",
           "compute_execute", "comm_unique_id", "comm_init", "comm_free", "comm_info", "graph_partition", "sg_bfs_trace", "sg_ctrl_debug", "sg_ablation_bfs"]
SG_PRED_DEGREE_RANGE, SG_PRED_U32_RANGE, SG_PRED_I32_RANGE, SG_PRED_F64_RANGE, SG_PRED_IN_BITMAP = 0, 1, 2, 3, 4
SG_OP_SET_U32, SG_OP_SET_I32, SG_OP_SET_F64, SG_OP_ADD_U32, SG_OP_ADD_F64 = 0, 1, 2, 3, 4

_lib = None


def load():
    """Load libsygraph.so (raises if it was not built: there is no fallback path)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i64, i32, c_int = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_int
    pp = ctypes.POINTER(ctypes.c_void_p)
    sig = {
        "graph_load_csr": (c_int, [i64, i64, vp, vp, vp, c_int, c_int, vp, vp, pp]),
        "graph_partition": (c_int, [vp, ctypes.POINTER(i64), ctypes.POINTER(i64)]),
        "sg_bfs_trace": (c_int, [vp, vp, vp, vp, vp, vp, i32]),
        "sg_ctrl_debug": (c_int, [vp, vp]),
        "sg_ablation_bfs": (c_int, [vp, i32, vp, i32, vp, ctypes.POINTER(SgStats)]),
        "comm_unique_id": (c_int, [ctypes.c_char_p]),
        "comm_init": (c_int, [ctypes.c_char_p, c_int, c_int, c_int, pp]),
        "comm_free": (c_int, [vp]),
        "comm_info": (c_int, [vp, ctypes.POINTER(c_int), ctypes.POINTER(c_int)]),
        "graph_free": (c_int, [vp]),
        "graph_info": (c_int, [vp, vp, vp, vp, vp, vp]),
        "frontier_init": (c_int, [vp, pp]),
        "frontier_free": (c_int, [vp]),
        "frontier_insert": (c_int, [vp, vp, i64, c_int, vp]),
        "frontier_fill_all": (c_int, [vp, vp]),
        "frontier_clear": (c_int, [vp, vp]),
        "frontier_count": (c_int, [vp, ctypes.POINTER(i64), vp]),
        "frontier_view": (c_int, [vp, pp, pp, ctypes.POINTER(i64), ctypes.POINTER(i64)]),
        "frontier_op": (c_int, [vp, vp, c_int, vp]),
        "frontier_or_into": (c_int, [vp, vp, vp]),
        "advance": (c_int, [vp, vp, vp, c_int, vp, vp]),
        "run_bfs": (c_int, [vp, i32, vp, ctypes.POINTER(SgOpts), ctypes.POINTER(SgStats)]),
        "run_sssp": (c_int, [vp, i32, vp, ctypes.POINTER(SgOpts), ctypes.POINTER(SgStats)]),
        "run_cc": (c_int, [vp, vp, ctypes.POINTER(SgOpts), ctypes.POINTER(SgStats)]),
        "run_bc": (c_int, [vp, vp, i32, vp, ctypes.POINTER(SgOpts), ctypes.POINTER(SgStats)]),
        "sg_opts_default": (None, [ctypes.POINTER(SgOpts)]),
        "sg_last_error": (ctypes.c_char_p, []),
        "sg_version": (ctypes.c_char_p, []),
        "sg_profile": (c_int, [vp, c_int]),
        "sg_profile_read": (c_int, [vp, ctypes.POINTER(SgKprof)]),
        "sg_launch_count": (i64, []),
        "frontier_filter": (c_int, [vp, vp, c_int, vp, ctypes.c_double, ctypes.c_double, vp]),
        "compute_execute": (c_int, [vp, c_int, vp, ctypes.c_double, vp]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib


def _check(rc):
    if rc != SG_OK:
        raise SgError(rc, load().sg_last_error().decode())


def _stream_ptr(stream):
    import torch
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _ptr_mem(a):
    """(pointer, SG_MEM_*) of a torch tensor or numpy array (must be contiguous)."""
    if a is None:
        return None, SG_MEM_HOST
    if isinstance(a, np.ndarray):
        assert a.flags.c_contiguous
        return a.ctypes.data, SG_MEM_HOST
    import torch
    assert isinstance(a, torch.Tensor) and a.is_contiguous()
    return a.data_ptr(), (SG_MEM_DEVICE if a.is_cuda else SG_MEM_HOST)


def opts(stream=None, direction=SG_DIR_AUTO, alpha=5.0, beta=48.0, max_iters=0, heavy_degree=0, small_degree=0,
         host_loop=False, segmented=0, one_layer=False, coarsening=0, sssp_delta=0, scsr=0, owned_only=False):
    """segmented: BFS hub tier with the visited slice in shared memory (0 auto, 1 off, 2 always);
    one_layer: ablation without the summary layer; coarsening: words per warp grab (0 auto);
    scsr: BFS heavy push over the destination-segmented arc copy (0 auto, 1 off, 2 always)."""
    o = SgOpts()
    load().sg_opts_default(ctypes.byref(o))
    o.stream = _stream_ptr(stream)
    o.direction, o.alpha, o.beta, o.max_iters = direction, alpha, beta, max_iters
    o.heavy_degree, o.small_degree, o.host_loop = heavy_degree, small_degree, int(host_loop)
    o.segmented, o.one_layer, o.coarsening, o.sssp_delta = segmented, int(one_layer), coarsening, sssp_delta
    o.scsr = scsr
    o.owned_only = int(owned_only)
    return o


# ------------------------------------------------------------------------------ graph
class Graph:
    def __init__(self, handle, n, nnz, has_weights):
        self.handle, self.n, self.nnz, self.has_weights = handle, n, nnz, has_weights

    def free(self):
        if self.handle:
            graph_free(self)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def graph_load_csr(row_ptr, col_idx, weights=None, validate=False, stream=None, borrow=False, comm=None,
                   directed=False) -> Graph:
    """row_ptr int64[n+1], col_idx int32[nnz], weights uint8[nnz] (numpy/host tensors or CUDA tensors).
    borrow (CUDA tensors only): keep the tensors' memory instead of copying (SG_F_BORROW); the
    returned Graph holds references to them.  comm (a Comm): collective partitioned load — this
    rank keeps its owned destination range (graph_partition) and run_* become collective."""
    rp, m1 = _ptr_mem(row_ptr)
    ci, m2 = _ptr_mem(col_idx)
    w, m3 = _ptr_mem(weights)
    n = int(row_ptr.shape[0]) - 1
    nnz = int(col_idx.shape[0])
    mems = {m1, m2} | ({m3} if weights is not None else set())
    if len(mems) != 1:
        raise ValueError("row_ptr, col_idx and weights must all be host or all be device arrays")
    h = ctypes.c_void_p()
    flags = (SG_F_VALIDATE if validate else 0) | (SG_F_BORROW if borrow else 0) | (SG_F_DIRECTED if directed else 0)
    _check(load().graph_load_csr(n, nnz, rp, ci if nnz else None, w, m1, flags, _stream_ptr(stream),
                                 comm.handle if comm is not None else None, ctypes.byref(h)))
    G = Graph(h.value, n, nnz, weights is not None)
    G.comm = comm
    if borrow:
        G._borrowed = (row_ptr, col_idx, weights)
    return G


def graph_partition(g: Graph):
    """(lo, hi): the destination range this rank owns ([0, n) for a single-GPU graph)."""
    lo, hi = ctypes.c_int64(), ctypes.c_int64()
    _check(load().graph_partition(g.handle, ctypes.byref(lo), ctypes.byref(hi)))
    return lo.value, hi.value


# ------------------------------------------------------------------------ communicator
class Comm:
    """Ranks of a 1-D destination partition (include/sygraph.h comm_*); free after its graphs."""

    def __init__(self, handle, nranks, rank):
        self.handle, self.nranks, self.rank = handle, nranks, rank

    def free(self):
        if self.handle:
            _check(load().comm_free(self.handle))
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def comm_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(load().comm_unique_id(buf))
    return buf.raw


def comm_init(uid: bytes, nranks: int, rank: int, device: int = 0) -> Comm:
    h = ctypes.c_void_p()
    _check(load().comm_init(ctypes.create_string_buffer(uid, 128), int(nranks), int(rank), int(device),
                            ctypes.byref(h)))
    return Comm(h.value, nranks, rank)


def comm_from_torch(group=None, device: int | None = None) -> Comm:
    """Bootstrap a Comm over an initialised torch.distributed process group (gloo or nccl): rank 0
    creates the id, torch broadcasts it (plumbing only)."""
    import torch
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    obj = [comm_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    if device is None:
        device = torch.cuda.current_device() if torch.cuda.is_available() else 0
    return comm_init(obj[0], world, rank, device)


def graph_info(g: Graph):
    """(n, nnz, row_ptr, col_idx, weights) — the device pointers the graph reads (ints; 0 = none)."""
    n, nnz = ctypes.c_int64(), ctypes.c_int64()
    rp, ci, w = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
    _check(load().graph_info(g.handle, ctypes.byref(n), ctypes.byref(nnz), ctypes.byref(rp), ctypes.byref(ci),
                             ctypes.byref(w)))
    return n.value, nnz.value, rp.value or 0, ci.value or 0, w.value or 0


def graph_free(g: Graph):
    _check(load().graph_free(g.handle))
    g.handle = None


# --------------------------------------------------------------------------- frontier
class Frontier:
    def __init__(self, handle, g):
        self.handle, self.g = handle, g

    def free(self):
        if self.handle:
            frontier_free(self)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def frontier_init(g: Graph) -> Frontier:
    h = ctypes.c_void_p()
    _check(load().frontier_init(g.handle, ctypes.byref(h)))
    return Frontier(h.value, g)


def frontier_free(f: Frontier):
    _check(load().frontier_free(f.handle))
    f.handle = None


def frontier_insert(f: Frontier, vertices, stream=None):
    if isinstance(vertices, (list, tuple)):
        vertices = np.asarray(vertices, dtype=np.int32)
    p, mem = _ptr_mem(vertices)
    _check(load().frontier_insert(f.handle, p, int(vertices.shape[0]), mem, _stream_ptr(stream)))


def frontier_fill_all(f: Frontier, stream=None):
    _check(load().frontier_fill_all(f.handle, _stream_ptr(stream)))


def frontier_clear(f: Frontier, stream=None):
    _check(load().frontier_clear(f.handle, _stream_ptr(stream)))


def frontier_count(f: Frontier, stream=None) -> int:
    out = ctypes.c_int64()
    _check(load().frontier_count(f.handle, ctypes.byref(out), _stream_ptr(stream)))
    return out.value


class _CudaArray:
    def __init__(self, ptr, n, typestr):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}


def frontier_view(f: Frontier):
    """(bits, summ) as zero-copy uint64 CUDA tensors (layer 1, layer 2)."""
    import torch
    b, s = ctypes.c_void_p(), ctypes.c_void_p()
    n1, n2 = ctypes.c_int64(), ctypes.c_int64()
    _check(load().frontier_view(f.handle, ctypes.byref(b), ctypes.byref(s), ctypes.byref(n1), ctypes.byref(n2)))
    bits = torch.as_tensor(_CudaArray(b.value, n1.value, "<u8"), device="cuda")
    summ = torch.as_tensor(_CudaArray(s.value, n2.value, "<u8"), device="cuda")
    return bits, summ


def frontier_op(dst: Frontier, src: Frontier, op: int, stream=None):
    _check(load().frontier_op(dst.handle, src.handle, op, _stream_ptr(stream)))


def frontier_filter(fin: Frontier, fout: Frontier | None, pred: int, array=None, a: float = 0.0, b: float = 0.0,
                    stream=None):
    """filter::inplace (fout None) / filter::external (Table 2) with a SG_PRED_* predicate."""
    _check(load().frontier_filter(fin.handle, fout.handle if fout is not None else None, pred,
                                  array.data_ptr() if array is not None else None, float(a), float(b),
                                  _stream_ptr(stream)))


def compute_execute(f: Frontier, op: int, array, value: float, stream=None):
    """compute::execute (Table 2): SG_OP_* applied to array[v] for every active v."""
    _check(load().compute_execute(f.handle, op, array.data_ptr(), float(value), _stream_ptr(stream)))


def frontier_or_into(f: Frontier, dst, stream=None):
    _check(load().frontier_or_into(f.handle, dst.data_ptr(), _stream_ptr(stream)))


# ---------------------------------------------------------------------------- advance
def advance(g: Graph, fin: Frontier, fout: Frontier | None, functor: int, state: dict, stream=None):
    """One push advance superstep (stream ordered).  ``state`` holds the functor's tensors:
    BFS {level, visited, depth}; SSSP {dist}; CC {label}; BC {level, visited, sigma, exp2_per_level,
    depth}."""
    if functor == SG_FN_BFS:
        st = SgBfsState(state["level"].data_ptr(), state["visited"].data_ptr(), int(state["depth"]))
    elif functor == SG_FN_SSSP:
        st = SgSsspState(state["dist"].data_ptr())
    elif functor == SG_FN_CC:
        st = SgCcState(state["label"].data_ptr())
    elif functor == SG_FN_BC_SIGMA:
        e = state.get("exp2_per_level")
        st = SgBcState(state["level"].data_ptr(), state["visited"].data_ptr(), state["sigma"].data_ptr(),
                       e.data_ptr() if e is not None else None, int(state["depth"]))
    else:
        raise ValueError(functor)
    _check(load().advance(g.handle, fin.handle, fout.handle if fout is not None else None, functor,
                          ctypes.byref(st), _stream_ptr(stream)))


# ------------------------------------------------------------------------- algorithms
def _out_tensor(n, dtype, out):
    import torch
    if out is None:
        out = torch.empty(n, dtype=dtype, device="cuda")
    assert out.is_cuda and out.dtype == dtype and out.numel() == n and out.is_contiguous()
    return out


def run_bfs(g: Graph, src: int, level=None, o: SgOpts | None = None, **kw):
    """BFS levels (uint32 as torch.int32 storage reinterpreted; INF32 = unreached) and stats."""
    import torch
    level = _out_tensor(g.n, torch.int32, level)
    o = o or opts(**kw)
    st = SgStats()
    _check(load().run_bfs(g.handle, int(src), level.data_ptr(), ctypes.byref(o), ctypes.byref(st)))
    return level, st


def run_sssp(g: Graph, src: int, dist=None, o: SgOpts | None = None, **kw):
    import torch
    dist = _out_tensor(g.n, torch.int32, dist)
    o = o or opts(**kw)
    st = SgStats()
    _check(load().run_sssp(g.handle, int(src), dist.data_ptr(), ctypes.byref(o), ctypes.byref(st)))
    return dist, st


def run_cc(g: Graph, label=None, o: SgOpts | None = None, **kw):
    import torch
    label = _out_tensor(g.n, torch.int32, label)
    o = o or opts(**kw)
    st = SgStats()
    _check(load().run_cc(g.handle, label.data_ptr(), ctypes.byref(o), ctypes.byref(st)))
    return label, st


def run_bc(g: Graph, sources, bc=None, o: SgOpts | None = None, **kw):
    import torch
    src = np.ascontiguousarray(np.asarray(sources, dtype=np.int32))
    bc = _out_tensor(g.n, torch.float64, bc)
    o = o or opts(**kw)
    st = SgStats()
    _check(load().run_bc(g.handle, src.ctypes.data if len(src) else None, len(src), bc.data_ptr(),
                         ctypes.byref(o), ctypes.byref(st)))
    return bc, st


def as_u32(t) -> np.ndarray:
    """Device int32 tensor holding uint32 values -> host numpy uint32."""
    return t.cpu().numpy().view(np.uint32)


def profile(g: Graph, enable: bool = True):
    _check(load().sg_profile(g.handle, int(enable)))


def profile_read(g: Graph) -> dict:
    arr = (SgKprof * SG_K_COUNT)()
    _check(load().sg_profile_read(g.handle, arr))
    return {K_NAMES[i]: dict(ms=arr[i].ms, bytes=arr[i].bytes, launches=arr[i].launches) for i in range(SG_K_COUNT)}


TRACE_KINDS = {0: "stop", 1: "push", 2: "pull", 3: "sweep", 4: "sparse"}


def bfs_trace(g: Graph) -> list:
    """Per-superstep trace of the last device-driven run_bfs on g (sg_bfs_trace): dicts with the
    superstep's kind, input frontier (words, n_f, m_f) and device time in us (decision to decision)."""
    cap = 48
    t = (ctypes.c_int64 * cap)()
    k = (ctypes.c_int32 * cap)()
    c, nf, mf = (ctypes.c_int64 * cap)(), (ctypes.c_int64 * cap)(), (ctypes.c_int64 * cap)()
    n = load().sg_bfs_trace(g.handle, t, k, c, nf, mf, cap)
    if n < 0:
        _check(n)
    out = []
    for i in range(n - 1):
        out.append({"step": i, "kind": TRACE_KINDS.get(k[i], k[i]), "words": c[i], "nf": nf[i], "mf": mf[i],
                    "us": (t[i + 1] - t[i]) / 1e3})
    return out


def ablation_bfs(g: Graph, src: int, word_bits: int, level=None, stream=None):
    """Word-width ablation BFS (sg_ablation_bfs): push-only 2LB with 32- or 64-bit words."""
    import torch
    level = _out_tensor(g.n, torch.int32, level)
    st = SgStats()
    _check(load().sg_ablation_bfs(g.handle, int(src), level.data_ptr(), int(word_bits), _stream_ptr(stream),
                                  ctypes.byref(st)))
    return level, st


def ctrl_debug(g: Graph) -> list:
    out = (ctypes.c_int64 * 16)()
    _check(load().sg_ctrl_debug(g.handle, out))
    return list(out)


def launch_count() -> int:
    return int(load().sg_launch_count())


def version() -> str:
    return load().sg_version().decode()
