"""The 1-D destination partition end to end on the GPU: world = 2 or 3 processes (ranks) share
this box's one B200, each with its own CUDA context, a communicator (comm_unique_id / comm_init)
and its partition of the graph (graph_load_csr(..., comm)).  Every superstep runs the real
kernels and the real exchange: the output kernels store each rank's owned slice into its peers'
replicas through CUDA IPC peer memory and meet at the in-kernel superstep barrier (xchg.cuh) —
the same code path as one rank per GPU over NVLink, where time-slicing of the shared GPU is the
only difference.  Results must equal the oracle; statistics must equal the single-GPU run's
(every rank takes the same direction decisions from the global sums)."""
import os

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu
INF = 0xFFFFFFFF


def _check(name, ok, errs):
    if not ok:
        errs.append(name)


def _worker(rank, world, q_id, q_out, case):
    import torch
    import paper_conf_icpp_carocc25_b200 as sg
    from paper_conf_icpp_carocc25_b200.partition import partition_ranges
    torch.cuda.set_device(0)
    errs = []
    try:
        if rank == 0:
            uid = sg.comm_unique_id()
            for _ in range(world - 1):
                q_id.put(uid)
        else:
            uid = q_id.get(timeout=120)
        comm = sg.comm_init(uid, world, rank, 0)
        if case == "bfs":
            g = gen.rmat(14, 16, permute=True)
            G = sg.graph_load_csr(g.row_ptr, g.col_idx, comm=comm)
            Gs = sg.graph_load_csr(g.row_ptr, g.col_idx)                 # single-GPU reference run
            lo, hi = sg.graph_partition(G)
            _check("partition bounds", (lo, hi) == partition_ranges(g.row_ptr, world)[rank], errs)
            roots = list(gen.sources(g, 3)) + [int(np.argmax(g.degrees()))]
            for s in roots:
                ref = oracle.bfs(g, int(s))
                for d in (sg.SG_DIR_AUTO, sg.SG_DIR_PUSH, sg.SG_DIR_PULL):
                    lv, st = sg.run_bfs(G, int(s), direction=d)
                    _check(f"bfs root {s} dir {d}", np.array_equal(sg.as_u32(lv), ref), errs)
                    _, st1 = sg.run_bfs(Gs, int(s), direction=d)
                    # same supersteps as the single-GPU run, except that the single-GPU run may
                    # skip the empty last one (dead-end lookahead, single GPU only)
                    extra = st.iterations - st1.iterations
                    _check(f"bfs stats root {s} dir {d}",
                           st.reached == st1.reached and extra in (0, 1) and
                           st.push_steps >= st1.push_steps and st.pull_steps >= st1.pull_steps and
                           st.push_steps + st.pull_steps == st.iterations, errs)
                lv, _ = sg.run_bfs(G, int(s), owned_only=True)
                _check(f"bfs owned_only root {s}", np.array_equal(sg.as_u32(lv)[lo:hi], ref[lo:hi]), errs)
            os.environ["SG_SPARSE"] = "1"        # fused small supersteps (peer inserts + clear barrier)
            for s in roots[:2]:
                lv, _ = sg.run_bfs(G, int(s))
                _check(f"bfs sparse root {s}", np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s))), errs)
            del os.environ["SG_SPARSE"]
            with pytest.raises(sg.SgError):
                sg.run_bfs(G, 0, host_loop=True)
        elif case == "sssp":
            g = gen.with_weights(gen.rmat(13, 16, permute=True), seed=5)
            G = sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights, comm=comm)
            for s in gen.sources(g, 3):
                d, _ = sg.run_sssp(G, int(s))
                _check(f"sssp {s}", np.array_equal(sg.as_u32(d), oracle.sssp(g, int(s))), errs)
        elif case == "cc":
            for name, g in (("gnm", gen.gnm(60_000, 45_000, seed=3)), ("rmat", gen.rmat(13, 8, permute=True)),
                            ("lattice", gen.lattice(120, 150, 0.55, seed=2))):
                G = sg.graph_load_csr(g.row_ptr, g.col_idx, comm=comm)
                ref = oracle.cc(g)
                for d in (sg.SG_DIR_AUTO, sg.SG_DIR_PUSH, sg.SG_DIR_PULL):
                    lab, _ = sg.run_cc(G, direction=d)
                    _check(f"cc {name} dir {d}", np.array_equal(lab.cpu().numpy(), ref), errs)
                os.environ["SG_CC_LBLOCK_KB"] = "16"                      # label-blocked pull, several blocks
                lab, _ = sg.run_cc(G, direction=sg.SG_DIR_PULL)
                del os.environ["SG_CC_LBLOCK_KB"]
                _check(f"cc {name} blocked", np.array_equal(lab.cpu().numpy(), ref), errs)
                G.free()
        elif case == "tiny":
            # n = 3000 < 4096: one rank owns every vertex, the others own nothing (empty ranges)
            g = gen.rmat(11, 8, permute=True)
            g = gen.from_edges(3000, *[np.asarray(a) for a in _edges_below(g, 3000)])
            G = sg.graph_load_csr(g.row_ptr, g.col_idx, comm=comm)
            lo, hi = sg.graph_partition(G)
            _check("tiny bounds", (lo, hi) == partition_ranges(g.row_ptr, world)[rank], errs)
            for s in gen.sources(g, 2):
                lv, _ = sg.run_bfs(G, int(s))
                _check(f"tiny bfs {s}", np.array_equal(sg.as_u32(lv), oracle.bfs(g, int(s))), errs)
            lab, _ = sg.run_cc(G)
            _check("tiny cc", np.array_equal(lab.cpu().numpy(), oracle.cc(g)), errs)
        torch.cuda.synchronize()
        q_out.put((rank, errs, None))
    except Exception as e:   # report instead of hanging the parent
        import traceback
        q_out.put((rank, errs, traceback.format_exc()[-1500:]))


def _edges_below(g, n):
    rows = np.repeat(np.arange(g.n), g.degrees())
    keep = (rows < n) & (g.col_idx < n) & (rows < g.col_idx)
    return rows[keep], g.col_idx[keep].astype(np.int64)


@pytest.mark.parametrize("world,case", [(2, "bfs"), (3, "bfs"), (2, "sssp"), (3, "sssp"), (2, "cc"), (3, "cc"),
                                        (2, "tiny"), (4, "tiny")])
def test_partitioned_ranks_on_one_gpu(world, case):
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    q_id, q_out = ctx.Queue(), ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, q_id, q_out, case)) for r in range(world)]
    for p in ps:
        p.start()
    res = []
    try:
        for _ in ps:
            res.append(q_out.get(timeout=600))
    finally:
        for p in ps:
            p.join(timeout=120)
            if p.exitcode is None:
                p.kill()
    for rank, errs, tb in sorted(res, key=lambda r: r[0]):
        assert tb is None, f"rank {rank} raised:\n{tb}"
        assert not errs, f"rank {rank}: {errs}"
