"""Fixed cost of one device-driven BFS superstep: BFS on a path graph (one vertex per level, so
every superstep is pure overhead), per-superstep device time from sg_bfs_trace.
    python scripts/micro/superstep_overhead.py [n] [--env K=V ...]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 64
envs = [a for a in sys.argv[1:] if "=" in a] or [""]
for big in (False, True):
    g = gen.path(n) if not big else gen.from_edges(1 << 24, list(range(n - 1)), list(range(1, n)))
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
    for env in envs:
        saved = dict(os.environ)
        for kv in filter(None, env.split(",")):
            k, _, v = kv.partition("=")
            os.environ[k] = v
        for _ in range(3):
            sg.run_bfs(G, 0, lv)
        us = []
        for _ in range(5):
            _, st = sg.run_bfs(G, 0, lv)
            tr = sg.bfs_trace(G)
            us += [t["us"] for t in tr[1:-1]]
        kinds = sorted({t["kind"] for t in tr})
        print(f"n_vertices={g.n:9d} {env or 'default':22s} kinds {kinds}: median {statistics.median(us):.2f} us "
              f"per superstep (min {min(us):.2f}), BFS {st.device_ms * 1e3:.1f} us for {st.iterations} supersteps",
              flush=True)
        os.environ.clear()
        os.environ.update(saved)
