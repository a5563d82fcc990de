"""Wall-clock parts of one end-to-end BFS step on config 4 (graph_load_csr from pinned host
memory, first run_bfs on the fresh graph, a second run_bfs, graph free).

    python scripts/e2e_parts.py [reps] [--resident]   (--resident: another graph stays loaded, as in bench.py)"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 3
g = gen.make_config_graph(4)
roots = gen.config_sources(4, g)
rp_h = torch.from_numpy(g.row_ptr).pin_memory()
ci_h = torch.from_numpy(g.col_idx).pin_memory()
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
stream = torch.cuda.current_stream()
keep = sg.graph_load_csr(rp_h, ci_h, stream=stream) if "--resident" in sys.argv else None   # as in bench.py
for r in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    G = sg.graph_load_csr(rp_h, ci_h, stream=stream)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    sg.run_bfs(G, int(roots[0]), lv)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    sg.run_bfs(G, int(roots[1]), lv)
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    G.free()
    torch.cuda.synchronize()
    t4 = time.perf_counter()
    print(f"load {1e3*(t1-t0):.1f} ms  first bfs {1e3*(t2-t1):.1f} ms  second bfs {1e3*(t3-t2):.2f} ms  free {1e3*(t4-t3):.1f} ms", flush=True)
