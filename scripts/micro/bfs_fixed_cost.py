"""Fixed cost of one device-driven BFS outside its supersteps: run_bfs on edgeless graphs (the
BFS stops at once: 0 supersteps), so device_ms = control-block copies + prologue (level pass
over n vertices, frontier / visited initialisation) + graph launch.
    python scripts/micro/bfs_fixed_cost.py"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

for n in (64, 1 << 20, 1 << 24):
    g = gen.empty_graph(n)
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    lv = torch.empty(n, dtype=torch.int32, device="cuda")
    for _ in range(3):
        sg.run_bfs(G, 0, lv)
    ts = [sg.run_bfs(G, 0, lv)[1].device_ms * 1e3 for _ in range(20)]
    _, st = sg.run_bfs(G, 0, lv)
    print(f"n = {n:9d}: {statistics.median(ts):7.1f} us per BFS (min {min(ts):.1f}), {st.iterations} supersteps", flush=True)
