"""Host-side cost of a graph load / first BFS / free cycle (the e2e bench step without the
H2D time dominating): config-2 and config-4 graphs, 3 cycles each.
    python scripts/micro/load_cycle.py"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

for cfg in (2, 4):
    g = gen.make_config_graph(cfg)
    rp = torch.from_numpy(g.row_ptr).pin_memory()
    ci = torch.from_numpy(g.col_idx).pin_memory()
    lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
    s = int(gen.config_sources(cfg, g)[0])
    for i in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        G = sg.graph_load_csr(rp, ci)
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        sg.run_bfs(G, s, lv)
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        sg.run_bfs(G, s, lv)
        torch.cuda.synchronize()
        t3 = time.perf_counter()
        G.free()
        torch.cuda.synchronize()
        t4 = time.perf_counter()
        print(f"config {cfg} cycle {i}: load {1e3 * (t1 - t0):8.1f} ms, first BFS {1e3 * (t2 - t1):8.1f} ms, "
              f"second {1e3 * (t3 - t2):7.2f} ms, free {1e3 * (t4 - t3):7.1f} ms", flush=True)
