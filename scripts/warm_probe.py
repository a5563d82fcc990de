"""Repeatedly time 20 graph-mode BFS (C4) in one process for ~60 s: is a fresh box slow at first?

    python scripts/warm_probe.py [seconds]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

T = float(sys.argv[1]) if len(sys.argv) > 1 else 60.0
t0 = time.time()
g = gen.make_config_graph(4)
roots = gen.config_sources(4, g)
G = sg.graph_load_csr(g.row_ptr, g.col_idx)
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
print("setup s", round(time.time() - t0, 1), flush=True)
t1 = time.time()
while time.time() - t1 < T:
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for r in roots[:20]:
        sg.run_bfs(G, int(r), level=lv, direction=sg.SG_DIR_AUTO)
    e1.record()
    torch.cuda.synchronize()
    print(round(time.time() - t1, 1), "ms/BFS", round(e0.elapsed_time(e1) / 20, 4), flush=True)
