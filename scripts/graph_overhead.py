"""Graph-mode BFS device time for one root vs the same BFS in the host-driven loop (config 4).

    python scripts/graph_overhead.py [root_index] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

ri = int(sys.argv[1]) if len(sys.argv) > 1 else 0
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
g = gen.make_config_graph(4)
roots = gen.config_sources(4, g)
G = sg.graph_load_csr(g.row_ptr, g.col_idx)
r = int(roots[ri])
for mode in ("graph", "host"):
    ts = []
    for i in range(reps + 2):
        lv, st = sg.run_bfs(G, r, direction=sg.SG_DIR_AUTO, host_loop=(mode == "host"))
        torch.cuda.synchronize()
        ts.append(st.as_dict()["device_ms"])
    ts = sorted(ts[2:])
    print(mode, "median ms", round(ts[len(ts) // 2], 4), "min", round(ts[0], 4), st.as_dict()["iterations"])
