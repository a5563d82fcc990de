"""Repro helper: BFS with the segmented hub tier forced, on RMAT-21 (3 segments)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 21
g = gen.rmat(scale, 8, permute=True)
G = sg.graph_load_csr(g.row_ptr, g.col_idx)
s = int(gen.sources(g, 1)[0])
lv, st = sg.run_bfs(G, s, direction=sg.SG_DIR_PUSH, segmented=2, host_loop=True)
print("match", np.array_equal(sg.as_u32(lv), oracle.bfs(g, s)), st.as_dict())
