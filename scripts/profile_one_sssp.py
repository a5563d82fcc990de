"""Run one SSSP on config 2 (for ncu launch lists): python scripts/profile_one_sssp.py [reps]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 1
host = "host" in sys.argv[2:]   # host-driven loop (ncu cannot profile kernels inside conditional graph nodes)
g = gen.make_config_graph(2)
src = int(gen.config_sources(2, g)[0])
G = sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights)
for r in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    d, st = sg.run_sssp(G, src, host_loop=host)
    torch.cuda.synchronize()
    print(round(1e3 * (time.perf_counter() - t0), 3), "ms wall", st.as_dict())
