"""Median device time of C2 SSSP (graph-driven) and C3 CC over a few runs: python scripts/micro/sssp_time.py"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

g = gen.make_config_graph(2)
G = sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights)
d = torch.empty(g.n, dtype=torch.int32, device="cuda")
for s in (0, int(gen.config_sources(2, g)[0])):
    for _ in range(3):
        sg.run_sssp(G, s, d)
    sts = [sg.run_sssp(G, s, d)[1] for _ in range(10)]
    ts = [st.device_ms for st in sts]
    print(f"C2 SSSP from {s}: {statistics.median(ts):.3f} ms (min {min(ts):.3f} max {max(ts):.3f}), "
          f"{sts[-1].iterations} supersteps, {sts[-1].arcs_pushed} arcs", flush=True)
