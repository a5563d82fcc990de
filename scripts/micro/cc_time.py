"""Median device time of C3 CC (graph-driven, label-blocked pulls): python scripts/micro/cc_time.py"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

g = gen.make_config_graph(3)
G = sg.graph_load_csr(g.row_ptr, g.col_idx)
lab = torch.empty(g.n, dtype=torch.int32, device="cuda")
for _ in range(2):
    sg.run_cc(G, lab)
ts = [sg.run_cc(G, lab)[1].device_ms for _ in range(8)]
print(f"C3 CC {statistics.median(ts):.3f} ms (min {min(ts):.3f})", flush=True)
