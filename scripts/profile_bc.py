"""One 32-source batch of BC on config 5 (for ncu captures of the cooperative kernels)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

g = gen.make_config_graph(5)
G = sg.graph_load_csr(g.row_ptr, g.col_idx)
srcs = gen.config_sources(5, g)[:32]
bc, st = sg.run_bc(G, srcs)
torch.cuda.synchronize()
print(st.as_dict())
