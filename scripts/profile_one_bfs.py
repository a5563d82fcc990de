"""Run one BFS on config 4 (for ncu captures of single kernels).

    python scripts/profile_one_bfs.py [push|pull|auto] [root_index]

Under ncu, select the launch with -k regex:<kernel> -s <skip> -c 1 (e.g. the level-3 push in
push-only mode is the 4th k_push_words launch: -s 3)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "auto"
ri = int(sys.argv[2]) if len(sys.argv) > 2 else 0
cfg = int(os.environ.get("SG_CONFIG", "4"))
g = gen.make_config_graph(cfg)
roots = gen.config_sources(cfg, g)
G = sg.graph_load_csr(g.row_ptr, g.col_idx)
d = {"push": sg.SG_DIR_PUSH, "pull": sg.SG_DIR_PULL, "auto": sg.SG_DIR_AUTO}[mode]
seg = int(os.environ.get("SG_SEGMENTED", "0"))
alpha = float(os.environ.get("SG_ALPHA", "14"))
# host-driven loop: ncu cannot profile kernels inside graphs with conditional nodes
lv, st = sg.run_bfs(G, int(roots[ri]), direction=d, host_loop=True, segmented=seg, alpha=alpha)
torch.cuda.synchronize()
print(st.as_dict())
