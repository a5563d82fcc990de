"""B200 re-run of the paper's Fig. 7 ablation (§5.1).

The paper measures BFS on Indochina-2004 (7.4M vertices, 194M edges, web graph) with a plain
bitmap, then +MSI (subgroup = word), +CF (coarsening), +2LB, and all of them (4.43x on V100S).
Here: a synthetic stand-in with that shape (R-MAT scale 23, edge factor 12, unpermuted: ~190M arcs,
skewed degrees, id locality) and config 4, push-only BFS like the paper's, adding the B200 design
steps one at a time.  Every variant's levels are checked against the first variant's.

    python scripts/ablation.py [--roots 4]   -> one JSON line per (graph, variant)
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

BIG = 1 << 30
VARIANTS = [
    ("plain bitmap (1 layer, warp per word, CF=1)",
     dict(one_layer=True, small_degree=-1, heavy_degree=BIG, segmented=1, coarsening=1, host_loop=True,
          direction=sg.SG_DIR_PUSH)),
    ("+ coarsening (auto CF)",
     dict(one_layer=True, small_degree=-1, heavy_degree=BIG, segmented=1, host_loop=True, direction=sg.SG_DIR_PUSH)),
    ("+ 2LB (summary-layer compaction)",
     dict(small_degree=-1, heavy_degree=BIG, segmented=1, host_loop=True, direction=sg.SG_DIR_PUSH)),
    ("+ degree tiers (thread / warp / TMA CTA-grid)",
     dict(segmented=1, host_loop=True, direction=sg.SG_DIR_PUSH)),
    ("+ segmented hub tier (visited slice in smem)",
     dict(segmented=0, host_loop=True, direction=sg.SG_DIR_PUSH)),
    ("+ device-driven loop (CUDA graph)",
     dict(segmented=0, direction=sg.SG_DIR_PUSH)),
    ("+ direction optimisation (all, default)",
     dict()),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--roots", type=int, default=4)
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    graphs = [("rmat23_ef12 (Indochina-shaped)", lambda: gen.rmat(23, 12, permute=False)),
              ("config4 kron24_ef32", lambda: gen.make_config_graph(4))]
    for gname, mk in graphs:
        g = mk()
        G = sg.graph_load_csr(g.row_ptr, g.col_idx)
        roots = gen.sources(g, args.roots)
        deg = g.degrees()
        level = torch.empty(g.n, dtype=torch.int32, device="cuda")
        ref = {}
        base = None
        for name, kw in VARIANTS:
            o = sg.opts(**kw)
            times, teps = [], []
            for s in roots:
                sg.run_bfs(G, int(s), level, o)            # warm-up / graph build
                st = None
                t = []
                for _ in range(args.reps):
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record()
                    _, st = sg.run_bfs(G, int(s), level, o)
                    b.record()
                    torch.cuda.synchronize()
                    t.append(a.elapsed_time(b))
                lv = sg.as_u32(level)
                if int(s) not in ref:
                    ref[int(s)] = lv.copy()
                assert np.array_equal(lv, ref[int(s)]), (name, s)
                ms = statistics.median(t)
                times.append(ms)
                teps.append(int(deg[lv != 0xFFFFFFFF].sum()) // 2 / (ms / 1e3) / 1e9)
            ms = statistics.median(times)
            base = base or ms
            print(json.dumps({"graph": gname, "n": g.n, "nnz": g.nnz, "variant": name, "ms_per_bfs": ms,
                              "gteps": statistics.median(teps), "speedup_vs_plain": base / ms}), flush=True)
        # word width (§4.3: 32-bit words "to match a warp on NVIDIA"): the self-contained
        # push-only 2LB BFS of ablate.cu with 32- and 64-bit words, otherwise identical
        for wb in (32, 64):
            times, teps = [], []
            for s in roots:
                sg.ablation_bfs(G, int(s), wb, level)
                t = []
                for _ in range(args.reps):
                    _, st = sg.ablation_bfs(G, int(s), wb, level)
                    t.append(st.device_ms)
                lv = sg.as_u32(level)
                assert np.array_equal(lv, ref[int(s)]), ("word", wb, s)
                ms = statistics.median(t)
                times.append(ms)
                teps.append(int(deg[lv != 0xFFFFFFFF].sum()) // 2 / (ms / 1e3) / 1e9)
            print(json.dumps({"graph": gname, "n": g.n, "nnz": g.nnz,
                              "variant": f"word-width ablation: {wb}-bit words, paper mapping (warp per word, "
                                         f"lanes stride the list), 2LB, push-only, host loop",
                              "ms_per_bfs": statistics.median(times), "gteps": statistics.median(teps)}), flush=True)
        del G


if __name__ == "__main__":
    main()
